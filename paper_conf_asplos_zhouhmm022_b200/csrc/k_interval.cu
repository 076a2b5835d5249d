// k_interval.cu -- SURVEY 8(f) f1: accessed intervals, their parallel merge and the
// adaptive copy plan (section 6.1, Figures 4 and 5).
//
// The paper merges the [start, end] intervals a kernel's instructions access when
// they are "adjacent or overlapped", on the GPU: sort the end points,
// +1/-1 markers, a prefix scan, start / end flags, two more scans and a scatter
// (Figure 4), after a warp-level "interval compaction".  The
// B200 design keeps the compaction and the sort but merges with one scan pair
// over intervals sorted by start instead of 2N marker end points:
//   M_i   = max(end_0 .. end_{i-1})                       (exclusive max scan)
//   f_i   = i == 0 || start_i > M_i + 1                   (i opens a merged interval)
//   g_i   = f_0 + .. + f_i - 1                            (its output index)
//   out[g_i].start = start_i if f_i;  out[g_i - 1].end = M_i if f_i and i > 0;
//   out[last].end = max(M_{n-1}, end_{n-1}).
// A marker prefix sum over the sorted end points is 0 exactly where M_i + 1 <
// start_i, so both give the same merged set (the definition, C13).
//
//   k_iv_in / k_iv_rec   warp compaction of the input (or record) intervals -> SoA (S, E)
//   k_iv_range           min / max start and the number of descents (sorted input: no sort)
//   k_rs_hist/_scatter   stable LSD radix sort of (S, E) by S - min, 8-bit digits over the
//                        varying bits only; block-local ranking with __match_any_sync
//   k_iv_tile_max, k_iv_merge<false/true>   the merge scans above (tile carries between)
//   k_iv_plan            per-object clipping of the merged set for the copy plan
//
// All integer; the result is unique, so parity with the oracle is bit-exact.
#include <algorithm>

#include "ve_internal.cuh"

namespace ve {

constexpr int IV_T = 256;                  // threads per block
constexpr int IV_ITEMS = 8;                // items per thread
constexpr int IV_TILE = IV_T * IV_ITEMS;   // items per tile (block)
constexpr int IV_NW = IV_T / 32;
constexpr unsigned FULLM = 0xFFFFFFFFu;

// ---- warp interval compaction ---------------------------------------------
// Lane i joins lane i-1's run when both hold intervals and start_i lies in
// [start_{i-1}, end_{i-1} + 1]; a run is then the single interval [start_head, max end]
// (every member starts inside the union of its predecessors).  Returns true on the
// lane that emits its run's interval (the run's last lane) with it in (s, e).
__device__ __forceinline__ bool warp_compact(bool ok, uint64_t& s, uint64_t& e) {
  const int lane = threadIdx.x & 31;
  const uint64_t ps = __shfl_up_sync(FULLM, s, 1), pe = __shfl_up_sync(FULLM, e, 1);
  const bool pok = __shfl_up_sync(FULLM, (int)ok, 1) != 0;
  const bool join = ok && lane > 0 && pok && s >= ps && (pe == ~0ull || s <= pe + 1);
  bool f = !join;               // segment heads (lanes without an interval are their own segment)
  uint64_t hs = s, me = e;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {   // segmented inclusive scan: (head start, max end)
    const uint64_t hs2 = __shfl_up_sync(FULLM, hs, d), me2 = __shfl_up_sync(FULLM, me, d);
    const bool f2 = __shfl_up_sync(FULLM, (int)f, d) != 0;
    if (lane >= d) {
      if (!f) { hs = hs2; me = me2 > me ? me2 : me; }
      f = f || f2;
    }
  }
  const bool next_join = __shfl_down_sync(FULLM, (int)join, 1) != 0 && lane < 31;
  s = hs;
  e = me;
  return ok && !next_join;
}

// Emitted intervals collect in a per-warp shared buffer and go to (S, E) 32+ at a
// time with one global claim (a claim per window would serialise ~N/32 atomics on
// one counter).  n is warp-uniform; the buffer never holds more than 63 entries.
constexpr int WB = 64;
struct WarpBuf {
  uint64_t s[WB], e[WB];
};

__device__ __forceinline__ void wb_flush(WarpBuf& b, uint32_t& n, uint64_t* S, uint64_t* E,
                                         unsigned long long* cnt) {
  const int lane = threadIdx.x & 31;
  if (n == 0) return;
  unsigned long long base = 0;
  if (lane == 0) base = atomicAdd(cnt, (unsigned long long)n);
  base = __shfl_sync(FULLM, base, 0);
  for (uint32_t i = lane; i < n; i += 32) {
    S[base + i] = b.s[i];
    E[base + i] = b.e[i];
  }
  __syncwarp();
  n = 0;
}

__device__ __forceinline__ void wb_append(WarpBuf& b, uint32_t& n, bool emit, uint64_t s, uint64_t e, uint64_t* S,
                                          uint64_t* E, unsigned long long* cnt) {
  const int lane = threadIdx.x & 31;
  const unsigned m = __ballot_sync(FULLM, emit);
  if (emit) {
    const uint32_t p = n + __popc(m & ((1u << lane) - 1u));
    b.s[p] = s;
    b.e[p] = e;
  }
  n += __popc(m);
  __syncwarp();
  if (n >= 32) wb_flush(b, n, S, E, cnt);
}

__global__ void __launch_bounds__(IV_T) k_iv_in(const ve_interval* in, uint64_t n, uint64_t* S, uint64_t* E,
                                                unsigned long long* cnt) {
  __shared__ WarpBuf wbuf[IV_NW];
  WarpBuf& b = wbuf[threadIdx.x >> 5];
  uint32_t bn = 0;
  const uint64_t nw = (n + 31) / 32, stride = (uint64_t)gridDim.x * IV_NW;
  for (uint64_t w = (uint64_t)blockIdx.x * IV_NW + (threadIdx.x >> 5); w < nw; w += stride) {
    const uint64_t i = w * 32 + (threadIdx.x & 31);
    uint64_t s = 1, e = 0;
    if (i < n) { s = in[i].start; e = in[i].end; }
    const bool ok = i < n && s <= e;      // start > end: the empty set (R1)
    const bool emit = warp_compact(ok, s, e);
    wb_append(b, bn, emit, s, e, S, E, cnt);
  }
  wb_flush(b, bn, S, E, cnt);
}

__global__ void __launch_bounds__(IV_T) k_iv_rec(const ve_record* r, uint64_t n, uint32_t n_pcs, uint64_t* S,
                                                 uint64_t* E, unsigned long long* cnt) {
  __shared__ WarpBuf wbuf[IV_NW];
  WarpBuf& b = wbuf[threadIdx.x >> 5];
  uint32_t bn = 0;
  const uint64_t nw = (n + 31) / 32, stride = (uint64_t)gridDim.x * IV_NW;
  // IV_U windows per iteration, their 3 x IV_U loads issued before any is used (2.94 -> 2.84 ms on
  // the cfg2 gemm epoch)
  constexpr int IV_U = 4;
  for (uint64_t w0 = (uint64_t)blockIdx.x * IV_NW + (threadIdx.x >> 5); w0 < nw; w0 += IV_U * stride) {
    uint64_t ad[IV_U], va[IV_U], pmv[IV_U];
#pragma unroll
    for (int u = 0; u < IV_U; ++u) {
      const uint64_t i = (w0 + u * stride) * 32 + (threadIdx.x & 31);
      ad[u] = va[u] = 0;
      pmv[u] = ~0ull;                        // (an absent record: invalid pc)
      if (w0 + u * stride < nw && i < n) {
        const unsigned long long* q = reinterpret_cast<const unsigned long long*>(&r[i]);
        ad[u] = __ldcs(q); va[u] = __ldcs(q + 1); pmv[u] = __ldcs(q + 2);
      }
    }
#pragma unroll
    for (int u = 0; u < IV_U; ++u) {
      if (w0 + u * stride >= nw) break;      // (warp-uniform)
      const uint64_t i = (w0 + u * stride) * 32 + (threadIdx.x & 31);
      uint64_t s = 0, e = 0;
      bool ok = false;
      if (i < n) {
        const uint32_t pc = (uint32_t)pmv[u], meta = (uint32_t)(pmv[u] >> 32);
        ok = rec_valid(ad[u], va[u], pc, meta, n_pcs) && !meta_shared(meta);   // R2
        s = ad[u];
        e = ad[u] + (1ull << meta_lg(meta)) - 1ull;
      }
      const bool emit = warp_compact(ok, s, e);
      wb_append(b, bn, emit, s, e, S, E, cnt);
    }
  }
  wb_flush(b, bn, S, E, cnt);
}

// out[0] = min start, out[1] = max start, out[2] = number of i with S[i] < S[i-1]
__global__ void __launch_bounds__(IV_T) k_iv_range(const uint64_t* S, uint64_t n, unsigned long long* out) {
  uint64_t mn = ~0ull, mx = 0, dsc = 0;
  for (uint64_t i = (uint64_t)blockIdx.x * IV_T + threadIdx.x; i < n; i += (uint64_t)gridDim.x * IV_T) {
    const uint64_t v = S[i];
    mn = v < mn ? v : mn;
    mx = v > mx ? v : mx;
    if (i > 0 && v < S[i - 1]) ++dsc;
  }
  for (int o = 16; o; o >>= 1) {
    const uint64_t a = __shfl_xor_sync(FULLM, mn, o), b = __shfl_xor_sync(FULLM, mx, o);
    mn = a < mn ? a : mn;
    mx = b > mx ? b : mx;
    dsc += __shfl_xor_sync(FULLM, dsc, o);
  }
  if ((threadIdx.x & 31) == 0) {
    atomicMin(&out[0], (unsigned long long)mn);
    atomicMax(&out[1], (unsigned long long)mx);
    if (dsc) atomicAdd(&out[2], (unsigned long long)dsc);
  }
}

// ---- stable LSD radix sort of (S, E) by key S - kmin ---------------------------------
// Tile b holds items [b*IV_TILE, (b+1)*IV_TILE); warp w of the tile takes the
// IV_ITEMS*32 consecutive items from w*IV_ITEMS*32, row by row (row j = 32 consecutive
// items), so (warp, row, lane) order is the item order and ranks stay stable.
__device__ __forceinline__ uint32_t rs_digit(uint64_t s, uint64_t kmin, uint32_t shift) {
  return (uint32_t)(((s - kmin) >> shift) & 255u);
}

// hist[d * nblk + b] = items of tile b with digit d
__global__ void __launch_bounds__(IV_T) k_rs_hist(const uint64_t* S, uint64_t n, uint64_t kmin, uint32_t shift,
                                                  uint32_t* hist, uint32_t nblk) {
  __shared__ uint32_t h[256];
  h[threadIdx.x] = 0;
  __syncthreads();
  const uint64_t t0 = (uint64_t)blockIdx.x * IV_TILE;
#pragma unroll
  for (int j = 0; j < IV_ITEMS; ++j) {
    const uint64_t i = t0 + (uint64_t)j * IV_T + threadIdx.x;
    if (i < n) atomicAdd(&h[rs_digit(S[i], kmin, shift)], 1u);
  }
  __syncthreads();
  hist[(uint64_t)threadIdx.x * nblk + blockIdx.x] = h[threadIdx.x];
}

__global__ void __launch_bounds__(IV_T) k_rs_scatter(const uint64_t* __restrict__ Si, const uint64_t* __restrict__ Ei,
                                                     uint64_t n, uint64_t kmin, uint32_t shift,
                                                     const uint32_t* __restrict__ off, uint32_t nblk,
                                                     uint64_t* __restrict__ So, uint64_t* __restrict__ Eo) {
  __shared__ uint32_t wc[IV_NW][256];   // per-warp digit counts, then per-warp digit offsets
  __shared__ uint32_t go[256];          // global offset of (digit, tile)
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int d = lane; d < 256; d += 32) wc[w][d] = 0;
  go[threadIdx.x] = off[(uint64_t)threadIdx.x * nblk + blockIdx.x];
  __syncwarp();
  const uint64_t wb = (uint64_t)blockIdx.x * IV_TILE + (uint64_t)w * IV_ITEMS * 32;
  uint64_t s[IV_ITEMS], e[IV_ITEMS];
  uint32_t rk[IV_ITEMS], dg[IV_ITEMS];
#pragma unroll
  for (int j = 0; j < IV_ITEMS; ++j) {
    const uint64_t i = wb + (uint64_t)j * 32 + lane;
    const bool v = i < n;
    s[j] = v ? Si[i] : 0;
    e[j] = v ? Ei[i] : 0;
    dg[j] = v ? rs_digit(s[j], kmin, shift) : 256u;
    const unsigned act = __ballot_sync(FULLM, v);
    rk[j] = 0;
    if (v) {
      const unsigned peers = __match_any_sync(act, dg[j]);
      const int leader = __ffs(peers) - 1;
      uint32_t base = 0;
      if (lane == leader) {
        base = wc[w][dg[j]];
        wc[w][dg[j]] = base + (uint32_t)__popc(peers);
      }
      base = __shfl_sync(peers, base, leader);
      rk[j] = base + (uint32_t)__popc(peers & ((1u << lane) - 1u));
    }
    __syncwarp();
  }
  __syncthreads();
  // per digit: exclusive prefix over the warps of the tile, and the tile-local start of
  // the digit (exclusive scan of the digit totals over the 256 threads)
  __shared__ uint32_t ls[256];
  __shared__ uint32_t wsum[IV_NW];
  {
    const int d = threadIdx.x;
    uint32_t run = 0;
    for (int k = 0; k < IV_NW; ++k) {
      const uint32_t c = wc[k][d];
      wc[k][d] = run;
      run += c;
    }
    uint32_t x = run;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(FULLM, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) wsum[w] = x;
    __syncthreads();
    uint32_t pre = 0;
    for (int k = 0; k < w; ++k) pre += wsum[k];
    ls[d] = pre + x - run;
  }
  __syncthreads();
  // stage the tile in shared memory in (digit, rank) order, then write every digit's run
  // out contiguously: consecutive threads store consecutive addresses
  __shared__ uint64_t sk[IV_TILE], sv[IV_TILE];
#pragma unroll
  for (int j = 0; j < IV_ITEMS; ++j) {
    if (dg[j] < 256u) {
      const uint32_t lp = ls[dg[j]] + wc[w][dg[j]] + rk[j];
      sk[lp] = s[j];
      sv[lp] = e[j];
    }
  }
  __syncthreads();
  const uint64_t t0 = (uint64_t)blockIdx.x * IV_TILE;
  const uint32_t nv = (uint32_t)(n - t0 < (uint64_t)IV_TILE ? n - t0 : (uint64_t)IV_TILE);
  for (uint32_t idx = threadIdx.x; idx < nv; idx += IV_T) {
    const uint64_t key = sk[idx];
    const uint32_t d = rs_digit(key, kmin, shift);
    const uint64_t p = (uint64_t)go[d] + (idx - ls[d]);
    So[p] = key;
    Eo[p] = sv[idx];
  }
}

// ---- exclusive scans (u32 sums, u64 max) ------------------------------------------------
template <typename T, typename Op>
__device__ __forceinline__ T block_excl_scan(T v, Op op, T id, T* sm, T& total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  T x = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const T y = __shfl_up_sync(FULLM, x, d);
    if (lane >= d) x = op(y, x);
  }
  if (lane == 31) sm[w] = x;
  __syncthreads();
  T pre = id, tot = id;
#pragma unroll
  for (int k = 0; k < IV_NW; ++k) {
    const T z = sm[k];
    if (k < w) pre = op(pre, z);
    tot = op(tot, z);
  }
  __syncthreads();
  T ex = __shfl_up_sync(FULLM, x, 1);
  if (lane == 0) ex = id;
  total = tot;
  return op(pre, ex);
}
struct OpAdd { __device__ uint32_t operator()(uint32_t a, uint32_t b) const { return a + b; } };
struct OpMax { __device__ uint64_t operator()(uint64_t a, uint64_t b) const { return a > b ? a : b; } };

// one block: in-place exclusive sum scan of a[0..n)
__global__ void __launch_bounds__(IV_T) k_scan_sum_1(uint32_t* a, uint64_t n) {
  __shared__ uint32_t sm[IV_NW];
  uint32_t carry = 0;
  for (uint64_t b = 0; b < n; b += IV_T) {
    const uint64_t i = b + threadIdx.x;
    const uint32_t v = i < n ? a[i] : 0u;
    uint32_t tot;
    const uint32_t ex = block_excl_scan(v, OpAdd(), 0u, sm, tot);
    if (i < n) a[i] = carry + ex;
    carry += tot;
  }
}
// one block: in-place exclusive max scan of a[0..n) (identity 0; a[0] becomes 0)
__global__ void __launch_bounds__(IV_T) k_scan_max_1(unsigned long long* a, uint64_t n) {
  __shared__ uint64_t sm[IV_NW];
  uint64_t carry = 0;
  for (uint64_t b = 0; b < n; b += IV_T) {
    const uint64_t i = b + threadIdx.x;
    const uint64_t v = i < n ? a[i] : 0ull;
    uint64_t tot;
    const uint64_t ex = block_excl_scan<uint64_t>(v, OpMax(), 0ull, sm, tot);
    if (i < n) a[i] = carry > ex ? carry : ex;
    carry = carry > tot ? carry : tot;
  }
}

// large exclusive sum scan: per-block totals, a 1-block scan of them, then per-block apply
constexpr uint64_t SC_TILE = (uint64_t)IV_T * 16;
__global__ void __launch_bounds__(IV_T) k_scan_part(const uint32_t* a, uint64_t n, uint32_t* part) {
  __shared__ uint32_t sm[IV_NW];
  const uint64_t b0 = (uint64_t)blockIdx.x * SC_TILE;
  uint32_t acc = 0;
  for (uint64_t i = b0 + threadIdx.x; i < b0 + SC_TILE && i < n; i += IV_T) acc += a[i];
  uint32_t tot;
  block_excl_scan(acc, OpAdd(), 0u, sm, tot);
  if (threadIdx.x == 0) part[blockIdx.x] = tot;
}
__global__ void __launch_bounds__(IV_T) k_scan_apply(uint32_t* a, uint64_t n, const uint32_t* part) {
  __shared__ uint32_t sm[IV_NW];
  const uint64_t b0 = (uint64_t)blockIdx.x * SC_TILE;
  uint32_t carry = part[blockIdx.x];
  for (uint64_t r = b0; r < b0 + SC_TILE && r < n; r += IV_T) {
    const uint64_t i = r + threadIdx.x;
    const uint32_t v = i < n ? a[i] : 0u;
    uint32_t tot;
    const uint32_t ex = block_excl_scan(v, OpAdd(), 0u, sm, tot);
    if (i < n) a[i] = carry + ex;
    carry += tot;
  }
}

// ---- the merge over sorted (S, E) -------------------------------------------------------
__global__ void __launch_bounds__(IV_T) k_iv_tile_max(const uint64_t* E, uint64_t n, unsigned long long* tmax) {
  const uint64_t t0 = (uint64_t)blockIdx.x * IV_TILE;
  uint64_t m = 0;
  for (int j = 0; j < IV_ITEMS; ++j) {
    const uint64_t i = t0 + (uint64_t)j * IV_T + threadIdx.x;
    if (i < n) m = E[i] > m ? E[i] : m;
  }
  for (int o = 16; o; o >>= 1) {
    const uint64_t y = __shfl_xor_sync(FULLM, m, o);
    m = y > m ? y : m;
  }
  __shared__ uint64_t sm[IV_NW];
  if ((threadIdx.x & 31) == 0) sm[threadIdx.x >> 5] = m;
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int k = 1; k < IV_NW; ++k) m = sm[k] > m ? sm[k] : m;
    tmax[blockIdx.x] = m > sm[0] ? m : sm[0];
  }
}

// Walk a tile in item order (rows of IV_T): Mi = exclusive max of E (carry tcarry from the
// tiles before), fi = i == 0 || S_i > Mi + 1.  EMIT = false: count the flags into fcnt[b];
// EMIT = true: write the merged intervals (foff = flags before the tile).
template <bool EMIT>
__global__ void __launch_bounds__(IV_T) k_iv_merge(const uint64_t* __restrict__ S, const uint64_t* __restrict__ E,
                                                   uint64_t n, const unsigned long long* __restrict__ tcarry,
                                                   uint32_t* __restrict__ fcnt, const uint32_t* __restrict__ foff,
                                                   ve_interval* __restrict__ out) {
  __shared__ uint64_t smx[IV_NW];
  __shared__ uint32_t ssm[IV_NW];
  const uint64_t t0 = (uint64_t)blockIdx.x * IV_TILE;
  uint64_t carry = tcarry[blockIdx.x];
  uint32_t fc = EMIT ? foff[blockIdx.x] : 0u;   // flags before this row
  for (int j = 0; j < IV_ITEMS; ++j) {
    const uint64_t i = t0 + (uint64_t)j * IV_T + threadIdx.x;
    const bool v = i < n;
    const uint64_t s = v ? S[i] : 0ull, e = v ? E[i] : 0ull;
    uint64_t tmx;
    const uint64_t ex = block_excl_scan<uint64_t>(e, OpMax(), 0ull, smx, tmx);
    const uint64_t M = carry > ex ? carry : ex;
    const bool f = v && (i == 0 || (M != ~0ull && s > M + 1));
    uint32_t tf;
    const uint32_t fx = block_excl_scan(f ? 1u : 0u, OpAdd(), 0u, ssm, tf);
    if (EMIT && v) {
      const uint64_t g = (uint64_t)fc + fx + (f ? 1u : 0u);   // flags in [0, i]
      if (f) {
        out[g - 1].start = s;
        if (i > 0) out[g - 2].end = M;
      }
      if (i == n - 1) out[g - 1].end = M > e ? M : e;
    }
    fc += tf;
    carry = carry > tmx ? carry : tmx;
  }
  if (!EMIT && threadIdx.x == 0) fcnt[blockIdx.x] = fc;
}

// ---- copy plan: clip the merged set to every object (objects sorted by base) -------------
// acc[j] = {n_segments, accessed bytes, lo (min), hi (max)} of sorted object j; bad[0] != 0
// if the input is not sorted, disjoint and non-adjacent.
__global__ void __launch_bounds__(IV_T) k_iv_plan(const ve_interval* m, uint64_t n, const uint64_t* ob,
                                                  const uint64_t* oe, uint32_t nobj, unsigned long long* acc,
                                                  unsigned int* bad) {
  for (uint64_t i = (uint64_t)blockIdx.x * IV_T + threadIdx.x; i < n; i += (uint64_t)gridDim.x * IV_T) {
    const uint64_t s = m[i].start, e = m[i].end;
    if (s > e || (i > 0 && (m[i - 1].end == ~0ull || s <= m[i - 1].end + 1))) atomicOr(bad, 1u);
    uint32_t lo = 0, hi = nobj;      // first object with end > s
    while (lo < hi) {
      const uint32_t mid = (lo + hi) >> 1;
      if (oe[mid] > s) hi = mid; else lo = mid + 1;
    }
    for (uint32_t j = lo; j < nobj && ob[j] <= e; ++j) {
      const uint64_t cs = s > ob[j] ? s : ob[j], ce = e < oe[j] - 1 ? e : oe[j] - 1;
      atomicAdd(&acc[4 * j + 0], 1ull);
      atomicAdd(&acc[4 * j + 1], (unsigned long long)(ce - cs + 1));
      atomicMin(&acc[4 * j + 2], (unsigned long long)cs);
      atomicMax(&acc[4 * j + 3], (unsigned long long)ce);
    }
  }
}

static unsigned grid_for(const ve_ctx* c, uint64_t items_per_block, uint64_t n) {
  uint64_t b = (n + items_per_block - 1) / items_per_block;
  const uint64_t cap = (uint64_t)c->num_sms * 8;
  if (b > cap) b = cap;
  return (unsigned)(b ? b : 1);
}

// exclusive sum scan of a[0..n) in place (scratch part[] of >= n / SC_TILE + 1 entries)
static void scan_sum(uint32_t* a, uint64_t n, uint32_t* part, cudaStream_t s) {
  const uint64_t nb = (n + SC_TILE - 1) / SC_TILE;
  if (nb <= 1) {
    count_launch();
    k_scan_sum_1<<<1, IV_T, 0, s>>>(a, n);
    return;
  }
  count_launch();
  k_scan_part<<<(unsigned)nb, IV_T, 0, s>>>(a, n, part);
  count_launch();
  k_scan_sum_1<<<1, IV_T, 0, s>>>(part, nb);
  count_launch();
  k_scan_apply<<<(unsigned)nb, IV_T, 0, s>>>(a, n, part);
}

// Sort + merge the m compacted intervals in (S, E) (ping-pong buffers S2, E2) into d_out.
// Stable LSD radix sort of the pairs (S[i], E[i]), i < m, by S (ping-pong with S2/E2; on
// return S/E point at the sorted arrays).  Skipped when S is already non-decreasing.
// scr: sort_scratch_bytes(m) bytes of device scratch.  Also used by f3 (k_temporal.cu).
size_t sort_scratch_bytes(uint64_t m) {
  const uint64_t ntile = (m + IV_TILE - 1) / IV_TILE;
  const uint64_t nh = ntile * 256;
  return 64 + 4 * nh + 4 * (nh / SC_TILE + 2) + 16;
}

ve_status sort_pairs(ve_ctx* c, uint64_t*& S, uint64_t*& E, uint64_t*& S2, uint64_t*& E2, uint64_t m, uint8_t* scr,
                     cudaStream_t s) {
  unsigned long long* rng = (unsigned long long*)scr;   // [4]
  const unsigned long long init[4] = {~0ull, 0ull, 0ull, 0ull};
  cudaError_t e = cudaMemcpyAsync(rng, init, sizeof(init), cudaMemcpyHostToDevice, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "intervals: range init");
  count_launch();
  k_iv_range<<<grid_for(c, IV_T, m), IV_T, 0, s>>>(S, m, rng);
  unsigned long long hr[4];
  e = cudaMemcpyAsync(hr, rng, sizeof(hr), cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c, e, "intervals: range");
  const uint64_t ntile = (m + IV_TILE - 1) / IV_TILE;
  uint32_t* hist = (uint32_t*)(scr + 64);
  const uint64_t nh = ntile * 256;
  uint32_t* part = hist + nh;
  if (hr[2] != 0) {   // not sorted yet: LSD passes over the bits in which the starts differ
    const uint64_t span = hr[1] - hr[0];
    const int bits = span ? 64 - __builtin_clzll(span) : 0;
    for (int sh = 0; sh < bits; sh += 8) {
      count_launch();
      k_rs_hist<<<(unsigned)ntile, IV_T, 0, s>>>(S, m, hr[0], (uint32_t)sh, hist, (uint32_t)ntile);
      scan_sum(hist, nh, part, s);
      count_launch();
      k_rs_scatter<<<(unsigned)ntile, IV_T, 0, s>>>(S, E, m, hr[0], (uint32_t)sh, hist, (uint32_t)ntile, S2, E2);
      std::swap(S, S2);
      std::swap(E, E2);
    }
  }
  return VE_OK;
}

static ve_status merge_sorted_pass(ve_ctx* c, uint64_t* S, uint64_t* E, uint64_t* S2, uint64_t* E2, uint64_t m,
                                   uint8_t* scr, ve_interval* d_out, uint64_t* h_n, cudaStream_t s) {
  ve_status st = sort_pairs(c, S, E, S2, E2, m, scr, s);
  if (st != VE_OK) return st;
  cudaError_t e;
  const uint64_t ntile = (m + IV_TILE - 1) / IV_TILE;
  const uint64_t nh = ntile * 256;
  uint32_t* part = (uint32_t*)(scr + 64) + nh;
  // merge: tile maxima -> exclusive carries, flag counts -> offsets, emit
  unsigned long long* tcar = (unsigned long long*)(((uintptr_t)(part + nh / SC_TILE + 2) + 15) & ~(uintptr_t)15);
  uint32_t* fcnt = (uint32_t*)(tcar + ntile);
  count_launch();
  k_iv_tile_max<<<(unsigned)ntile, IV_T, 0, s>>>(E, m, tcar);
  count_launch();
  k_scan_max_1<<<1, IV_T, 0, s>>>(tcar, ntile);
  count_launch();
  k_iv_merge<false><<<(unsigned)ntile, IV_T, 0, s>>>(S, E, m, tcar, fcnt, nullptr, nullptr);
  uint32_t last = 0;
  e = cudaMemcpyAsync(&last, fcnt + ntile - 1, 4, cudaMemcpyDeviceToHost, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "intervals: flag count");
  scan_sum(fcnt, ntile, part, s);
  uint32_t last_off = 0;
  e = cudaMemcpyAsync(&last_off, fcnt + ntile - 1, 4, cudaMemcpyDeviceToHost, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "intervals: flag offsets");
  count_launch();
  k_iv_merge<true><<<(unsigned)ntile, IV_T, 0, s>>>(S, E, m, tcar, nullptr, fcnt, d_out);
  e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c, e, "intervals: merge");
  *h_n = (uint64_t)last_off + last;
  return VE_OK;
}

// workspace: 4 arrays of cap u64 + scan / carry scratch
static size_t iv_bytes(uint64_t cap) {
  const uint64_t ntile = (cap + IV_TILE - 1) / IV_TILE;
  const uint64_t nh = ntile * 256;
  return 32 * cap + 64 + 4 * nh + 4 * (nh / SC_TILE + 2) + 8 * ntile + 4 * ntile + 256;
}

static ve_status iv_alloc(ve_ctx* c, uint64_t cap, uint8_t** buf, cudaStream_t s) {
  cudaError_t e = cudaMallocAsync((void**)buf, iv_bytes(cap), s);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(c, VE_ERR_NOMEM, "intervals: workspace");
  }
  return VE_OK;
}

// ---- LoadSpy temporal load redundancy in record order (C17) ----------
// 1. ordered compaction of the valid global-space loads into (address, record index)
// 2. stable sort by address (sort_pairs): each address's loads stay in record order
// 3. gather each sorted load's value / meta (one random read per load), then judge every
//    sorted neighbour pair of one address, i.e. (last load, load), sequentially
__device__ __forceinline__ bool tl_load(const ve_record* r, uint64_t i, uint64_t n, uint32_t n_pcs, uint64_t& addr) {
  if (i >= n) return false;
  const unsigned long long* q = reinterpret_cast<const unsigned long long*>(&r[i]);
  addr = __ldg(q);
  const uint64_t val = __ldg(q + 1), pm = __ldg(q + 2);
  const uint32_t meta = (uint32_t)(pm >> 32);
  return rec_valid(addr, val, (uint32_t)pm, meta, n_pcs) && !meta_shared(meta) && !meta_store(meta);
}

__global__ void __launch_bounds__(IV_T) k_tl_count(const ve_record* r, uint64_t n, uint32_t n_pcs, uint32_t* cnt) {
  const uint64_t t0 = (uint64_t)blockIdx.x * IV_TILE;
  uint32_t c = 0;
  for (int j = 0; j < IV_ITEMS; ++j) {
    uint64_t a;
    c += tl_load(r, t0 + (uint64_t)j * IV_T + threadIdx.x, n, n_pcs, a) ? 1u : 0u;
  }
  c = __reduce_add_sync(FULLM, c);
  __shared__ uint32_t sm[IV_NW];
  if ((threadIdx.x & 31) == 0) sm[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t t = 0;
    for (int k = 0; k < IV_NW; ++k) t += sm[k];
    cnt[blockIdx.x] = t;
  }
}

__global__ void __launch_bounds__(IV_T) k_tl_write(const ve_record* r, uint64_t n, uint32_t n_pcs, const uint32_t* off,
                                                   uint64_t* S, uint64_t* E) {
  __shared__ uint32_t sm[IV_NW];
  const uint64_t t0 = (uint64_t)blockIdx.x * IV_TILE;
  uint32_t carry = off[blockIdx.x];
  for (int j = 0; j < IV_ITEMS; ++j) {
    const uint64_t i = t0 + (uint64_t)j * IV_T + threadIdx.x;
    uint64_t a = 0;
    const bool f = tl_load(r, i, n, n_pcs, a);
    uint32_t tot;
    const uint32_t ex = block_excl_scan(f ? 1u : 0u, OpAdd(), 0u, sm, tot);
    if (f) {
      S[carry + ex] = a;
      E[carry + ex] = i;
    }
    carry += tot;
  }
}

// (temporal, redundant) += (group size, redundant lanes) for key; lanes of equal keys share one
// update, into the block's shared counters for keys < TL_SK (flushed at exit), else global
constexpr uint32_t TL_SK = 1024;
__device__ __forceinline__ void tl_add(uint32_t* sc, unsigned long long* out, bool act, uint32_t key, uint32_t red) {
  const unsigned am = __ballot_sync(FULLM, act);
  if (!act) return;
  const unsigned g = __match_any_sync(am, key);
  const uint32_t nr = __popc(__ballot_sync(g, red != 0u) & g);
  if ((int)(threadIdx.x & 31) == __ffs(g) - 1) {
    if (key < TL_SK) {
      atomicAdd(&sc[2 * key], (uint32_t)__popc(g));
      if (nr) atomicAdd(&sc[2 * key + 1], nr);
    } else {
      atomicAdd(&out[2 * (uint64_t)key], (unsigned long long)__popc(g));
      if (nr) atomicAdd(&out[2 * (uint64_t)key + 1], (unsigned long long)nr);
    }
  }
}

// sorted position j -> the value bits and (pc | meta << 32) of its record: the one random
// gather of the pass (the judge then reads neighbours sequentially)
__global__ void __launch_bounds__(IV_T) k_tl_gather(const ve_record* r, const uint64_t* E, uint64_t m, uint64_t* V,
                                                    uint64_t* PM) {
  const uint64_t stride = (uint64_t)gridDim.x * IV_T;
  uint64_t j = (uint64_t)blockIdx.x * IV_T + threadIdx.x;
  for (; j + 3 * stride < m; j += 4 * stride) {     // four random reads in flight per thread
    uint64_t v[4], pm[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const unsigned long long* q = reinterpret_cast<const unsigned long long*>(&r[E[j + u * stride]]);
      v[u] = __ldg(q + 1);
      pm[u] = __ldg(q + 2);
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) { V[j + u * stride] = v[u]; PM[j + u * stride] = pm[u]; }
  }
  for (; j < m; j += stride) {
    const unsigned long long* q = reinterpret_cast<const unsigned long long*>(&r[E[j]]);
    V[j] = __ldg(q + 1);
    PM[j] = __ldg(q + 2);
  }
}

// pairs != null: also the (pc, object) table (f3 per pair): row pc, column = object id (nobj: none)
__device__ __forceinline__ void tl_add_global(unsigned long long* out, bool act, uint64_t key, uint32_t red) {
  const unsigned am = __ballot_sync(FULLM, act);
  if (!act) return;
  const unsigned g = __match_any_sync(am, key);
  const uint32_t nr = __popc(__ballot_sync(g, red != 0u) & g);
  if ((int)(threadIdx.x & 31) == __ffs(g) - 1) {
    atomicAdd(&out[2 * key], (unsigned long long)__popc(g));
    if (nr) atomicAdd(&out[2 * key + 1], (unsigned long long)nr);
  }
}

__global__ void __launch_bounds__(IV_T) k_tl_judge(const uint64_t* S, const uint64_t* V, const uint64_t* PM,
                                                   uint64_t m, const uint64_t* ob, const uint64_t* oe,
                                                   const uint32_t* oid, uint32_t nobj, uint32_t n_pcs,
                                                   unsigned long long* out, unsigned long long* pairs) {
  __shared__ uint32_t sc[2 * TL_SK];   // per-block counters of the first TL_SK keys (< 2^32 per block)
  for (uint32_t i = threadIdx.x; i < 2 * TL_SK; i += IV_T) sc[i] = 0;
  __syncthreads();
  const uint64_t stride = (uint64_t)gridDim.x * IV_T;
  for (uint64_t b = (uint64_t)blockIdx.x * IV_T; b < m; b += stride) {   // block-uniform trip count
    const uint64_t j = b + threadIdx.x;
    bool temporal = false;
    uint32_t red = 0, pc = 0, okey = 0;
    bool has_obj = false;
    if (j > 0 && j < m && S[j] == S[j - 1]) {
      temporal = true;
      const uint64_t pmi = PM[j], pmp = PM[j - 1];
      red = (V[j] == V[j - 1] && ((pmi >> 32) & 3u) == ((pmp >> 32) & 3u)) ? 1u : 0u;
      pc = (uint32_t)pmi;
      const uint64_t a = S[j];
      uint32_t lo = 0, hi = nobj;          // first object with base > a
      while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (ob[mid] <= a) lo = mid + 1; else hi = mid;
      }
      if (lo > 0 && a < oe[lo - 1]) { has_obj = true; okey = n_pcs + oid[lo - 1]; }
    }
    tl_add(sc, out, temporal, pc, red);
    tl_add(sc, out, has_obj, okey, red);
    if (pairs) {                           // (block-uniform: every lane takes part)
      const uint64_t pk = (uint64_t)pc * (nobj + 1) + (has_obj ? okey - n_pcs : nobj);
      tl_add_global(pairs, temporal, pk, red);
    }
  }
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < 2 * TL_SK; i += IV_T)
    if (sc[i]) atomicAdd(&out[i], (unsigned long long)sc[i]);
}

}  // namespace ve

using namespace ve;

extern "C" {

ve_status ve_temporal_loads_ex(ve_ctx* c, const ve_record* d_records, uint64_t n, uint64_t* h_out,
                               uint64_t* h_pairs, cudaStream_t s) {
  if (!c || !h_out) return VE_ERR_INVALID;
  const uint32_t nk = c->n_keys;
  ctx_begin(c, s);
  const uint64_t npairs = (uint64_t)c->cfg.n_pcs * (c->n_obj + 1);
  if (h_pairs && npairs > (1ull << 24)) return fail(c, VE_ERR_INVALID, "ve_temporal_loads_ex: n_pcs x (objects + 1) > 2^24");
  memset(h_out, 0, sizeof(uint64_t) * 2 * nk);
  if (h_pairs) memset(h_pairs, 0, sizeof(uint64_t) * 2 * npairs);
  if (n == 0) return VE_OK;
  if (!d_records || ((uintptr_t)d_records & 7)) return fail(c, VE_ERR_INVALID, "ve_temporal_loads: null or misaligned");
  if (n >= (1ull << 32)) return fail(c, VE_ERR_INVALID, "ve_temporal_loads: n >= 2^32");
  cudaSetDevice(c->device);
  const uint64_t ntile = (n + IV_TILE - 1) / IV_TILE;
  const size_t need = 32 * n + sort_scratch_bytes(n) + 4 * ntile + 4 * (ntile / SC_TILE + 2) + 16 * (size_t)nk + 64 +
                      (h_pairs ? 16 * npairs : 0);
  uint8_t* buf = nullptr;
  cudaError_t e = cudaMallocAsync((void**)&buf, need, s);
  if (e != cudaSuccess) { cudaGetLastError(); return fail(c, VE_ERR_NOMEM, "ve_temporal_loads: workspace"); }
  uint64_t* S = (uint64_t*)buf;
  uint64_t* E = S + n;
  uint64_t* S2 = E + n;
  uint64_t* E2 = S2 + n;
  uint8_t* scr = (uint8_t*)(E2 + n);
  uint32_t* tcnt = (uint32_t*)(scr + sort_scratch_bytes(n));
  uint32_t* part = tcnt + ntile;
  unsigned long long* d_out =
      (unsigned long long*)(((uintptr_t)(part + ntile / SC_TILE + 2) + 15) & ~(uintptr_t)15);
  count_launch();
  k_tl_count<<<(unsigned)ntile, IV_T, 0, s>>>(d_records, n, c->cfg.n_pcs, tcnt);
  uint32_t last = 0, last_off = 0;
  cudaMemcpyAsync(&last, tcnt + ntile - 1, 4, cudaMemcpyDeviceToHost, s);
  scan_sum(tcnt, ntile, part, s);
  cudaMemcpyAsync(&last_off, tcnt + ntile - 1, 4, cudaMemcpyDeviceToHost, s);
  count_launch();
  k_tl_write<<<(unsigned)ntile, IV_T, 0, s>>>(d_records, n, c->cfg.n_pcs, tcnt, S, E);
  e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) { cudaFreeAsync(buf, s); return cuda_fail(c, e, "ve_temporal_loads: compaction"); }
  const uint64_t m = (uint64_t)last_off + last;
  ve_status st = VE_OK;
  if (m > 1) {
    st = sort_pairs(c, S, E, S2, E2, m, scr, s);
    if (st == VE_OK) {
      unsigned long long* d_pairs = h_pairs ? d_out + 2 * (size_t)nk : nullptr;
      cudaMemsetAsync(d_out, 0, 16 * (size_t)nk + (h_pairs ? 16 * npairs : 0), s);
      count_launch();
      k_tl_gather<<<grid_for(c, IV_T, m), IV_T, 0, s>>>(d_records, E, m, S2, E2);   // the sort's spare buffers
      count_launch();
      k_tl_judge<<<grid_for(c, IV_T, m), IV_T, 0, s>>>(S, S2, E2, m, c->o.base, c->o.end, c->o.id, c->n_obj,
                                                       c->cfg.n_pcs, d_out, d_pairs);
      e = cudaMemcpyAsync(h_out, d_out, 16 * (size_t)nk, cudaMemcpyDeviceToHost, s);
      if (e == cudaSuccess && h_pairs) e = cudaMemcpyAsync(h_pairs, d_pairs, 16 * npairs, cudaMemcpyDeviceToHost, s);
      if (e == cudaSuccess) e = cudaStreamSynchronize(s);
      if (e != cudaSuccess) st = cuda_fail(c, e, "ve_temporal_loads");
    }
  }
  cudaFreeAsync(buf, s);
  return st;
}

ve_status ve_temporal_loads(ve_ctx* c, const ve_record* d_records, uint64_t n, uint64_t* h_out, cudaStream_t s) {
  return ve_temporal_loads_ex(c, d_records, n, h_out, nullptr, s);
}


ve_status ve_interval_merge(ve_ctx* c, const ve_interval* d_in, uint64_t n, ve_interval* d_out, uint64_t* h_n_out,
                            cudaStream_t s) {
  if (!c || !h_n_out) return VE_ERR_INVALID;
  *h_n_out = 0;
  if (n == 0) return VE_OK;
  ctx_begin(c, s);
  if (!d_in || !d_out) return fail(c, VE_ERR_INVALID, "ve_interval_merge: null interval array");
  if (n >= (1ull << 32)) return fail(c, VE_ERR_INVALID, "ve_interval_merge: n >= 2^32");
  cudaSetDevice(c->device);
  uint8_t* buf = nullptr;
  ve_status st = iv_alloc(c, n, &buf, s);
  if (st != VE_OK) return st;
  unsigned long long* cnt = (unsigned long long*)(buf + 32 * n);   // first word of the scratch
  cudaMemsetAsync(cnt, 0, 8, s);
  count_launch();
  k_iv_in<<<grid_for(c, (uint64_t)IV_NW * 32, n), IV_T, 0, s>>>(d_in, n, (uint64_t*)buf, (uint64_t*)buf + n, cnt);
  // the count lives where merge_sorted_pass keeps its range words: read it before
  unsigned long long m = 0;
  cudaError_t e = cudaMemcpyAsync(&m, cnt, 8, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) { cudaFreeAsync(buf, s); return cuda_fail(c, e, "ve_interval_merge"); }
  uint64_t* S = (uint64_t*)buf;
  if (m) st = merge_sorted_pass(c, S, S + n, S + 2 * n, S + 3 * n, m, buf + 32 * n, d_out, h_n_out, s);
  cudaFreeAsync(buf, s);
  return st;
}

ve_status ve_record_intervals(ve_ctx* c, const ve_record* d_records, uint64_t n, ve_interval* d_out,
                              uint64_t* h_n_out, cudaStream_t s) {
  if (!c || !h_n_out) return VE_ERR_INVALID;
  *h_n_out = 0;
  if (n == 0) return VE_OK;
  ctx_begin(c, s);
  if (!d_records || !d_out || ((uintptr_t)d_records & 7))
    return fail(c, VE_ERR_INVALID, "ve_record_intervals: null or misaligned array");
  if (n >= (1ull << 32)) return fail(c, VE_ERR_INVALID, "ve_record_intervals: n >= 2^32");
  cudaSetDevice(c->device);
  uint8_t* buf = nullptr;
  ve_status st = iv_alloc(c, n, &buf, s);
  if (st != VE_OK) return st;
  unsigned long long* cnt = (unsigned long long*)(buf + 32 * n);
  cudaMemsetAsync(cnt, 0, 8, s);
  count_launch();
  k_iv_rec<<<grid_for(c, (uint64_t)IV_NW * 32, n), IV_T, 0, s>>>(d_records, n, c->cfg.n_pcs, (uint64_t*)buf,
                                                                  (uint64_t*)buf + n, cnt);
  unsigned long long m = 0;
  cudaError_t e = cudaMemcpyAsync(&m, cnt, 8, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) { cudaFreeAsync(buf, s); return cuda_fail(c, e, "ve_record_intervals"); }
  uint64_t* S = (uint64_t*)buf;
  if (m) st = merge_sorted_pass(c, S, S + n, S + 2 * n, S + 3 * n, m, buf + 32 * n, d_out, h_n_out, s);
  cudaFreeAsync(buf, s);
  return st;
}

ve_status ve_plan_copies(ve_ctx* c, const ve_interval* d_merged, uint64_t n, uint32_t seg_max, uint32_t dense_pct,
                       ve_copy_plan* h_plan, cudaStream_t s) {
  if (!c || (c->n_obj && !h_plan)) return VE_ERR_INVALID;
  if (n && !d_merged) return fail(c, VE_ERR_INVALID, "ve_plan_copies: null interval array");
  if (dense_pct > 100) return fail(c, VE_ERR_INVALID, "ve_plan_copies: dense_pct > 100");
  ctx_begin(c, s);
  const uint32_t no = c->n_obj;
  if (no == 0) return VE_OK;
  cudaSetDevice(c->device);
  unsigned long long* acc = nullptr;
  cudaError_t e = cudaMallocAsync((void**)&acc, 32 * (size_t)no + 16, s);
  if (e != cudaSuccess) { cudaGetLastError(); return fail(c, VE_ERR_NOMEM, "ve_plan_copies: workspace"); }
  std::vector<unsigned long long> init(4 * (size_t)no + 2, 0ull);
  for (uint32_t j = 0; j < no; ++j) init[4 * j + 2] = ~0ull;
  e = cudaMemcpyAsync(acc, init.data(), 32 * (size_t)no + 16, cudaMemcpyHostToDevice, s);
  unsigned int* bad = (unsigned int*)(acc + 4 * no);
  if (n && e == cudaSuccess) {
    count_launch();
    k_iv_plan<<<grid_for(c, IV_T, n), IV_T, 0, s>>>(d_merged, n, c->o.base, c->o.end, no, acc, bad);
  }
  std::vector<unsigned long long> h(4 * (size_t)no + 2);
  if (e == cudaSuccess) e = cudaMemcpyAsync(h.data(), acc, 32 * (size_t)no + 16, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  cudaFreeAsync(acc, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "ve_plan_copies");
  if (((unsigned int*)&h[4 * no])[0])
    return fail(c, VE_ERR_INVALID, "ve_plan_copies: intervals not sorted, disjoint and non-adjacent");
  for (uint32_t j = 0; j < no; ++j) {   // sorted index j -> object id
    const HostObject& o = c->objs[j];
    ve_copy_plan& p = h_plan[o.id];
    p.n_segments = h[4 * j];
    p.accessed_bytes = h[4 * j + 1];
    p.lo = p.n_segments ? h[4 * j + 2] : 0;
    p.hi = h[4 * j + 3];
    p.direct_bytes = o.size;
    p.minmax_bytes = p.n_segments ? p.hi - p.lo + 1 : 0;
    const bool sparse = (unsigned __int128)100 * p.accessed_bytes < (unsigned __int128)dense_pct * p.minmax_bytes;
    p.choice = p.n_segments == 0 ? VE_COPY_NONE
                                 : (sparse && p.n_segments <= seg_max) ? VE_COPY_SEGMENT : VE_COPY_MINMAX;
    p.pad = 0;
  }
  return VE_OK;
}

}  // extern "C"
