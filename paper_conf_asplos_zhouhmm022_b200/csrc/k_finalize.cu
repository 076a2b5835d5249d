// k_finalize.cu -- report-time reductions (SURVEY 8(a) S8 top-k, S9 popcounts).
//
// K4: the exact (pc, object, value) histogram is compacted, re-aggregated into
// the per-PC and per-object views (Def 3.3 counts accesses per key),
// grouped by key, and reduced to n_distinct + top-k by (count desc, bits asc)
// with a chunked block-wide selection (levels until one chunk per key).
// K6: popcounts of the written / loaded element bitmaps per object (C3, C10).
#include <cuda_runtime.h>

#include <algorithm>
#include <vector>

#include "ve_internal.cuh"

#include <chrono>
#include <cstdlib>

namespace ve {

// VE_TIMING=2: per-stage timings of the report path on stderr
static void stage(const char* name, cudaStream_t s) {
  static const bool on = getenv("VE_TIMING") && atoi(getenv("VE_TIMING")) >= 2;
  static auto t0 = std::chrono::steady_clock::now();
  if (!on) return;
  cudaStreamSynchronize(s);
  const auto t1 = std::chrono::steady_clock::now();
  fprintf(stderr, "[ve]   %-18s %.3f ms\n", name, std::chrono::duration<double, std::milli>(t1 - t0).count());
  t0 = t1;
}

// ---- scratch management ------------------------------------------------------
static cudaError_t scratch_need(ve_ctx* c, size_t bytes) {
  if (c->scratch_bytes >= bytes) return cudaSuccess;
  c->scratch_bytes = 0;
  cudaError_t e = ctx_realloc(c, &c->scratch, bytes);
  if (e == cudaSuccess) c->scratch_bytes = bytes;
  return e;
}

__device__ __forceinline__ bool vinsert(HSlot* slots, unsigned long long* counts, uint64_t mask,
                                        unsigned long long* overflow, uint32_t tag, uint64_t bits,
                                        unsigned long long cnt) {
  // CAS first (empty slots are all-ones, occupied ones have pad 0): one round trip per probe
  uint64_t h = hist_hash(tag, bits) & mask;
  for (uint64_t probe = 0; probe <= mask; ++probe) {
    uint64_t olo, ohi;
    cas128_global(&slots[h], ~0ull, ~0ull, bits, (uint64_t)tag, olo, ohi);
    if ((olo == ~0ull && ohi == ~0ull) || (olo == bits && ohi == (uint64_t)tag)) {
      atomicAdd(&counts[h], cnt);
      return true;
    }
    h = (h + 1) & mask;
  }
  atomicExch(overflow, 1ull);
  return false;
}

// occupied main-table slots -> per-PC and per-object view table
__global__ void k_views(const HSlot* hs, const unsigned long long* hc, uint64_t hcap, uint32_t n_pcs,
                        HSlot* vs, unsigned long long* vc, uint64_t vmask, unsigned long long* overflow,
                        unsigned long long* n_entries) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < hcap; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t tag = hs[i].tag;
    if (tag == EMPTY_TAG) continue;
    const uint64_t bits = hs[i].bits;
    const unsigned long long cnt = hc[i];
    atomicAdd(n_entries, 1ull);
    const uint32_t pc = tag >> 16, koi = tag & 0xFFFFu;
    vinsert(vs, vc, vmask, overflow, pc, bits, cnt);
    if (koi != KO_NONE) vinsert(vs, vc, vmask, overflow, n_pcs + koi, bits, cnt);
  }
}

__global__ void k_occupancy(const HSlot* hs, uint64_t cap, unsigned long long* cnt);

// the exact histogram's entries of single-float-type keys, with
// their values truncated to K mantissa bits (NaNs kept), -> a view table of the
// approximate values.  akind[key] = kind << 2 | lg, or 0xFF (no approximate histogram).
__global__ void k_approx_views(const HSlot* hs, const unsigned long long* hc, uint64_t hcap, uint32_t n_pcs,
                               const uint8_t* akind, uint32_t K, HSlot* vs, unsigned long long* vc, uint64_t vmask,
                               unsigned long long* overflow) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < hcap; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t tag = hs[i].tag;
    if (tag == EMPTY_TAG) continue;
    const uint64_t bits = hs[i].bits;
    const unsigned long long cnt = hc[i];
    const uint32_t pc = tag >> 16, koi = tag & 0xFFFFu;
#pragma unroll
    for (int j = 0; j < 2; ++j) {
      if (j == 1 && koi == KO_NONE) break;
      const uint32_t key = j == 0 ? pc : n_pcs + koi;
      const uint32_t ak = akind[key];
      if (ak == 0xFFu) continue;
      const uint32_t kind = ak >> 2, lg = ak & 3u;
      int64_t ival;
      const bool nan = float_flags(bits, kind, lg, ival) & 1u;
      vinsert(vs, vc, vmask, overflow, key, nan ? bits : trunc_bits(bits, kind, lg, K), cnt);
    }
  }
}

ve_status approx_topk(ve_ctx* c, cudaStream_t s, const std::vector<uint8_t>& akind, std::vector<uint64_t>& ndistinct,
                      std::vector<ve_topk_entry>& top) {
  cudaError_t e;
  unsigned long long* d_small = nullptr;   // [0] overflow, [1] occupied
  uint8_t* d_ak = nullptr;
  e = cudaMallocAsync((void**)&d_small, 16, s);
  if (e == cudaSuccess) e = cudaMallocAsync((void**)&d_ak, akind.size(), s);
  if (e != cudaSuccess) return cuda_fail(c, e, "approx alloc");
  cudaMemsetAsync(d_small, 0, 16, s);
  cudaMemcpyAsync(d_ak, akind.data(), akind.size(), cudaMemcpyHostToDevice, s);
  count_launch();
  k_occupancy<<<c->num_sms * 4, 256, 0, s>>>(c->t.hslot, c->hcap, d_small + 1);
  unsigned long long occ = 0;
  e = cudaMemcpyAsync(&occ, d_small + 1, 8, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) { cudaFreeAsync(d_small, s); cudaFreeAsync(d_ak, s); return cuda_fail(c, e, "approx occupancy"); }
  ViewTable V;
  ve_status st = alloc_views(c, s, 2 * occ + 1, V);
  if (st != VE_OK) { cudaFreeAsync(d_small, s); cudaFreeAsync(d_ak, s); return st; }
  count_launch();
  k_approx_views<<<c->num_sms * 4, 256, 0, s>>>(c->t.hslot, c->t.hcount, c->hcap, c->cfg.n_pcs, d_ak,
                                                c->cfg.mant_bits, V.vs, V.vc, V.vcap - 1, d_small);
  unsigned long long ovf = 0;
  e = cudaMemcpyAsync(&ovf, d_small, 8, cudaMemcpyDeviceToHost, s);
  cudaFreeAsync(d_small, s);
  cudaFreeAsync(d_ak, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) { free_views(V, s); return cuda_fail(c, e, "approx views"); }
  if (ovf) { free_views(V, s); return fail(c, VE_ERR_CAPACITY, "approx: view table overflow"); }
  st = view_topk(c, V, s, ndistinct, top);
  free_views(V, s);
  return st;
}

// Warp-aggregated counter increment: lanes with equal keys share one atomic (the
// per-key counters are few and hot, so plain per-entry atomics serialise).
// Every lane of the warp must call it; returns this lane's slot (cursor value).
__device__ __forceinline__ unsigned long long warp_count(unsigned long long* ctr, bool active, uint32_t key) {
  const unsigned am = __ballot_sync(0xFFFFFFFFu, active);
  unsigned long long base = 0;
  if (active) {
    const unsigned g = __match_any_sync(am, key);
    const int lead = __ffs(g) - 1, lane = threadIdx.x & 31;
    if (lane == lead) base = atomicAdd(ctr, (unsigned long long)__popc(g));
    base = __shfl_sync(g, base, lead);
    base += __popc(g & ((1u << lane) - 1u));
  }
  return base;
}

// warp-uniform grid-stride loop over [0, n): every lane runs the same iterations
#define VE_WARP_LOOP(i, n)                                                                        \
  for (uint64_t i##_b = ((uint64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31u)); i##_b < (n);  \
       i##_b += (uint64_t)gridDim.x * blockDim.x)                                                 \
    for (uint64_t i = i##_b + (threadIdx.x & 31u), i##_once = 1; i##_once; i##_once = 0)

__global__ void k_view_count(const HSlot* vs, uint64_t vcap, unsigned long long* ndist) {
  VE_WARP_LOOP(i, vcap) {
    const uint32_t tag = i < vcap ? vs[i].tag : EMPTY_TAG;
    warp_count(&ndist[tag != EMPTY_TAG ? tag : 0], tag != EMPTY_TAG, tag);
  }
}

__global__ void k_view_scatter(const HSlot* vs, const unsigned long long* vc, uint64_t vcap,
                               const unsigned long long* off, unsigned long long* cursor, uint64_t* gbits,
                               uint64_t* gcnt) {
  VE_WARP_LOOP(i, vcap) {
    const uint32_t tag = i < vcap ? vs[i].tag : EMPTY_TAG;
    const bool act = tag != EMPTY_TAG;
    const unsigned long long p = warp_count(&cursor[act ? tag : 0], act, tag);
    if (act) {
      gbits[off[tag] + p] = vs[i].bits;
      gcnt[off[tag] + p] = vc[i];
    }
  }
}

struct Chunk {
  uint64_t start, out;
  uint32_t len, nout;
};

ve_status select_topk(ve_ctx* c, cudaStream_t s, uint64_t* gb[2], uint64_t* gc[2], std::vector<uint64_t> len,
                      std::vector<uint64_t> start, std::vector<ve_topk_entry>& top);

constexpr int TK_THREADS = 256;
constexpr int TK_PER = 16;
constexpr int TK_CHUNK = TK_THREADS * TK_PER;

// "a before b" in the top-k order: count desc, then bits asc
__device__ __forceinline__ bool before(uint64_t ca, uint64_t ba, uint64_t cb, uint64_t bb) {
  return ca > cb || (ca == cb && ba < bb);
}

__global__ void __launch_bounds__(TK_THREADS) k_topk_chunk(const Chunk* chunks, const uint64_t* ib,
                                                            const uint64_t* ic, uint64_t* ob, uint64_t* oc) {
  const Chunk ch = chunks[blockIdx.x];
  uint64_t b[TK_PER], c[TK_PER];
#pragma unroll
  for (int j = 0; j < TK_PER; ++j) {
    const uint32_t idx = threadIdx.x + j * TK_THREADS;
    if (idx < ch.len) { b[j] = ib[ch.start + idx]; c[j] = ic[ch.start + idx]; }
    else { b[j] = 0; c[j] = 0; }
  }
  __shared__ uint64_t sb[TK_THREADS / 32], sc[TK_THREADS / 32];
  __shared__ uint64_t pb_s, pc_s;
  // previous pick; "after prev" = before(prev, e).  Start with a sentinel above everything.
  uint64_t pb = 0, pcnt = ~0ull;
  bool first = true;
  for (uint32_t r = 0; r < ch.nout; ++r) {
    uint64_t bb = ~0ull, bc = 0;
    bool have = false;
#pragma unroll
    for (int j = 0; j < TK_PER; ++j) {
      const uint32_t idx = threadIdx.x + j * TK_THREADS;
      if (idx >= ch.len) continue;
      const bool after = first || before(pcnt, pb, c[j], b[j]);
      if (after && (!have || before(c[j], b[j], bc, bb))) { bb = b[j]; bc = c[j]; have = true; }
    }
    // warp reduce (no candidate = count 0, bits ~0: loses to every real entry since counts >= 1)
    for (int o = 16; o > 0; o >>= 1) {
      const uint64_t ob2 = __shfl_xor_sync(0xFFFFFFFFu, bb, o);
      const uint64_t oc2 = __shfl_xor_sync(0xFFFFFFFFu, bc, o);
      if (before(oc2, ob2, bc, bb)) { bb = ob2; bc = oc2; }
    }
    if ((threadIdx.x & 31) == 0) { sb[threadIdx.x >> 5] = bb; sc[threadIdx.x >> 5] = bc; }
    __syncthreads();
    if (threadIdx.x == 0) {
      uint64_t xb = sb[0], xc = sc[0];
      for (int wdx = 1; wdx < TK_THREADS / 32; ++wdx)
        if (before(sc[wdx], sb[wdx], xc, xb)) { xb = sb[wdx]; xc = sc[wdx]; }
      ob[ch.out + r] = xb;
      oc[ch.out + r] = xc;
      pb_s = xb;
      pc_s = xc;
    }
    __syncthreads();
    pb = pb_s;
    pcnt = pc_s;
    first = false;
  }
}

__global__ void k_occupancy(const HSlot* hs, uint64_t cap, unsigned long long* cnt) {
  unsigned long long local = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < cap; i += (uint64_t)gridDim.x * blockDim.x)
    local += (hs[i].tag != EMPTY_TAG);
  for (int o = 16; o > 0; o >>= 1) local += __shfl_xor_sync(0xFFFFFFFFu, local, o);
  if ((threadIdx.x & 31) == 0 && local) atomicAdd(cnt, local);
}

// The per-PC / per-object view table built from the main (pc, object, value) table:
// every entry of tag (pc, o) contributes to view key pc and to view key n_pcs + o.
ve_status build_views(ve_ctx* c, cudaStream_t s, ViewTable& V) {
  cudaError_t e;
  unsigned long long* d_small = nullptr;  // [0] overflow, [1] occupancy / entries
  e = cudaMallocAsync((void**)&d_small, 16, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "views alloc");
  cudaMemsetAsync(d_small, 0, 16, s);
  count_launch();
  k_occupancy<<<c->num_sms * 4, 256, 0, s>>>(c->t.hslot, c->hcap, d_small + 1);
  unsigned long long occ = 0;
  e = cudaMemcpyAsync(&occ, d_small + 1, 8, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) { cudaFreeAsync(d_small, s); return cuda_fail(c, e, "views occupancy"); }
  cudaMemsetAsync(d_small, 0, 16, s);
  ve_status st = alloc_views(c, s, 2 * occ, V);
  if (st != VE_OK) { cudaFreeAsync(d_small, s); return st; }
  count_launch();
  k_views<<<c->num_sms * 4, 256, 0, s>>>(c->t.hslot, c->t.hcount, c->hcap, c->cfg.n_pcs, V.vs, V.vc, V.vcap - 1,
                                         d_small, d_small + 1);
  unsigned long long h_small[2];
  e = cudaMemcpyAsync(h_small, d_small, 16, cudaMemcpyDeviceToHost, s);
  cudaFreeAsync(d_small, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c, e, "views build");
  if (h_small[0]) return fail(c, VE_ERR_CAPACITY, "finalize: view table overflow");
  return VE_OK;
}

// an empty view table for up to n entries (load <= 1/2)
ve_status alloc_views(ve_ctx* c, cudaStream_t s, uint64_t n, ViewTable& V) {
  uint64_t vcap = 1024;
  while (vcap < 2 * n) vcap <<= 1;
  V.vcap = vcap;
  cudaError_t e = cudaMallocAsync((void**)&V.vs, vcap * sizeof(HSlot), s);
  if (e == cudaSuccess) e = cudaMallocAsync((void**)&V.vc, vcap * 8, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "view table alloc");
  cudaMemsetAsync(V.vs, 0xFF, vcap * sizeof(HSlot), s);
  cudaMemsetAsync(V.vc, 0, vcap * 8, s);
  return VE_OK;
}

void free_views(ViewTable& V, cudaStream_t s) {
  if (V.vs) cudaFreeAsync(V.vs, s);
  if (V.vc) cudaFreeAsync(V.vc, s);
  V.vs = nullptr;
  V.vc = nullptr;
}

// Exact n_distinct and top-k (count desc, bits asc) of every key of a view table.
ve_status view_topk(ve_ctx* c, const ViewTable& V, cudaStream_t s, std::vector<uint64_t>& ndistinct,
                    std::vector<ve_topk_entry>& top) {
  const uint32_t nk = c->n_keys, K = c->cfg.topk;
  ndistinct.assign(nk, 0);
  top.assign((size_t)nk * K, ve_topk_entry{0, 0});
  cudaError_t e;
  const uint64_t vcap = V.vcap;
  HSlot* vs = V.vs;
  unsigned long long* vc = V.vc;
  unsigned long long* d_nd = nullptr;                  // ndist, off, cursor
  e = cudaMallocAsync((void**)&d_nd, (size_t)nk * 8 * 3, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "top-k alloc");
  unsigned long long* d_off = d_nd + nk;
  unsigned long long* d_cur = d_off + nk;
  cudaMemsetAsync(d_nd, 0, (size_t)nk * 8 * 3, s);
  const int grid = c->num_sms * 4;
  count_launch();
  k_view_count<<<grid, 256, 0, s>>>(vs, vcap, d_nd);
  e = cudaMemcpyAsync(ndistinct.data(), d_nd, (size_t)nk * 8, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) { cudaFreeAsync(d_nd, s); return cuda_fail(c, e, "finalize ndistinct"); }
  uint64_t nent = 1;
  for (uint32_t k = 0; k < nk; ++k) nent += ndistinct[k];
  uint64_t* gbuf = nullptr;
  e = cudaMallocAsync((void**)&gbuf, 4 * nent * 8, s);
  if (e != cudaSuccess) { cudaFreeAsync(d_nd, s); return cuda_fail(c, e, "top-k alloc"); }
  uint64_t* gb[2] = {gbuf, gbuf + 2 * nent};
  uint64_t* gc[2] = {gbuf + nent, gbuf + 3 * nent};
  unsigned long long* d_small = nullptr;
  cudaMallocAsync((void**)&d_small, 16, s);
  cudaMemsetAsync(d_small, 0, 16, s);
  e = cudaMemcpyAsync(ndistinct.data(), d_nd, (size_t)nk * 8, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) { cudaFreeAsync(d_small, s); return cuda_fail(c, e, "finalize ndistinct"); }
  std::vector<unsigned long long> off(nk);
  uint64_t acc = 0;
  for (uint32_t k = 0; k < nk; ++k) { off[k] = acc; acc += ndistinct[k]; }
  cudaMemcpyAsync(d_off, off.data(), (size_t)nk * 8, cudaMemcpyHostToDevice, s);
  count_launch();
  k_view_scatter<<<grid, 256, 0, s>>>(vs, vc, vcap, d_off, d_cur, gb[0], gc[0]);
  std::vector<uint64_t> len(ndistinct.begin(), ndistinct.end()), start(off.begin(), off.end());
  ve_status st = select_topk(c, s, gb, gc, len, start, top);
  cudaFreeAsync(d_small, s);
  cudaFreeAsync(gbuf, s);
  cudaFreeAsync(d_nd, s);
  if (st != VE_OK) return st;
  e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c, e, "finalize top-k");
  return VE_OK;
}

// Top-k by (count desc, bits asc) of every key whose distinct entries lie in
// gb/gc[0][start[k] .. start[k]+len[k]): chunked block-wide selection, repeated
// on the chunk winners until every key fits one chunk.
ve_status select_topk(ve_ctx* c, cudaStream_t s, uint64_t* gb[2], uint64_t* gc[2], std::vector<uint64_t> len,
                      std::vector<uint64_t> start, std::vector<ve_topk_entry>& top) {
  const uint32_t nk = c->n_keys, K = c->cfg.topk;
  cudaError_t e;
  unsigned long long* d_small = nullptr;
  int cur = 0;
  Chunk* d_chunks = nullptr;
  size_t chunk_cap = 0;
  for (int level = 0;; ++level) {
    std::vector<Chunk> chunks;
    std::vector<uint64_t> nlen(nk, 0), nstart(nk, 0);
    uint64_t outp = 0;
    bool single = true;
    for (uint32_t k = 0; k < nk; ++k) {
      if (len[k] == 0) continue;
      const uint64_t nch = (len[k] + TK_CHUNK - 1) / TK_CHUNK;
      if (nch > 1) single = false;
      nstart[k] = outp;
      for (uint64_t j = 0; j < nch; ++j) {
        Chunk ch;
        ch.start = start[k] + j * TK_CHUNK;
        ch.len = (uint32_t)std::min<uint64_t>(TK_CHUNK, len[k] - j * TK_CHUNK);
        ch.nout = std::min<uint32_t>(K, ch.len);
        ch.out = outp;
        outp += ch.nout;
        chunks.push_back(ch);
      }
      nlen[k] = outp - nstart[k];
    }
    if (chunks.empty()) break;
    if (chunks.size() > chunk_cap) {
      if (d_chunks) cudaFreeAsync(d_chunks, s);
      chunk_cap = chunks.size() * 2;
      e = cudaMallocAsync((void**)&d_chunks, chunk_cap * sizeof(Chunk), s);
      if (e != cudaSuccess) { cudaFreeAsync(d_small, s); return cuda_fail(c, e, "finalize chunks"); }
    }
    cudaMemcpyAsync(d_chunks, chunks.data(), chunks.size() * sizeof(Chunk), cudaMemcpyHostToDevice, s);
    stage("chunk build", s);
    count_launch();
    k_topk_chunk<<<(unsigned)chunks.size(), TK_THREADS, 0, s>>>(d_chunks, gb[cur], gc[cur], gb[1 - cur],
                                                                gc[1 - cur]);
    stage("topk level", s);
    cur = 1 - cur;
    len.swap(nlen);
    start.swap(nstart);
    if (single) {
      std::vector<uint64_t> hb(outp), hc(outp);
      cudaMemcpyAsync(hb.data(), gb[cur], outp * 8, cudaMemcpyDeviceToHost, s);
      cudaMemcpyAsync(hc.data(), gc[cur], outp * 8, cudaMemcpyDeviceToHost, s);
      e = cudaStreamSynchronize(s);
      if (e != cudaSuccess) break;
      for (uint32_t k = 0; k < nk; ++k)
        for (uint64_t j = 0; j < len[k]; ++j) top[(size_t)k * K + j] = ve_topk_entry{hb[start[k] + j], hc[start[k] + j]};
      break;
    }
  }
  if (d_chunks) cudaFreeAsync(d_chunks, s);
  (void)d_small;
  e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c, e, "finalize top-k");
  return VE_OK;
}

// ---- finalize with direct grouping ------------------------------------------------
// A key whose entries all carry one tag (a PC that touched one object, an object
// touched by one PC -- the common case) needs no re-aggregation: its main-table
// entries ARE its distinct values.  Only keys fed by several tags go through the
// view table.
constexpr uint32_t TAG_CAP = 1u << 16;

// Block-local key counters in shared memory: a block scans one contiguous chunk of
// the table and touches each hot global counter once (same-address global atomics
// from every warp serialise in L2).  Keys that do not fit the shared table fall
// back to warp-aggregated global atomics.
constexpr int BK_SLOTS = 512;
struct BlockKeys {
  uint32_t key[BK_SLOTS];
  unsigned long long cnt[BK_SLOTS];
  unsigned long long base[BK_SLOTS];
};
__device__ __forceinline__ void bk_init(BlockKeys& B) {
  for (int i = threadIdx.x; i < BK_SLOTS; i += blockDim.x) { B.key[i] = EMPTY_TAG; B.cnt[i] = 0; B.base[i] = 0; }
}
// slot of key in B (claimed if absent), -1 when the table is full
__device__ __forceinline__ int bk_slot(BlockKeys& B, uint32_t key) {
  uint32_t h = (uint32_t)mix64(key) & (BK_SLOTS - 1);
  for (int p = 0; p < 32; ++p) {
    uint32_t old = *(volatile uint32_t*)&B.key[h];
    if (old == EMPTY_TAG) old = atomicCAS(&B.key[h], EMPTY_TAG, key);
    if (old == EMPTY_TAG || old == key) return (int)h;
    h = (h + 1) & (BK_SLOTS - 1);
  }
  return -1;
}
// warp-aggregated add of 1 per active lane to B[key]; returns the lane's slot (or -1)
__device__ __forceinline__ int bk_add(BlockKeys& B, bool active, uint32_t key) {
  const unsigned am = __ballot_sync(0xFFFFFFFFu, active);
  int sl = -1;
  if (active) {
    const unsigned g = __match_any_sync(am, key);
    const int lead = __ffs(g) - 1, lane = threadIdx.x & 31;
    if (lane == lead) {
      sl = bk_slot(B, key);
      if (sl >= 0) atomicAdd(&B.cnt[sl], (unsigned long long)__popc(g));
    }
    sl = __shfl_sync(g, sl, lead);
  }
  return sl;
}
__device__ __forceinline__ void block_chunk(uint64_t n, uint64_t& lo, uint64_t& hi) {
  const uint64_t per = (n + gridDim.x - 1) / gridDim.x;
  lo = (uint64_t)blockIdx.x * per;
  hi = lo + per < n ? lo + per : n;
  if (lo > hi) lo = hi;
}

__global__ void __launch_bounds__(256) k_occ_count(const uint32_t* bm, uint64_t nw, unsigned long long* total) {
  unsigned long long n = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nw; i += (uint64_t)gridDim.x * blockDim.x)
    n += __popc(bm[i]);
  for (int o = 16; o; o >>= 1) n += __shfl_xor_sync(0xFFFFFFFFu, n, o);
  if ((threadIdx.x & 31) == 0 && n) atomicAdd(total, n);
}

// the occupied slots of the value table, listed from its occupancy bitmap (order-free: every consumer
// aggregates); *total = their number (one warp-aggregated atomic per 32 bitmap words)
__global__ void __launch_bounds__(256) k_occ_list(const uint32_t* bm, uint64_t nw, uint32_t* flat,
                                                  unsigned long long* total) {
  const int lane = threadIdx.x & 31;
  for (uint64_t b = blockIdx.x * (uint64_t)blockDim.x; b < nw; b += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t i = b + threadIdx.x;
    uint32_t w = i < nw ? bm[i] : 0u;
    const uint32_t k = __popc(w);
    uint32_t x = k;                                    // inclusive warp scan of the counts
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, o);
      if (lane >= o) x += y;
    }
    const uint32_t wsum = __shfl_sync(0xFFFFFFFFu, x, 31);
    unsigned long long base = 0;
    if (lane == 31 && wsum) base = atomicAdd(total, (unsigned long long)wsum);
    base = __shfl_sync(0xFFFFFFFFu, base, 31) + (x - k);
    for (; w; w &= w - 1) flat[base++] = (uint32_t)((i << 5) + (uint32_t)(__ffs(w) - 1));
  }
}

// the distinct tags of the occupied slots (the table's occupancy list: O(entries), not O(capacity))
// and their entry counts
__global__ void k_tagscan(const HSlot* hs, const uint32_t* occ, const unsigned long long* n_occ, uint32_t* tags,
                          unsigned long long* tcnt, unsigned long long* ovf) {
  __shared__ BlockKeys B;
  bk_init(B);
  __syncthreads();
  uint64_t lo, hi;
  block_chunk(*n_occ, lo, hi);
  for (uint64_t b = lo; b < hi; b += blockDim.x) {
    const uint64_t j = b + threadIdx.x;
    const uint32_t tag = j < hi ? hs[occ[j]].tag : EMPTY_TAG;
    const bool act = tag != EMPTY_TAG;
    const int sl = bk_add(B, act, tag);
    if (act && sl < 0) {   // shared table full: count this entry globally
      uint32_t h = (uint32_t)mix64(tag) & (TAG_CAP - 1);
      bool done = false;
      for (int p = 0; p < 64 && !done; ++p) {
        uint32_t old = *(volatile uint32_t*)&tags[h];
        if (old == EMPTY_TAG) old = atomicCAS(&tags[h], EMPTY_TAG, tag);
        if (old == EMPTY_TAG || old == tag) done = true;
        else h = (h + 1) & (TAG_CAP - 1);
      }
      if (done) atomicAdd(&tcnt[h], 1ull);
      else atomicExch(ovf, 1ull);
    }
  }
  __syncthreads();
  for (int j = threadIdx.x; j < BK_SLOTS; j += blockDim.x) {
    const uint32_t tag = B.key[j];
    if (tag == EMPTY_TAG || !B.cnt[j]) continue;
    uint32_t h = (uint32_t)mix64(tag) & (TAG_CAP - 1);
    bool done = false;
    for (int p = 0; p < 64 && !done; ++p) {
      uint32_t old = *(volatile uint32_t*)&tags[h];
      if (old == EMPTY_TAG) old = atomicCAS(&tags[h], EMPTY_TAG, tag);
      if (old == EMPTY_TAG || old == tag) done = true;
      else h = (h + 1) & (TAG_CAP - 1);
    }
    if (done) atomicAdd(&tcnt[h], B.cnt[j]);
    else atomicExch(ovf, 1ull);
  }
}

// Direct keys' entries are written to their segment at positions reserved per block
// (count pass, one global reservation per key, scatter pass); the other keys'
// entries are aggregated in the view table.
__global__ void k_emit(const HSlot* hs, const unsigned long long* hc, const uint32_t* occ_idx,
                       const unsigned long long* n_occ, uint32_t n_pcs, const uint8_t* direct,
                       const unsigned long long* off, unsigned long long* cur, uint64_t* gb, uint64_t* gc, HSlot* vs,
                       unsigned long long* vc, uint64_t vmask, unsigned long long* ovf) {
  __shared__ BlockKeys B;
  bk_init(B);
  __syncthreads();
  uint64_t lo, hi;
  block_chunk(*n_occ, lo, hi);
  auto key_of = [&](uint32_t tag, int side, bool occ, bool& act, bool& dir) -> uint32_t {
    const uint32_t koi = tag & 0xFFFFu;
    act = occ && !(side == 1 && koi == KO_NONE);
    const uint32_t key = act ? (side == 0 ? (tag >> 16) : n_pcs + koi) : 0;
    dir = act && direct[key];
    return key;
  };
  // pass 1: per-key entry counts of the chunk (of the occupied-slot list)
  for (uint64_t b = lo; b < hi; b += blockDim.x) {
    const uint64_t j = b + threadIdx.x;
    const uint64_t i = j < hi ? occ_idx[j] : 0;
    const uint32_t tag = j < hi ? hs[i].tag : EMPTY_TAG;
    for (int side = 0; side < 2; ++side) {
      bool act, dir;
      const uint32_t key = key_of(tag, side, tag != EMPTY_TAG, act, dir);
      bk_add(B, dir, key);
    }
  }
  __syncthreads();
  // one reservation per key; the counts become the block's cursors
  for (int j = threadIdx.x; j < BK_SLOTS; j += blockDim.x) {
    const uint32_t key = B.key[j];
    if (key != EMPTY_TAG && B.cnt[j]) B.base[j] = off[key] + atomicAdd(&cur[key], B.cnt[j]);
    B.cnt[j] = 0;
  }
  __syncthreads();
  // pass 2: scatter (entries of keys that missed the shared table reserve globally)
  for (uint64_t b = lo; b < hi; b += blockDim.x) {
    const uint64_t j = b + threadIdx.x;
    const uint64_t i = j < hi ? occ_idx[j] : 0;
    const uint32_t tag = j < hi ? hs[i].tag : EMPTY_TAG;
    const bool occ = tag != EMPTY_TAG;
    const uint64_t bits = occ ? hs[i].bits : 0;
    const unsigned long long cnt = occ ? hc[i] : 0;
    for (int side = 0; side < 2; ++side) {
      bool act, dir;
      const uint32_t key = key_of(tag, side, occ, act, dir);
      const int lane = threadIdx.x & 31;
      const unsigned am = __ballot_sync(0xFFFFFFFFu, dir);
      if (dir) {
        const unsigned g = __match_any_sync(am, key);
        const int lead = __ffs(g) - 1;
        unsigned long long p = 0;
        if (lane == lead) {
          const int sl = bk_slot(B, key);
          p = sl >= 0 ? B.base[sl] + atomicAdd(&B.cnt[sl], (unsigned long long)__popc(g))
                      : off[key] + atomicAdd(&cur[key], (unsigned long long)__popc(g));
        }
        p = __shfl_sync(g, p, lead) + __popc(g & ((1u << lane) - 1u));
        gb[p] = bits;
        gc[p] = cnt;
      } else if (act) {
        vinsert(vs, vc, vmask, ovf, key, bits, cnt);
      }
    }
  }
}

// the distinct tags found by k_tagscan, compacted: out[0] = count, then (tag, entries)
// pairs (up to TAGL_MAX; the host falls back to the full table beyond)
constexpr uint32_t TAGL_MAX = 8192;
// one thread per tag-table entry, one claim per warp (out[0] zeroed before the launch)
__global__ void __launch_bounds__(256) k_tag_compact(const uint32_t* tags, const unsigned long long* tcnt,
                                                    unsigned long long* out) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  const bool f = i < TAG_CAP && tags[i] != EMPTY_TAG;
  const unsigned m = __ballot_sync(0xFFFFFFFFu, f);
  if (!m) return;
  const int lane = threadIdx.x & 31;
  unsigned long long base = 0;
  if (lane == 0) base = atomicAdd(&out[0], (unsigned long long)__popc(m));
  base = __shfl_sync(0xFFFFFFFFu, base, 0);
  if (f) {
    const unsigned long long p = base + __popc(m & ((1u << lane) - 1u));
    if (p < TAGL_MAX) { out[1 + 2 * p] = tags[i]; out[2 + 2 * p] = tcnt[i]; }
  }
}

// Exact n_distinct and top-k of every key (PC keys, then object keys).
ve_status finalize_hist(ve_ctx* c, cudaStream_t s, std::vector<uint64_t>& ndistinct,
                        std::vector<ve_topk_entry>& top) {
  const uint32_t nk = c->n_keys, K = c->cfg.topk, npc = c->cfg.n_pcs;
  ndistinct.assign(nk, 0);
  top.assign((size_t)nk * K, ve_topk_entry{0, 0});
  cudaError_t e;
  const int grid = c->num_sms * 4;
  // 1. distinct tags and their entry counts; the occupied slots, compacted
  uint32_t* d_tags = nullptr;
  unsigned long long* d_tcnt = nullptr;
  unsigned long long* d_small = nullptr;     // [0] overflow, [1] occupied slots
  unsigned long long* d_tl = nullptr;        // compacted tag list
  // occupied slot indices, listed from the occupancy bitmap (the count read back to size the list)
  const uint64_t nbw = c->hcap >> 5;
  {
    const size_t need = 16;
    if (c->occ_flat_bytes < need || !c->occ_flat) {
      c->occ_flat_bytes = 0;
      e = ctx_realloc(c, &c->occ_flat, 1 << 16);
      if (e != cudaSuccess) return cuda_fail(c, e, "finalize occupancy alloc");
      c->occ_flat_bytes = 1 << 16;
    }
  }
  // pass 1: count (the list is written in pass 2 once it fits)
  unsigned long long* d_cnt = (unsigned long long*)c->occ_flat;
  cudaMemsetAsync(d_cnt, 0, 8, s);
  count_launch();
  k_occ_count<<<c->num_sms * 4, 256, 0, s>>>(c->t.occ_bm, nbw, d_cnt);
  unsigned long long tot = 0;
  cudaMemcpyAsync(&tot, d_cnt, 8, cudaMemcpyDeviceToHost, s);
  e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c, e, "finalize occupancy");
  c->last_nocc = tot;
  {
    const size_t need = (size_t)tot * 4 + 16;
    if (c->occ_flat_bytes < need) {      // grow-only (ctx_realloc: no device sync)
      c->occ_flat_bytes = 0;
      e = ctx_realloc(c, &c->occ_flat, need + need / 4);
      if (e != cudaSuccess) return cuda_fail(c, e, "finalize occupancy alloc");
      c->occ_flat_bytes = need + need / 4;
    }
  }
  unsigned long long* d_nocc = (unsigned long long*)c->occ_flat;
  uint32_t* d_occ = (uint32_t*)((uint8_t*)c->occ_flat + 16);
  cudaMemsetAsync(d_nocc, 0, 8, s);
  count_launch();
  k_occ_list<<<c->num_sms * 4, 256, 0, s>>>(c->t.occ_bm, nbw, d_occ, d_nocc);
  if (c->hcap > 0xFFFFFFFFull) return fail(c, VE_ERR_INVALID, "finalize: hist_capacity above 2^32");
  e = cudaMallocAsync((void**)&d_tags, TAG_CAP * 4, s);
  if (e == cudaSuccess) e = cudaMallocAsync((void**)&d_tcnt, TAG_CAP * 8, s);
  if (e == cudaSuccess) e = cudaMallocAsync((void**)&d_small, 16, s);
  if (e == cudaSuccess) e = cudaMallocAsync((void**)&d_tl, (1 + 2 * TAGL_MAX) * 8, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "finalize alloc");
  if (!c->pin) {
    e = cudaMallocHost(&c->pin, (1 + 2 * TAGL_MAX) * 8 + 64);
    if (e != cudaSuccess) { c->pin = nullptr; return cuda_fail(c, e, "finalize pinned buffer"); }
  }
  unsigned long long* hp = (unsigned long long*)c->pin;
  cudaMemsetAsync(d_tags, 0xFF, TAG_CAP * 4, s);
  cudaMemsetAsync(d_tcnt, 0, TAG_CAP * 8, s);
  cudaMemsetAsync(d_small, 0, 16, s);
  stage("start", s);
  count_launch();
  k_tagscan<<<grid, 256, 0, s>>>(c->t.hslot, d_occ, d_nocc, d_tags, d_tcnt, d_small);
  count_launch();
  cudaMemsetAsync(d_tl, 0, 8, s);
  k_tag_compact<<<(TAG_CAP + 255) / 256, 256, 0, s>>>(d_tags, d_tcnt, d_tl);
  cudaMemcpyAsync(hp, d_tl, (1 + 2 * TAGL_MAX) * 8, cudaMemcpyDeviceToHost, s);
  cudaMemcpyAsync(hp + 1 + 2 * TAGL_MAX, d_small, 8, cudaMemcpyDeviceToHost, s);
  e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) { cudaFreeAsync(d_small, s); return cuda_fail(c, e, "finalize tags"); }
  unsigned long long ovf = hp[1 + 2 * TAGL_MAX];
  std::vector<uint32_t> tags;
  std::vector<unsigned long long> tcnt;
  if (hp[0] <= TAGL_MAX) {
    tags.resize(hp[0]);
    tcnt.resize(hp[0]);
    for (size_t i = 0; i < hp[0]; ++i) { tags[i] = (uint32_t)hp[1 + 2 * i]; tcnt[i] = hp[2 + 2 * i]; }
  } else {
    tags.resize(TAG_CAP);
    tcnt.resize(TAG_CAP);
    cudaMemcpyAsync(tags.data(), d_tags, TAG_CAP * 4, cudaMemcpyDeviceToHost, s);
    cudaMemcpyAsync(tcnt.data(), d_tcnt, TAG_CAP * 8, cudaMemcpyDeviceToHost, s);
    e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) { cudaFreeAsync(d_small, s); return cuda_fail(c, e, "finalize tags"); }
  }
  cudaFreeAsync(d_tags, s);
  cudaFreeAsync(d_tcnt, s);
  cudaFreeAsync(d_tl, s);
  stage("tagscan+d2h", s);
  if (ovf) {                                  // too many distinct tags: aggregate every key
    cudaFreeAsync(d_small, s);
    ViewTable V;
    ve_status st = build_views(c, s, V);
    if (st == VE_OK) st = view_topk(c, V, s, ndistinct, top);
    free_views(V, s);
    return st;
  }
  // 2. classify keys: direct (one tag) or aggregated (several tags)
  std::vector<uint32_t> ntag(nk, 0);
  std::vector<uint64_t> ent(nk, 0);
  for (size_t i = 0; i < tags.size(); ++i) {
    if (tags[i] == EMPTY_TAG) continue;
    const uint32_t pk = tags[i] >> 16, koi = tags[i] & 0xFFFFu;
    ntag[pk]++;
    ent[pk] += tcnt[i];
    if (koi != KO_NONE) {
      ntag[npc + koi]++;
      ent[npc + koi] += tcnt[i];
    }
  }
  std::vector<uint8_t> direct(nk, 0);
  std::vector<unsigned long long> off(nk, 0);
  uint64_t pos = 0, agg_in = 0;
  for (uint32_t k = 0; k < nk; ++k) {
    if (ntag[k] == 1) {
      direct[k] = 1;
      off[k] = pos;
      ndistinct[k] = ent[k];
      pos += ent[k];
    } else if (ntag[k] > 1) {
      agg_in += ent[k];
    }
  }
  const uint64_t nent = pos + agg_in + 1;
  uint64_t* gbuf = nullptr;
  uint8_t* d_direct = nullptr;
  unsigned long long* d_off = nullptr;      // off, cur
  e = cudaMallocAsync((void**)&gbuf, 4 * nent * 8, s);
  if (e == cudaSuccess) e = cudaMallocAsync((void**)&d_direct, nk, s);
  if (e == cudaSuccess) e = cudaMallocAsync((void**)&d_off, 16ull * nk, s);
  if (e != cudaSuccess) { cudaFreeAsync(d_small, s); return cuda_fail(c, e, "finalize alloc"); }
  uint64_t* gb[2] = {gbuf, gbuf + 2 * nent};
  uint64_t* gc[2] = {gbuf + nent, gbuf + 3 * nent};
  cudaMemcpyAsync(d_direct, direct.data(), nk, cudaMemcpyHostToDevice, s);
  cudaMemcpyAsync(d_off, off.data(), 8ull * nk, cudaMemcpyHostToDevice, s);
  cudaMemsetAsync(d_off + nk, 0, 8ull * nk, s);
  ViewTable V;
  ve_status st = VE_OK;
  if (agg_in) st = alloc_views(c, s, agg_in, V);
  if (st != VE_OK) { cudaFreeAsync(d_small, s); return st; }
  stage("alloc", s);
  // 3. emit direct keys' entries, aggregate the others in the view table
  count_launch();
  k_emit<<<grid, 256, 0, s>>>(c->t.hslot, c->t.hcount, d_occ, d_nocc, npc, d_direct, d_off, d_off + nk, gb[0],
                              gc[0], V.vs, V.vc, V.vcap ? V.vcap - 1 : 0, d_small);
  if (agg_in) {
    unsigned long long* d_nd = nullptr;
    cudaMallocAsync((void**)&d_nd, 8ull * nk, s);
    cudaMemsetAsync(d_nd, 0, 8ull * nk, s);
    count_launch();
    k_view_count<<<grid, 256, 0, s>>>(V.vs, V.vcap, d_nd);
    std::vector<uint64_t> nd(nk);
    cudaMemcpyAsync(nd.data(), d_nd, 8ull * nk, cudaMemcpyDeviceToHost, s);
    cudaFreeAsync(d_nd, s);
    e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) { cudaFreeAsync(d_small, s); return cuda_fail(c, e, "finalize views"); }
    for (uint32_t k = 0; k < nk; ++k)
      if (!direct[k] && nd[k]) {
        off[k] = pos;
        ndistinct[k] = nd[k];
        pos += nd[k];
      }
    cudaMemcpyAsync(d_off, off.data(), 8ull * nk, cudaMemcpyHostToDevice, s);
    count_launch();
    k_view_scatter<<<grid, 256, 0, s>>>(V.vs, V.vc, V.vcap, d_off, d_off + nk, gb[0], gc[0]);
  }
  stage("emit+views", s);
  // 4. top-k per key
  std::vector<uint64_t> len(ndistinct.begin(), ndistinct.end()), start(off.begin(), off.end());
  st = select_topk(c, s, gb, gc, len, start, top);
  stage("select_topk", s);
  unsigned long long h_ovf = 0;
  cudaMemcpyAsync(&h_ovf, d_small, 8, cudaMemcpyDeviceToHost, s);
  free_views(V, s);
  cudaFreeAsync(gbuf, s);
  cudaFreeAsync(d_direct, s);
  cudaFreeAsync(d_off, s);
  cudaFreeAsync(d_small, s);
  e = cudaStreamSynchronize(s);
  if (st != VE_OK) return st;
  if (e != cudaSuccess) return cuda_fail(c, e, "finalize");
  if (h_ovf) return fail(c, VE_ERR_CAPACITY, "finalize: view table overflow");
  return VE_OK;
}

// (reference path: every key aggregated through the view table)
ve_status finalize_hist_views(ve_ctx* c, cudaStream_t s, std::vector<uint64_t>& ndistinct,
                              std::vector<ve_topk_entry>& top) {
  ViewTable V;
  ve_status st = build_views(c, s, V);
  if (st == VE_OK) st = view_topk(c, V, s, ndistinct, top);
  free_views(V, s);
  return st;
}

// ---- dense per-element counts -> exact histogram ------------------------------
// (one array per launch: the path of claims whose counts are mostly 0 -- sparse or high-cardinality reads)
// A dense counter cnt[e] of (pc, object) counts loads that read element e's unchanged
// pre-snapshot value, so it contributes cnt[e] occurrences of that value (C9).
// Each block aggregates its chunk of elements by value (warp match, then a small
// shared table) so runs of equal values (zero-filled regions) cost one global insert.
constexpr int DF_THREADS = 256;
constexpr int DF_SLOTS = 1024;
#ifndef VE_DF_CHUNK
#define VE_DF_CHUNK 2048
#endif
constexpr uint64_t DF_CHUNK = VE_DF_CHUNK;    // elements per block: many blocks keep the global inserts in flight

// The value statistics of the counted loads (C1 n_zero, C5 flags and ord range, C4 raw
// range, C7 truncated range) are taken here too, once per element weighted by its
// count: a counted load's value IS the element's pre value (k_analyze skips them).
struct DenseVal {
  unsigned long long s[6];   // zero, nan, nonint, not_f16, not_bf16, not_f32
  unsigned long long mn[3], mx[3];   // raw, ord, trunc
};
__device__ __forceinline__ unsigned long long wsum64(unsigned long long v) {
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xFFFFFFFFu, v, o);
  return v;
}
__device__ __forceinline__ unsigned long long wmin64(unsigned long long v) {
  for (int o = 16; o; o >>= 1) { const unsigned long long w = __shfl_xor_sync(0xFFFFFFFFu, v, o); v = w < v ? w : v; }
  return v;
}
__device__ __forceinline__ unsigned long long wmax64(unsigned long long v) {
  for (int o = 16; o; o >>= 1) { const unsigned long long w = __shfl_xor_sync(0xFFFFFFFFu, v, o); v = w > v ? w : v; }
  return v;
}

// Shared table of `ts` slots (dynamic shared memory: ts u64 value bits, then ts u32
// counts).  Blocks walk chunks of DF_CHUNK elements (chunk c, c + grid, ...).  The many-
// block launch (one chunk per block, ts = DF_SLOTS) keeps many HBM-table inserts in
// flight for high-cardinality arrays; the persistent launch (two blocks per SM, ts =
// DF_LC_SLOTS) aggregates a low-cardinality array across all its chunks, so each block
// inserts each distinct value about once.  A table filled past half is emptied into the
// HBM table between chunks.  Counts per block stay < 2^32 (dense counting is on only
// while the ctx has seen < 2^32 records).
constexpr uint32_t DF_LC_SLOTS = 8192;
constexpr uint32_t DF_LC_CHUNK = 32768;
constexpr uint64_t DF_PROBE_MIN = 1ull << 24;   // arrays probed for low cardinality   // elements between table-fill checks (persistent blocks)

// value statistics of `k` counted loads that read the value bits b (C1 n_zero, C5 flags
// and ord range, C4 raw range, C7 truncated range), accumulated per thread
__device__ __forceinline__ void df_stats(DenseVal& v, uint64_t b, unsigned long long k, uint32_t kind, uint32_t lg,
                                         uint32_t mant_bits) {
  if (b == 0ull) v.s[0] += k;
  uint32_t ff = 0;
  if (kind >= 2u) {
    int64_t ival;
    ff = float_flags(b, kind, lg, ival);
    for (int j = 0; j < 5; ++j) if (ff & (1u << j)) v.s[1 + j] += k;
  }
  v.mn[0] = b < v.mn[0] ? b : v.mn[0];
  v.mx[0] = b > v.mx[0] ? b : v.mx[0];
  if (!(ff & 1u)) {                    // NaNs excluded from ord / trunc (C5, C7)
    const uint64_t o = ord_key(b, kind, lg);
    v.mn[1] = o < v.mn[1] ? o : v.mn[1];
    v.mx[1] = o > v.mx[1] ? o : v.mx[1];
    if (kind >= 2u) {
      const uint64_t tr = trunc_bits(b, kind, lg, mant_bits);
      v.mn[2] = tr < v.mn[2] ? tr : v.mn[2];
      v.mx[2] = tr > v.mx[2] ? tr : v.mx[2];
    }
  }
}

// empty the block's table into the HBM table, taking each entry's value statistics once
__device__ __forceinline__ void df_table_flush(unsigned long long* sbits, uint32_t* scnt, uint32_t ts, uint32_t tag,
                                               DevTables& t, DenseVal& v, uint32_t kind, uint32_t lg,
                                               uint32_t mant_bits) {
  for (uint32_t i = threadIdx.x; i < ts; i += blockDim.x) {
    if (sbits[i] != ~0ull && scnt[i]) {
      df_stats(v, sbits[i], scnt[i], kind, lg, mant_bits);
      hist_insert_global_rf(t, tag, sbits[i], scnt[i]);
    }
    sbits[i] = ~0ull;
    scnt[i] = 0;
  }
}

template <int NT>
__global__ void __launch_bounds__(NT, 1) k_dense_flush(uint32_t* cnt, uint64_t n_elems, const uint8_t* pre,
                                                           uint32_t ew, uint32_t tag, uint64_t bmoff, DevTables t,
                                                           uint32_t meta, uint32_t mant_bits, uint32_t kp, uint32_t ko,
                                                           uint32_t ts, uint32_t csz, uint32_t setL,
                                                           const uint32_t* only_if = nullptr) {
  // (only_if: the fallback of the per-object flush -- run only when its table overflowed)
  if (only_if && *(volatile const uint32_t*)only_if == 0u) return;
  extern __shared__ unsigned long long df_smem[];
  unsigned long long* sbits = df_smem;
  uint32_t* scnt = reinterpret_cast<uint32_t*>(df_smem + ts);
  __shared__ DenseVal sv;
  __shared__ uint32_t sfill;
  for (uint32_t i = threadIdx.x; i < ts; i += NT) { sbits[i] = ~0ull; scnt[i] = 0; }
  if (threadIdx.x < 6) sv.s[threadIdx.x] = 0;
  if (threadIdx.x < 3) { sv.mn[threadIdx.x] = ~0ull; sv.mx[threadIdx.x] = 0; }
  if (threadIdx.x == 0) sfill = 0;
  const uint32_t kind = (meta >> 2) & 3u, lg = meta & 3u;
  DenseVal v;
  for (int i = 0; i < 6; ++i) v.s[i] = 0;
  for (int i = 0; i < 3; ++i) { v.mn[i] = ~0ull; v.mx[i] = 0; }
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const uint64_t nchunks = (n_elems + csz - 1) / csz;
  for (uint64_t ch = blockIdx.x; ch < nchunks; ch += gridDim.x) {
  const uint64_t lo = ch * csz, hi = lo + csz < n_elems ? lo + csz : n_elems;
  for (uint64_t base = lo; base < hi; base += NT) {
    const uint64_t e = base + threadIdx.x;
    uint32_t k = 0;
    uint64_t bits = 0;
    if (e < hi) {
      k = cnt[e];
      if (k) {
        cnt[e] = 0;
        const uint8_t* p = pre + e * ew;
        if (((uintptr_t)p & (ew - 1)) == 0) {
          bits = ew == 1 ? *p : ew == 2 ? *(const uint16_t*)p : ew == 4 ? *(const uint32_t*)p : *(const uint64_t*)p;
        } else {
          for (uint32_t i = 0; i < ew; ++i) bits |= (uint64_t)p[i] << (8 * i);
        }
      }
    }
    const unsigned km = __ballot_sync(0xFFFFFFFFu, k != 0);
    // C3: a counted load started at element e (K1 leaves these L bits to us); the
    // warp's 32 elements are one aligned bitmap word
    if (setL && lane == 0 && km) atomicOr(&t.L[bmoff + ((base + threadIdx.x) >> 5)], km);
    if (k) {
      const unsigned g = __match_any_sync(km, bits);
      // (a REDUX under per-lane group masks runs once per distinct mask: singletons skip it)
      const unsigned long long sum = __popc(g) == 1 ? (unsigned long long)k : __reduce_add_sync(g, k);
      if (lane == __ffs(g) - 1) {
        // shared slots are claimed by a 64-bit CAS of the value itself (empty = ~0, which
        // only an 8-byte element can hold: such values go straight to the global table)
        uint32_t h = (uint32_t)hist_hash(tag, bits) & (ts - 1);
        bool done = false;
        for (int probe = 0; probe < 8 && !done && ts && bits != ~0ull; ++probe) {   // (ts 0: direct)
          // look first (a warm table mostly holds the value already), claim only empty slots
          unsigned long long cur = *(volatile unsigned long long*)&sbits[h];
          if (cur == ~0ull) {
            cur = atomicCAS(&sbits[h], ~0ull, bits);
            if (cur == ~0ull) {
              atomicAdd(&sfill, 1u);
              cur = bits;
            }
          }
          if (cur == bits) {
            atomicAdd(&scnt[h], (uint32_t)sum);
            done = true;
          }
          h = (h + 1) & (ts - 1);
        }
        if (!done) {                     // straight to the HBM table: its statistics now
          df_stats(v, bits, sum, kind, lg, mant_bits);
          hist_insert_global_rf(t, tag, bits, sum);
        }
      }
    }
  }
  __syncthreads();
  if (sfill > ts / 2) {                    // a table past half full: empty it between chunks
    df_table_flush(sbits, scnt, ts, tag, t, v, kind, lg, mant_bits);
    __syncthreads();
    if (threadIdx.x == 0) sfill = 0;
    __syncthreads();
  }
  }
  __syncthreads();
  df_table_flush(sbits, scnt, ts, tag, t, v, kind, lg, mant_bits);
  // value statistics: warp, block, then both keys' rows (PC key kp, object key ko)
  for (int i = 0; i < 6; ++i) {
    const unsigned long long x = wsum64(v.s[i]);
    if (lane == 0 && x) atomicAdd(&sv.s[i], x);
  }
  for (int i = 0; i < 3; ++i) {
    const unsigned long long a = wmin64(v.mn[i]), b = wmax64(v.mx[i]);
    if (lane == 0) { atomicMin(&sv.mn[i], a); atomicMax(&sv.mx[i], b); }
  }
  __syncthreads();
  if (threadIdx.x < 2) {
    const uint64_t key = threadIdx.x ? ko : kp;
    const int f[6] = {F_ZERO, F_NAN, F_NONINT, F_NF16, F_NBF16, F_NF32};
    for (int i = 0; i < 6; ++i)
      if (sv.s[i]) atomicAdd(&t.sum[key * NSUM + f[i]], sv.s[i]);
    for (int i = 0; i < 3; ++i) {
      if (sv.mn[i] != ~0ull) atomicMin(&t.mn[key * NMM + i], sv.mn[i]);
      if (sv.mx[i] != 0ull) atomicMax(&t.mx[key * NMM + i], sv.mx[i]);
    }
  }
}

// Cardinality probe of a dense array: the distinct values among up to 64 Ki counted
// elements sampled at a fixed stride (one block); out[0] = distinct (capped near 4096).
struct SampleJob {
  const uint32_t* cnt;
  const uint8_t* pre;     // the claim's side snapshot
  uint64_t n_elems;
  uint32_t ew, pad;
};
__device__ void dense_sample_body(const uint32_t* cnt, uint64_t n_elems, const uint8_t* pre, uint32_t ew,
                                  unsigned int* out);
// every claim's cardinality probe in one launch (one block per claim)
__global__ void __launch_bounds__(1024) k_dense_sample_many(const SampleJob* jobs, unsigned int* out) {
  const SampleJob j = jobs[blockIdx.x];
  dense_sample_body(j.cnt, j.n_elems, j.pre, j.ew, out + blockIdx.x);
}
__global__ void __launch_bounds__(1024) k_dense_sample(const uint32_t* cnt, uint64_t n_elems, const uint8_t* pre,
                                                      uint32_t ew, unsigned int* out) {
  dense_sample_body(cnt, n_elems, pre, ew, out);
}
__device__ void dense_sample_body(const uint32_t* cnt, uint64_t n_elems, const uint8_t* pre, uint32_t ew,
                                  unsigned int* out) {
  extern __shared__ unsigned long long tb[];   // 8192 slots (dynamic: 64 KiB)
  __shared__ unsigned int nd;
  for (int i = threadIdx.x; i < 8192; i += 1024) tb[i] = ~0ull;
  if (threadIdx.x == 0) nd = 0;
  __syncthreads();
  const uint64_t stride = n_elems > 65536 ? n_elems / 65536 : 1;
  for (uint64_t s = threadIdx.x; s < 65536 && s * stride < n_elems; s += 1024) {
    if (*(volatile unsigned int*)&nd > 4096) break;
    const uint64_t e = s * stride;
    if (!cnt[e]) continue;
    const uint8_t* p = pre + e * ew;
    uint64_t bits = 0;
    for (uint32_t i = 0; i < ew; ++i) bits |= (uint64_t)p[i] << (8 * i);
    if (bits == ~0ull) bits = ~1ull;   // (the probe only estimates)
    uint32_t h = (uint32_t)mix64(bits) & 8191u;
    for (int probe = 0; probe < 64; ++probe) {
      unsigned long long old = *(volatile unsigned long long*)&tb[h];   // look first: no CAS storm on one value
      if (old == bits) break;
      if (old == ~0ull) {
        old = atomicCAS(&tb[h], ~0ull, bits);
        if (old == ~0ull) { atomicAdd(&nd, 1u); break; }
        if (old == bits) break;
      }
      h = (h + 1) & 8191u;
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) out[0] = nd;
}

// ---- fused per-object flush of the dense counters (all claims of one object in one pass) --------
// Every claim j of object o counts, per element e, the records of one (pc, access type) whose value
// was e's PRE value (side 0, loads) or e's POST value (side 1, DENSE_POST): their histogram entries
// are (tag_j, side value of e) with count c_j(e).  One pass over the object reads each snapshot side
// once and every claim's counters (k_dense_obj) and aggregates
//   H0_side(v) = #elements with side value v (one insert per element and side), and
//   D_j(v)    = sum of (c_j(e) - m_j) over the elements where c_j(e) != m_j,
// m_j being the claim's base multiplicity (the mode of c_j over 32 sampled elements): stencils read
// every element once per PC, so H0 carries the whole count and corrections are few (clamped faces).
// Then (k_dense_emit) claim j's count of v over the object is m_j * H0_side(v) + D_j(v); positive
// counts go to the HBM table with their value statistics (C1 n_zero, C4-C7), so no zero-count entry
// is ever created.
constexpr int DO_THREADS = 1024;
// table slots (block and global): 16 bytes {value bits, cls << 56 | (count + 2^55)}: cls 0 / 1 = H0 of
// the pre / post side, 2 + j = correction of claim j; the biased 56-bit count takes signed adds
constexpr uint32_t DO_TS = 12288;                // 192 KiB of shared memory
constexpr uint64_t DO_EMPTY = 0xFFull << 56;
constexpr uint64_t DO_BIAS = 1ull << 55;
constexpr uint64_t DO_M56 = (1ull << 56) - 1ull;
constexpr int DO_MAXC = DENSE_PER_OBJ;
constexpr uint64_t DO_CH = 65536;               // elements per chunk
struct DoClaim {
  uint32_t* cnt;        // counters (zeroed by the flush)
  uint32_t tag, meta;   // (pc << 16 | object id), access type
  uint32_t side, kp;    // 0 pre / 1 post; PC key row
  uint32_t m, pad;      // base multiplicity (>= 1): the mode of the counts, sampled by k_dense_mode
};
struct DoArgs {
  DoClaim c[DO_MAXC];
  uint32_t nc, ew, ko, mant_bits;
  uint64_t ne;          // whole elements
  const uint8_t* snap[2];
  uint64_t bmoff;
};
struct DoStat {          // per-claim value statistics (shared, then the two key rows)
  unsigned long long s[6];   // zero, nan, nonint, not_f16, not_bf16, not_f32
  unsigned long long mn[3], mx[3];
};

__device__ __forceinline__ uint64_t do_load(const uint8_t* p, uint32_t ew) {
  return ew == 1 ? *p : ew == 2 ? *(const uint16_t*)p : ew == 4 ? *(const uint32_t*)p : *(const uint64_t*)p;
}

struct DoSlot {
  uint64_t v, w;        // value bits; cls << 56 | biased count
};
__device__ __forceinline__ uint32_t do_h(uint32_t cls, uint64_t v) {
  uint32_t h = ((uint32_t)v ^ (uint32_t)(v >> 32) ^ (cls * 0x9E3779B9u)) * 0x85EBCA6Bu;
  h ^= h >> 15;
  h *= 0xC2B2AE35u;
  h ^= h >> 13;
  return (uint32_t)(((uint64_t)h * DO_TS) >> 32);
}
// add d to (cls, v) in the block table (claims a slot with a 128-bit CAS); false when 64 probes found
// no place
__device__ __forceinline__ bool do_add(DoSlot* ts, uint32_t cls, uint64_t v, long long d, uint32_t* fill) {
  uint32_t h = do_h(cls, v);
  for (int probe = 0; probe < 64; ++probe) {
    DoSlot* s = &ts[h];
    uint64_t lo, hi;
    asm volatile("ld.volatile.shared.v2.u64 {%0, %1}, [%2];"
                 : "=l"(lo), "=l"(hi) : "r"((uint32_t)__cvta_generic_to_shared(s)) : "memory");
    const uint32_t sc = (uint32_t)(hi >> 56);
    // (an empty slot reads (0, EMPTY): a match of value 0 is confirmed by the CAS, never taken from the read)
    if (sc == cls && lo == v && v != 0ull) { atomicAdd((unsigned long long*)&s->w, (unsigned long long)d); return true; }
    if (sc == 0xFFu || (sc == cls && lo == v)) {
      uint64_t olo, ohi;
      cas128_shared(s, 0ull, DO_EMPTY, v, ((uint64_t)cls << 56) | DO_BIAS, olo, ohi);
      if (ohi == DO_EMPTY && olo == 0ull) {
        atomicAdd(fill, 1u);
        atomicAdd((unsigned long long*)&s->w, (unsigned long long)d);
        return true;
      }
      if ((uint32_t)(ohi >> 56) == cls && olo == v) {
        atomicAdd((unsigned long long*)&s->w, (unsigned long long)d);
        return true;
      }
    }
    h = h + 1 == DO_TS ? 0u : h + 1;
  }
  return false;
}
__device__ __forceinline__ long long do_cnt(uint64_t w) { return (long long)(w & DO_M56) - (long long)DO_BIAS; }
// read-only lookup (no concurrent writers): the count of (cls, v), 0 if absent
__device__ __forceinline__ long long do_get(const DoSlot* ts, uint32_t cls, uint64_t v) {
  uint32_t h = do_h(cls, v);
  for (int probe = 0; probe < 64; ++probe) {
    const DoSlot& s = ts[h];
    const uint32_t sc = (uint32_t)(s.w >> 56);
    if (sc == 0xFFu) return 0;
    if (sc == cls && s.v == v) return do_cnt(s.w);
    h = h + 1 == DO_TS ? 0u : h + 1;
  }
  return 0;
}

// value statistics of k counted records that carry the bits v (C1 n_zero, C5 flags and ord range,
// C4 raw range, C7 truncated range), accumulated per thread
struct DoAcc {
  unsigned long long s[6];
  unsigned long long mn[3], mx[3];
};
__device__ __forceinline__ void do_acc_init(DoAcc& a) {
#pragma unroll
  for (int i = 0; i < 6; ++i) a.s[i] = 0;
#pragma unroll
  for (int i = 0; i < 3; ++i) { a.mn[i] = ~0ull; a.mx[i] = 0; }
}
__device__ __forceinline__ void do_acc(DoAcc& a, uint64_t v, unsigned long long k, uint32_t meta, uint32_t mant_bits) {
  const uint32_t kind = (meta >> 2) & 3u, lg = meta & 3u;
  if (v == 0ull) a.s[0] += k;
  uint32_t ff = 0;
  if (kind >= 2u) {
    int64_t ival;
    ff = float_flags(v, kind, lg, ival);
#pragma unroll
    for (int i = 0; i < 5; ++i) if (ff & (1u << i)) a.s[1 + i] += k;
  }
  a.mn[0] = v < a.mn[0] ? v : a.mn[0];
  a.mx[0] = v > a.mx[0] ? v : a.mx[0];
  if (!(ff & 1u)) {                        // NaNs excluded from ord / trunc (C5, C7)
    const uint64_t o = ord_key(v, kind, lg);
    a.mn[1] = o < a.mn[1] ? o : a.mn[1];
    a.mx[1] = o > a.mx[1] ? o : a.mx[1];
    if (kind >= 2u) {
      const uint64_t tr = trunc_bits(v, kind, lg, mant_bits);
      a.mn[2] = tr < a.mn[2] ? tr : a.mn[2];
      a.mx[2] = tr > a.mx[2] ? tr : a.mx[2];
    }
  }
}
// fold a thread's statistics into the block's row of claim j (a warp reduction first)
__device__ __forceinline__ void do_acc_fold(DoStat& S, DoAcc& a) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int i = 0; i < 6; ++i) {
    unsigned long long x = a.s[i];
    for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(0xFFFFFFFFu, x, o);
    if (lane == 0 && x) atomicAdd(&S.s[i], x);
  }
#pragma unroll
  for (int i = 0; i < 3; ++i) {
    unsigned long long x = a.mn[i], y = a.mx[i];
    for (int o = 16; o; o >>= 1) {
      const unsigned long long xx = __shfl_xor_sync(0xFFFFFFFFu, x, o), yy = __shfl_xor_sync(0xFFFFFFFFu, y, o);
      x = xx < x ? xx : x;
      y = yy > y ? yy : y;
    }
    if (lane == 0) {
      if (x != ~0ull) atomicMin(&S.mn[i], x);
      if (y != 0ull) atomicMax(&S.mx[i], y);
    }
  }
}

// base multiplicity of every claim: the most frequent count among 32 pseudo-random elements
// (one warp per claim; a regular stride could land on a stencil's faces every time)
__global__ void k_dense_mode(const uint32_t* const* cnt, const uint64_t* ne, uint32_t* m) {
  const int lane = threadIdx.x & 31;
  const uint32_t j = blockIdx.x;
  const uint64_t n = ne[j];
  const uint64_t e = n ? mix64(((uint64_t)j << 32) ^ (uint64_t)lane ^ 0x5bd1e995ull) % n : 0;
  const uint32_t c = n ? cnt[j][e] : 0u;
  const unsigned g = __match_any_sync(0xFFFFFFFFu, c);
  const uint32_t best = __reduce_max_sync(0xFFFFFFFFu, ((uint32_t)__popc(g) << 5) | (31u - (uint32_t)lane));
  const uint32_t mm = __shfl_sync(0xFFFFFFFFu, c, 31 - (int)(best & 31u));
  if (lane == 0) m[j] = mm;
}

// The object's (class, value) table in global memory: H0 of each side and the corrections D_j,
// same slot format as the block table (empty = all ones).  Sized by the host from the sampled
// cardinality; a full table sets *ovf and the claims take the per-array flush instead (exact).
__device__ __forceinline__ bool gt_add(DoSlot* gt, uint32_t mask, uint32_t cls, uint64_t v, long long d, uint32_t* ovf) {
  uint32_t h = (uint32_t)mix64(v ^ ((uint64_t)cls << 58)) & mask;
  for (uint32_t probe = 0; probe <= mask && probe < 256u; ++probe) {
    DoSlot* sl = &gt[h];
    uint64_t lo, hi;
    ld128_volatile(sl, lo, hi);
    const uint32_t sc = (uint32_t)(hi >> 56);
    // (an empty slot reads (~0, ~0): a match of value ~0 is confirmed by the CAS, never taken from the read)
    if (sc == cls && lo == v && v != ~0ull) { atomicAdd((unsigned long long*)&sl->w, (unsigned long long)d); return true; }
    if (sc == 0xFFu || (sc == cls && lo == v)) {
      uint64_t olo, ohi;
      cas128_global(sl, ~0ull, ~0ull, v, ((uint64_t)cls << 56) | DO_BIAS, olo, ohi);
      if ((olo == ~0ull && ohi == ~0ull) || ((uint32_t)(ohi >> 56) == cls && olo == v)) {
        atomicAdd((unsigned long long*)&sl->w, (unsigned long long)d);
        return true;
      }
    }
    h = (h + 1) & mask;
  }
  atomicExch(ovf, 1u);
  return false;
}
__device__ __forceinline__ long long gt_get(const DoSlot* gt, uint32_t mask, uint32_t cls, uint64_t v) {
  uint32_t h = (uint32_t)mix64(v ^ ((uint64_t)cls << 58)) & mask;
  for (uint32_t probe = 0; probe <= mask && probe < 256u; ++probe) {
    const DoSlot& sl = gt[h];
    const uint32_t sc = (uint32_t)(sl.w >> 56);
    if (sc == 0xFFu && sl.v == ~0ull) return 0;
    if (sc == cls && sl.v == v) return do_cnt(sl.w);
    h = (h + 1) & mask;
  }
  return 0;
}

// Pass 1 of the per-object flush: one read of every claim's counters and of each snapshot side.
// H0 goes to the block table (one insert per element and side; values that do not fit go to the
// global table), corrections (elements where c_j(e) != m_j: a stencil's clamped faces) straight to
// the global table; at exit the block table is added into the global one.  No block barrier in the
// loop and no per-claim emission here: the block table holds H0 only, so it never needs draining
// (round 2's version drained it every few chunks -- 7 x 4096 contended HBM inserts per drain --
// and checked its fill under a barrier every 8 batches: 20.6% of its stall samples).  The counters
// are left as they are (zeroed by a memset after the emission, or by the fallback flush).
// NC: the claims' loops run NC iterations (an instantiation per bound: a single-claim object -- T_out's
// post values, vol, a -- does not pay for eight predicated iterations per element)
template <int NC>
__global__ void __launch_bounds__(DO_THREADS, 1) k_dense_obj(const __grid_constant__ DoArgs A, DevTables t, DoSlot* gt,
                                                             uint32_t gmask, uint32_t* ovf) {
  extern __shared__ __align__(16) uint8_t do_smem[];
  DoSlot* ts = reinterpret_cast<DoSlot*>(do_smem);
  __shared__ uint32_t s_fill;
  const int tid = threadIdx.x, lane = tid & 31;
  for (uint32_t i = tid; i < DO_TS; i += blockDim.x) { ts[i].v = 0; ts[i].w = DO_EMPTY; }
  if (tid == 0) s_fill = 0;
  uint32_t sides = 0;                                  // bit s: some claim reads side s
  for (uint32_t j = 0; j < A.nc; ++j) sides |= 1u << A.c[j].side;
  __syncthreads();
  const uint64_t nch = (A.ne + DO_CH - 1) / DO_CH;
  for (uint64_t ch = blockIdx.x; ch < nch; ch += gridDim.x) {
    const uint64_t lo = ch * DO_CH, hi = lo + DO_CH < A.ne ? lo + DO_CH : A.ne;
    // the loads of a batch (the counters of all claims, the snapshot sides) are issued one batch
    // ahead, so they are in flight while the previous batch is inserted
    uint32_t ncj[NC];
    uint64_t nsv0 = 0, nsv1 = 0;
    auto issue = [&](uint64_t b) {
      const uint64_t e = b + tid;
      const bool in = e < hi;
#pragma unroll
      for (int j = 0; j < NC; ++j) ncj[j] = ((uint32_t)j < A.nc && in) ? __ldcs(A.c[j].cnt + e) : 0u;
      nsv0 = (in && A.snap[0]) ? do_load(A.snap[0] + e * A.ew, A.ew) : 0ull;
      nsv1 = (in && A.snap[1]) ? do_load(A.snap[1] + e * A.ew, A.ew) : 0ull;
    };
    issue(lo);
    for (uint64_t base = lo; base < hi; base += DO_THREADS) {
      const uint64_t e = base + tid;
      const bool in = e < hi;
      uint32_t cj[NC];
#pragma unroll
      for (int j = 0; j < NC; ++j) cj[j] = ncj[j];
      const uint64_t sv0 = nsv0, sv1 = nsv1;
      if (base + DO_THREADS < hi) issue(base + DO_THREADS);
      uint32_t corr = 0;                               // claims whose count differs from their base
      bool lbit = false;
#pragma unroll
      for (int j = 0; j < NC; ++j) {
        if ((uint32_t)j >= A.nc) break;
        if (cj[j] && A.c[j].side == 0u) lbit = true;
        if (in && cj[j] != A.c[j].m) corr |= 1u << j;
      }
      // C3: a counted pre-value load started at element e (K1 leaves these L bits to the flush)
      const unsigned lm = __ballot_sync(0xFFFFFFFFu, lbit);
      if (lane == 0 && lm) atomicOr(&t.L[A.bmoff + (base + (uint64_t)(tid & ~31)) / 32], lm);
      // H0: no MATCH (it costs more than the shared atomics it would merge on a varied side)
#pragma unroll
      for (int sd = 0; sd < 2; ++sd) {
        if (!((sides >> sd) & 1u)) continue;
        const uint64_t v = sd ? sv1 : sv0;
        const unsigned am = __ballot_sync(0xFFFFFFFFu, in);
        if (!am) continue;
        const int l0 = __ffs(am) - 1;
        const uint64_t v0 = ((uint64_t)__shfl_sync(0xFFFFFFFFu, (uint32_t)(v >> 32), l0) << 32) |
                            __shfl_sync(0xFFFFFFFFu, (uint32_t)v, l0);
        // the lanes holding lane l0's value form one group (all of them for a = 1.0 or vol; most
        // for a mostly-constant side), the others insert one element each
        const unsigned eq0 = __ballot_sync(0xFFFFFFFFu, in && v == v0);
        const unsigned rest = am & ~eq0;
        unsigned eq1 = 0;
        int l1 = 32;
        if (rest) {                                  // a second group: the first other lane's value
          l1 = __ffs(rest) - 1;
          const uint64_t v1 = ((uint64_t)__shfl_sync(0xFFFFFFFFu, (uint32_t)(v >> 32), l1) << 32) |
                              __shfl_sync(0xFFFFFFFFu, (uint32_t)v, l1);
          eq1 = __ballot_sync(0xFFFFFFFFu, in && v == v1);
        }
        const bool g0 = (eq0 >> lane) & 1u, g1 = (eq1 >> lane) & 1u;
        if (in && ((!g0 && !g1) || lane == l0 || lane == l1)) {
          const long long c = g0 ? (long long)__popc(eq0) : g1 ? (long long)__popc(eq1) : 1ll;
          if (!do_add(ts, (uint32_t)sd, v, c, &s_fill)) gt_add(gt, gmask, (uint32_t)sd, v, c, ovf);
        }
      }
      if (__any_sync(0xFFFFFFFFu, corr != 0u)) {       // (stencils: only at their faces)
#pragma unroll
        for (int j = 0; j < NC; ++j) {
          if ((uint32_t)j >= A.nc) break;
          const bool act = (corr >> j) & 1u;
          const unsigned am = __ballot_sync(0xFFFFFFFFu, act);
          if (act) {
            const long long d = (long long)cj[j] - (long long)A.c[j].m;
            const uint64_t v = A.c[j].side ? sv1 : sv0;
            const unsigned g = __match_any_sync(am, v);
            long long sum = d;
            if (__popc(g) > 1) {                       // group sum: a shuffle from each member
              sum = 0;
              for (unsigned gg = g; gg; gg &= gg - 1) sum += __shfl_sync(g, d, __ffs(gg) - 1);
            }
            if (lane == __ffs(g) - 1 && sum != 0) gt_add(gt, gmask, 2u + (uint32_t)j, v, sum, ovf);
          }
        }
      }
    }
  }
  __syncthreads();
  // every block's table holds about the same values (T_in's 4096): each block walks it from its own
  // offset, so the blocks' global adds meet different slots instead of all the same ones at once
  // (the spill held 31% of the stall samples)
  const uint32_t off = (uint32_t)(((uint64_t)blockIdx.x * DO_TS) / gridDim.x);
  for (uint32_t k = tid; k < DO_TS; k += blockDim.x) {
    const uint32_t i = k + off < DO_TS ? k + off : k + off - DO_TS;
    const uint64_t w = ts[i].w;
    if ((uint32_t)(w >> 56) != 0xFFu) gt_add(gt, gmask, (uint32_t)(w >> 56), ts[i].v, do_cnt(w), ovf);
  }
}

// Pass 2: the claims' histogram entries and value statistics.  For every H0 entry (side, v) and
// every claim j of that side, claim j's count of v over the whole object is m_j * H0(v) + D_j(v)
// (every corrected element's value is in H0); positive counts go to the HBM table, so no zero-count
// entry is ever created.  Skipped when pass 1 overflowed the global table (the fallback runs).
__global__ void __launch_bounds__(256) k_dense_emit(const __grid_constant__ DoArgs A, DevTables t, const DoSlot* gt,
                                                    uint32_t gmask, const uint32_t* ovf) {
  if (*(volatile const uint32_t*)ovf) return;
  __shared__ DoStat st;
  const int tid = threadIdx.x;
  for (uint32_t j = 0; j < A.nc; ++j) {
    if (tid < 6) st.s[tid] = 0;
    if (tid < 3) { st.mn[tid] = ~0ull; st.mx[tid] = 0; }
    __syncthreads();
    const uint32_t sd = A.c[j].side;
    DoAcc acc;
    do_acc_init(acc);
    for (uint32_t i = blockIdx.x * blockDim.x + tid; i <= gmask; i += gridDim.x * blockDim.x) {
      const uint64_t w = gt[i].w;
      if ((uint32_t)(w >> 56) != sd) continue;
      const uint64_t v = gt[i].v;
      const long long k = (long long)A.c[j].m * do_cnt(w) + gt_get(gt, gmask, 2u + j, v);
      if (k > 0) {
        hist_insert_global_rf(t, A.c[j].tag, v, (unsigned long long)k);
        do_acc(acc, v, (unsigned long long)k, A.c[j].meta, A.mant_bits);
      }
    }
    do_acc_fold(st, acc);
    __syncthreads();
    if (tid < 2) {
      const uint64_t key = tid ? A.ko : A.c[j].kp;
      const int f[6] = {F_ZERO, F_NAN, F_NONINT, F_NF16, F_NBF16, F_NF32};
      for (int i = 0; i < 6; ++i)
        if (st.s[i]) atomicAdd(&t.sum[key * NSUM + f[i]], st.s[i]);
      for (int i = 0; i < 3; ++i) {
        if (st.mn[i] != ~0ull) atomicMin(&t.mn[key * NMM + i], st.mn[i]);
        if (st.mx[i] != 0ull) atomicMax(&t.mx[key * NMM + i], st.mx[i]);
      }
    }
    __syncthreads();
  }
}

// Flush every claimed dense array into the exact histogram.  The base multiplicity m of every
// claim is sampled first (k_dense_mode, one sync): claims read about m >= 1 times per element
// (stencils, re-read weights) are flushed per object by k_dense_obj (H0 + corrections); claims
// whose counts are mostly 0 (sparse or one-off reads) take the per-array k_dense_flush.
ve_status dense_flush(ve_ctx* c, cudaStream_t s) {
  if (!c->dense_cap || !c->n_obj || !c->dense_dirty) return VE_OK;
  const size_t ns = (size_t)DENSE_PER_OBJ * c->n_obj;
  std::vector<uint32_t> dpc(ns);
  std::vector<unsigned long long> doff(ns);
  cudaError_t e = cudaMemcpyAsync(dpc.data(), c->o.dense_pc, ns * 4, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(doff.data(), c->o.dense_off, ns * 8, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c, e, "dense_flush");
  struct Cl { uint32_t i, ck; unsigned long long off; };
  std::vector<Cl> cl;
  for (uint32_t i = 0; i < c->n_obj; ++i)
    for (int j = 0; j < DENSE_PER_OBJ; ++j) {
      const uint32_t ck = dpc[DENSE_PER_OBJ * i + j];
      const unsigned long long off = doff[DENSE_PER_OBJ * i + j];
      if (ck == DENSE_FREE || ck == DENSE_OFF || off == DENSE_NOT_READY || off == DENSE_NONE) continue;
      const HostObject& o = c->objs[i];
      if (!((ck & DENSE_POST) ? o.post : o.pre)) continue;   // (claims are made only where the side exists)
      cl.push_back(Cl{i, ck, off});
    }
  c->dense_dirty = false;      // every claimed array is read and re-zeroed by its flush
  if (cl.empty()) return VE_OK;
  // base multiplicities
  const size_t nc = cl.size();
  std::vector<uint64_t> hb(2 * nc);
  for (size_t k = 0; k < nc; ++k) {
    hb[k] = (uint64_t)(uintptr_t)((uint32_t*)c->dense_pool + cl[k].off);
    hb[nc + k] = c->objs[cl[k].i].size / c->objs[cl[k].i].ew;
  }
  void* dm = nullptr;
  e = cudaMallocAsync(&dm, 2 * nc * 8 + nc * 4, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "dense_flush alloc");
  std::vector<uint32_t> mh(nc);
  cudaMemcpyAsync(dm, hb.data(), 2 * nc * 8, cudaMemcpyHostToDevice, s);
  count_launch();
  k_dense_mode<<<(unsigned)nc, 32, 0, s>>>((const uint32_t* const*)dm, (const uint64_t*)dm + nc,
                                          (uint32_t*)((uint8_t*)dm + 2 * nc * 8));
  // and the cardinality of each claim's side values (the H0 table holds ~DO_TS * 0.7 distinct values)
  unsigned int* dnd = (unsigned int*)((uint8_t*)dm + 2 * nc * 8);   // (reuses nothing: a second buffer below)
  (void)dnd;
  std::vector<unsigned int> nd(nc, ~0u);
  unsigned int* d_probe = nullptr;
  e = cudaMallocAsync((void**)&d_probe, 4 * nc, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "dense_flush probe alloc");
  cudaFuncSetAttribute(k_dense_sample_many, cudaFuncAttributeMaxDynamicSharedMemorySize, 8192 * 8);
  {
    std::vector<SampleJob> sj(nc);
    for (size_t k = 0; k < nc; ++k) {
      const HostObject& o = c->objs[cl[k].i];
      sj[k] = SampleJob{(const uint32_t*)((uint32_t*)c->dense_pool + cl[k].off),
                        (const uint8_t*)((cl[k].ck & DENSE_POST) ? o.post : o.pre), o.n_elems, o.ew, 0};
    }
    SampleJob* d_sj = nullptr;
    e = cudaMallocAsync((void**)&d_sj, nc * sizeof(SampleJob), s);
    if (e != cudaSuccess) return cuda_fail(c, e, "dense_flush probe jobs");
    cudaMemcpyAsync(d_sj, sj.data(), nc * sizeof(SampleJob), cudaMemcpyHostToDevice, s);
    count_launch();
    k_dense_sample_many<<<(unsigned)nc, 1024, 8192 * 8, s>>>(d_sj, d_probe);
    cudaFreeAsync(d_sj, s);
    e = cudaStreamSynchronize(s);     // (sj is a host vector of this scope)
    if (e != cudaSuccess) return cuda_fail(c, e, "dense_flush probe");
  }
  cudaMemcpyAsync(mh.data(), (uint8_t*)dm + 2 * nc * 8, nc * 4, cudaMemcpyDeviceToHost, s);
  cudaMemcpyAsync(nd.data(), d_probe, 4 * nc, cudaMemcpyDeviceToHost, s);
  cudaFreeAsync(dm, s);
  cudaFreeAsync(d_probe, s);
  e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c, e, "k_dense_mode");
  const size_t smem = (size_t)DO_TS * sizeof(DoSlot);
  cudaFuncSetAttribute(k_dense_obj<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaFuncSetAttribute(k_dense_obj<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaFuncSetAttribute(k_dense_obj<DO_MAXC>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaFuncSetAttribute(k_dense_flush<DF_THREADS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(DF_SLOTS * 12));
  // per object: its claims for the fused flush (others: the per-array flush right away)
  std::vector<DoArgs> objargs;
  std::vector<std::vector<size_t>> objcl;        // claim indices (into cl) of each DoArgs
  std::vector<uint32_t> objmask;                 // global table slots - 1
  std::vector<uint32_t> objidx;
  for (uint32_t i = 0; i < c->n_obj; ++i) {
    const HostObject& o = c->objs[i];
    DoArgs A;
    memset(&A, 0, sizeof(A));
    std::vector<size_t> mine;
    uint32_t ndmax = 0;
    for (size_t k = 0; k < nc; ++k) {
      if (cl[k].i != i) continue;
      const uint32_t ck = cl[k].ck, pc = ck & 0xFFFFu, meta = (ck >> 16) & 0x3Fu;
      const bool post = (ck & DENSE_POST) != 0u;
      uint32_t* arr = (uint32_t*)c->dense_pool + cl[k].off;
      if (mh[k] == 0u || nd[k] > 4096u) {   // mostly unread elements, or many values: per-array flush
        // (many values: no block table -- it would fill at once and every element would probe it in
        // vain before its global insert; cfg3's 21 such arrays: see DESIGN 5 "dense flush")
#ifndef VE_DF_DIRECT
#define VE_DF_DIRECT 1
#endif
        const uint32_t ts = (VE_DF_DIRECT && nd[k] > 4096u) ? 0u : (uint32_t)DF_SLOTS;
        const uint64_t blocks = (o.n_elems + DF_CHUNK - 1) / DF_CHUNK;
        count_launch();
        k_dense_flush<DF_THREADS><<<(unsigned)blocks, DF_THREADS, ts * 12, s>>>(
            arr, o.n_elems, (const uint8_t*)(post ? o.post : o.pre), o.ew, (pc << 16) | o.id, o.bmoff, c->t, meta,
            c->cfg.mant_bits, pc, c->cfg.n_pcs + o.id, ts, (uint32_t)DF_CHUNK, post ? 0u : 1u);
        continue;
      }
      DoClaim& d = A.c[A.nc++];
      d.cnt = arr;
      d.meta = meta;
      d.side = post ? 1u : 0u;
      d.tag = (pc << 16) | (o.id & 0xFFFFu);
      d.kp = pc;
      d.m = mh[k];
      A.snap[d.side] = (const uint8_t*)(post ? o.post : o.pre);
      mine.push_back(k);
      ndmax = std::max(ndmax, nd[k]);
    }
    if (!A.nc) continue;
    A.ew = o.ew;
    A.ko = c->cfg.n_pcs + o.id;
    A.mant_bits = c->cfg.mant_bits;
    A.ne = o.size / o.ew;                  // whole elements (K1 counts only those)
    A.bmoff = o.bmoff;
    // global (class, value) table: H0 of <= 2 sides and <= nc correction classes over the sampled
    // cardinality (<= 4096 here), at most half full
    uint64_t want = 2ull * (2u + A.nc) * (uint64_t)std::max(ndmax + 64u, 1024u), cap = 1024;
    while (cap < want) cap <<= 1;
    objargs.push_back(A);
    objcl.push_back(mine);
    objmask.push_back((uint32_t)(cap - 1));
    objidx.push_back(i);
  }
  if (!objargs.empty()) {
    size_t tot = 0;
    std::vector<size_t> toff(objargs.size());
    for (size_t q = 0; q < objargs.size(); ++q) { toff[q] = tot; tot += ((size_t)objmask[q] + 1) * sizeof(DoSlot); }
    const size_t fo = tot;
    tot += 4 * objargs.size();
    uint8_t* gbuf = nullptr;
    e = cudaMallocAsync((void**)&gbuf, tot, s);
    if (e != cudaSuccess) return cuda_fail(c, e, "dense_flush table alloc");
    cudaMemsetAsync(gbuf, 0xFF, fo, s);
    cudaMemsetAsync(gbuf + fo, 0, tot - fo, s);
    for (size_t q = 0; q < objargs.size(); ++q) {
      const DoArgs& A = objargs[q];
      const HostObject& o = c->objs[objidx[q]];
      DoSlot* gt = (DoSlot*)(gbuf + toff[q]);
      uint32_t* ovf = (uint32_t*)(gbuf + fo) + q;
      uint64_t blocks = (A.ne + DO_CH - 1) / DO_CH;
      if (blocks > (uint64_t)c->num_sms) blocks = (uint64_t)c->num_sms;
      if (blocks == 0) blocks = 1;
      count_launch();
      if (A.nc <= 1) k_dense_obj<1><<<(unsigned)blocks, DO_THREADS, smem, s>>>(A, c->t, gt, objmask[q], ovf);
      else if (A.nc <= 4) k_dense_obj<4><<<(unsigned)blocks, DO_THREADS, smem, s>>>(A, c->t, gt, objmask[q], ovf);
      else k_dense_obj<DO_MAXC><<<(unsigned)blocks, DO_THREADS, smem, s>>>(A, c->t, gt, objmask[q], ovf);
      uint64_t eb = ((uint64_t)objmask[q] + 1) / 256;
      eb = std::max<uint64_t>(1, std::min<uint64_t>(eb, 4ull * c->num_sms));
      count_launch();
      k_dense_emit<<<(unsigned)eb, 256, 0, s>>>(A, c->t, gt, objmask[q], ovf);
      // fallback (only when the table overflowed: the kernels return at once otherwise): the
      // per-array flush of every claim, exact at any cardinality
      for (size_t k : objcl[q]) {
        const uint32_t ck = cl[k].ck, pc = ck & 0xFFFFu, meta = (ck >> 16) & 0x3Fu;
        const bool post = (ck & DENSE_POST) != 0u;
        uint32_t* arr = (uint32_t*)c->dense_pool + cl[k].off;
        const uint64_t fb = std::min<uint64_t>((o.n_elems + DF_CHUNK - 1) / DF_CHUNK, 2ull * c->num_sms);   // (grid-stride)
        count_launch();
        k_dense_flush<DF_THREADS><<<(unsigned)fb, DF_THREADS, DF_SLOTS * 12, s>>>(
            arr, o.n_elems, (const uint8_t*)(post ? o.post : o.pre), o.ew, (pc << 16) | o.id, o.bmoff, c->t, meta,
            c->cfg.mant_bits, pc, c->cfg.n_pcs + o.id, (uint32_t)DF_SLOTS, (uint32_t)DF_CHUNK, post ? 0u : 1u, ovf);
      }
      for (uint32_t j = 0; j < A.nc; ++j) cudaMemsetAsync(A.c[j].cnt, 0, o.n_elems * 4, s);   // counters for the next epoch
    }
    cudaFreeAsync(gbuf, s);
  }
  e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "dense flush launch");
  unsigned long long glob[8];
  e = cudaMemcpyAsync(glob, c->t.glob, sizeof(glob), cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c, e, "dense_flush");
  if (glob[G_OVERFLOW]) {
    c->poisoned = true;
    return fail(c, VE_ERR_CAPACITY, "value histogram capacity exceeded (hist_capacity)");
  }
  return VE_OK;
}

// ---- K6: bitmap popcounts -------------------------------------------------
__global__ void k_bitmap_counts(const uint32_t* W, const uint32_t* L, const uint64_t* bmoff, const uint64_t* nwords,
                                unsigned long long* out /* [n][3] */) {
  const uint32_t o = blockIdx.y;
  const uint64_t base = bmoff[o], nw = nwords[o];
  unsigned long long cw = 0, cl = 0, cu = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nw; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t w = W[base + i], l = L[base + i];
    cw += __popc(w);
    cl += __popc(l);
    cu += __popc(w | l);
  }
  for (int s = 16; s > 0; s >>= 1) {
    cw += __shfl_xor_sync(0xFFFFFFFFu, cw, s);
    cl += __shfl_xor_sync(0xFFFFFFFFu, cl, s);
    cu += __shfl_xor_sync(0xFFFFFFFFu, cu, s);
  }
  if ((threadIdx.x & 31) == 0) {
    if (cw) atomicAdd(&out[3 * o + 0], cw);
    if (cl) atomicAdd(&out[3 * o + 1], cl);
    if (cu) atomicAdd(&out[3 * o + 2], cu);
  }
}

ve_status bitmap_counts(ve_ctx* c, cudaStream_t s, std::vector<ve_obj_stats>& out) {
  const uint32_t n = c->n_obj;
  out.assign(n, ve_obj_stats{0, 0, 0, 0, 0});
  if (n == 0) return VE_OK;
  std::vector<uint64_t> host(2 * n);
  uint64_t maxw = 0;
  for (uint32_t i = 0; i < n; ++i) {
    host[i] = c->objs[i].bmoff;
    host[n + i] = c->objs[i].bmwords;
    maxw = std::max<uint64_t>(maxw, c->objs[i].bmwords);
  }
  void* d = nullptr;
  cudaError_t e = cudaMallocAsync(&d, 2 * n * 8 + 3 * n * 8, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "bitmap_counts alloc");
  uint64_t* d_off = (uint64_t*)d;
  unsigned long long* d_out = (unsigned long long*)((uint8_t*)d + 2 * n * 8);
  cudaMemcpyAsync(d_off, host.data(), 2 * n * 8, cudaMemcpyHostToDevice, s);
  cudaMemsetAsync(d_out, 0, 3 * n * 8, s);
  uint64_t gx = (maxw + 255) / 256;
  if (gx > 64) gx = 64;
  if (gx == 0) gx = 1;
  count_launch();
  k_bitmap_counts<<<dim3((unsigned)gx, n), 256, 0, s>>>(c->t.W, c->t.L, d_off, d_off + n, d_out);
  std::vector<unsigned long long> h(3 * n);
  cudaMemcpyAsync(h.data(), d_out, 3 * n * 8, cudaMemcpyDeviceToHost, s);
  cudaFreeAsync(d, s);
  e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c, e, "bitmap_counts");
  // out is indexed by object id
  for (uint32_t i = 0; i < n; ++i) {
    const HostObject& ho = c->objs[i];
    ve_obj_stats& st = out[ho.id];
    st.n_elems = ho.n_elems;
    st.n_written = h[3 * i + 0];
    st.n_loaded_eq = h[3 * i + 1];
    st.n_touched = h[3 * i + 2];
  }
  return VE_OK;
}

}  // namespace ve
