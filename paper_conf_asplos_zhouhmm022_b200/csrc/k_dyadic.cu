// k_dyadic.cu -- SURVEY 8(f) f2: dyadic-scaled exact linear fit (ve_dyadic_fit).
//
// Def 3.7 (structured values) over the EXACT values of the records
// (reading R10): a float encodes the dyadic rational (-1)^s M 2^E, so with
// T = the key's largest number of fractional bits every Y = y 2^T is an integer and the
// points (addr, Y) are collinear exactly when the points (addr, y) are.  Three streaming
// passes over the AoS records (24 B each, read once per pass; HBM-bound):
//   D1  per key: NaN / inf -> fail; T = max fractional bits; min / max address
//   D2  anchors P = (min x, min Y at that x), Q = (max x, min Y at that x), Y = M 2^(E+T);
//       only records at a key's extreme x decode their value
//   (every record's |Y| < 2^62 bound is checked in D3, which computes Y anyway)
//   D3  every record: collinear with P and Q (exact 128-bit cross product) and, at P.x or
//       Q.x, equal to the anchor; else fail
// Keys as in K1: the PC key and the object key of the first byte (SHARED pseudo-object for
// shared-space records); invalid records are skipped.  D1 aggregates keys < DY_SK in shared
// memory per CTA (flushed at exit), the rest with global atomics.
#include <cuda_runtime.h>
#include <stdint.h>

#include <vector>

#include "ve_internal.cuh"

namespace ve {

constexpr uint32_t DY_T = 256;
constexpr uint32_t DY_SK = 512;
constexpr unsigned long long DY_NONE = ~0ull;

struct DyKey {                  // global per-key state
  unsigned int T, fail;
  unsigned long long minx, maxx;
  unsigned long long py, qy;    // Y + 2^63 (order-preserving), DY_NONE = no anchor yet
  unsigned long long x2, xl;    // C23: second-smallest / second-largest distinct address (DY_NONE / 0: none)
  unsigned long long n, n_off;  // C23: records, records off the interior line
};
constexpr uint32_t DY_NOTRUNC = 0xFFFFFFFFu;

// C22 / C23 with truncation: the value a float record carries after Def 3.8's truncation (C7);
// a NaN / inf stays non-finite (its exponent is kept), so dy_exact still fails it
__device__ __forceinline__ uint64_t dy_value(uint64_t b, uint32_t meta, uint32_t tr) {
  const uint32_t kind = meta_kind(meta);
  return (tr != DY_NOTRUNC && kind >= 2u) ? trunc_bits(b, kind, meta_lg(meta), tr) : b;
}

// exact value of the bits as M 2^E with M odd or zero; false for NaN / inf.  Unsigned values
// >= 2^63 report M = 2^62 (they fail the |Y| < 2^62 bound for any T).
__device__ __forceinline__ bool dy_exact(uint64_t b, uint32_t kind, uint32_t lg, long long& M, int& E) {
  if (kind < 2u) {
    if (kind == 0u) {
      M = (b >> 63) ? (1ll << 62) : (long long)b;
    } else {
      const uint32_t sh = 64u - (8u << lg);
      M = (long long)(b << sh) >> sh;
    }
    E = 0;
  } else {
    int eb, mb;
    if (kind == 3u) { eb = 8; mb = 7; }
    else if (lg == 1u) { eb = 5; mb = 10; }
    else if (lg == 2u) { eb = 8; mb = 23; }
    else { eb = 11; mb = 52; }
    const uint64_t ex = (b >> mb) & ((1ull << eb) - 1ull);
    if (ex == (1ull << eb) - 1ull) return false;
    const uint64_t man = b & ((1ull << mb) - 1ull);
    const int bias = (1 << (eb - 1)) - 1;
    const uint64_t sig = ex ? (man | (1ull << mb)) : man;
    E = ex ? (int)ex - bias - mb : 1 - bias - mb;
    M = ((b >> (eb + mb)) & 1ull) ? -(long long)sig : (long long)sig;
  }
  if (M == 0) { E = 0; return true; }
  const int tz = __ffsll(M) - 1;        // strip trailing zero bits: M odd
  M >>= tz;
  E += tz;
  return true;
}

// Y = M 2^s, s >= 0; false if |Y| >= 2^62
__device__ __forceinline__ bool dy_scaled(long long M, int s, long long& Y) {
  if (M == 0) { Y = 0; return true; }
  const unsigned long long a = M < 0 ? (unsigned long long)(-(M + 1)) + 1ull : (unsigned long long)M;
  const int bits = 64 - __clzll(a);
  if (bits + s > 62) return false;
  Y = M * (1ll << s);
  return true;
}

struct DyRec {
  uint64_t x, v;
  uint32_t pc, meta;
  uint32_t nk, k[2];
};

// the thread's last object [cb, ce) -> key: records of a warp window mostly stay in one object
struct DyObjCache {
  uint64_t cb = 1, ce = 0;
  uint32_t key = 0;
};

__device__ __forceinline__ bool dy_load(const ve_record* r, uint64_t i, const DevObjects& o, uint32_t n_pcs,
                                        DyRec& d, DyObjCache& oc) {
  const unsigned long long* q = reinterpret_cast<const unsigned long long*>(&r[i]);
  d.x = __ldg(q);
  d.v = __ldg(q + 1);
  const unsigned long long pm = __ldg(q + 2);
  d.pc = (uint32_t)pm;
  d.meta = (uint32_t)(pm >> 32);
  if (!rec_valid(d.x, d.v, d.pc, d.meta, n_pcs)) return false;
  d.nk = 1;
  d.k[0] = d.pc;
  if (meta_shared(d.meta)) {
    d.k[d.nk++] = n_pcs + o.n;
  } else if (d.x >= oc.cb && d.x < oc.ce) {
    d.k[d.nk++] = oc.key;
  } else {
    uint32_t lo = 0, hi = o.n;          // first object with base > x
    while (lo < hi) {
      const uint32_t mid = (lo + hi) >> 1;
      if (o.base[mid] <= d.x) lo = mid + 1; else hi = mid;
    }
    if (lo > 0 && d.x < o.end[lo - 1]) {
      oc.cb = o.base[lo - 1];
      oc.ce = o.end[lo - 1];
      oc.key = n_pcs + o.id[lo - 1];
      d.k[d.nk++] = oc.key;
    }
  }
  return true;
}

__global__ void __launch_bounds__(DY_T) k_dy_scan(const ve_record* r, uint64_t n, DevObjects o, uint32_t n_pcs,
                                                  uint32_t nk, DyKey* K, uint32_t tr, int count) {
  __shared__ unsigned int sT[DY_SK], sF[DY_SK];
  __shared__ unsigned long long sMin[DY_SK], sMax[DY_SK];
  const uint32_t ns = nk < DY_SK ? nk : DY_SK;
  for (uint32_t i = threadIdx.x; i < ns; i += DY_T) { sT[i] = 0; sF[i] = 0; sMin[i] = DY_NONE; sMax[i] = 0; }
  __syncthreads();
  DyObjCache oc;
  // block-uniform trip count: every lane takes part in the warp aggregation below
  for (uint64_t b = (uint64_t)blockIdx.x * DY_T; b < n; b += (uint64_t)gridDim.x * DY_T) {
    const uint64_t i = b + threadIdx.x;
    DyRec d;
    d.nk = 0;
    const bool act = i < n && dy_load(r, i, o, n_pcs, d, oc);
    long long M = 0;
    int E = 0;
    const bool fin = act && dy_exact(dy_value(d.v, d.meta, tr), meta_kind(d.meta), meta_lg(d.meta), M, E);
    unsigned int t = (fin && E < 0) ? (unsigned int)(-E) : 0u;
    for (uint32_t j = 0; j < 2; ++j) {
      const uint32_t k = j < d.nk ? d.k[j] : 0xFFFFFFFFu;
      const unsigned g = __match_any_sync(0xFFFFFFFFu, k);
      if (g == 0xFFFFFFFFu) {
        // the whole warp on one key (the common case: a warp-wide access of one PC / object):
        // one update per warp instead of 32 contended shared-memory atomics
        if (k == 0xFFFFFFFFu) continue;
        unsigned long long mn = fin ? d.x : DY_NONE, mx = fin ? d.x : 0ull;
        unsigned int tt = t, ff = (!fin) ? 1u : 0u, hv = fin ? 1u : 0u;
        {                                  // 64-bit min / max from 32-bit warp reductions
          const unsigned mh = __reduce_min_sync(0xFFFFFFFFu, (unsigned)(mn >> 32));
          const unsigned ml = __reduce_min_sync(0xFFFFFFFFu, (unsigned)(mn >> 32) == mh ? (unsigned)mn : ~0u);
          const unsigned xh = __reduce_max_sync(0xFFFFFFFFu, (unsigned)(mx >> 32));
          const unsigned xl = __reduce_max_sync(0xFFFFFFFFu, (unsigned)(mx >> 32) == xh ? (unsigned)mx : 0u);
          mn = ((unsigned long long)mh << 32) | ml;
          mx = ((unsigned long long)xh << 32) | xl;
        }
        tt = __reduce_max_sync(0xFFFFFFFFu, tt);
        ff = __reduce_or_sync(0xFFFFFFFFu, ff);
        hv = __reduce_or_sync(0xFFFFFFFFu, hv);
        if (count && (threadIdx.x & 31u) == 0u) atomicAdd(&K[k].n, 32ull);   // (C23's record count)
        if ((threadIdx.x & 31u) == 0u) {
          if (k < ns) {
            if (ff) sF[k] = 1u;
            if (hv) {
              if (tt) atomicMax(&sT[k], tt);
              atomicMin(&sMin[k], mn);
              atomicMax(&sMax[k], mx);
            }
          } else {
            if (ff) K[k].fail = 1u;
            if (hv) {
              if (tt) atomicMax(&K[k].T, tt);
              atomicMin(&K[k].minx, mn);
              atomicMax(&K[k].maxx, mx);
            }
          }
        }
        continue;
      }
      if (k == 0xFFFFFFFFu) continue;
      if (count) atomicAdd(&K[k].n, 1ull);
      if (k < ns) {
        if (!fin) { sF[k] = 1u; continue; }
        if (t) atomicMax(&sT[k], t);
        atomicMin(&sMin[k], (unsigned long long)d.x);
        atomicMax(&sMax[k], (unsigned long long)d.x);
      } else {
        if (!fin) { K[k].fail = 1u; continue; }
        if (t) atomicMax(&K[k].T, t);
        atomicMin(&K[k].minx, (unsigned long long)d.x);
        atomicMax(&K[k].maxx, (unsigned long long)d.x);
      }
    }
  }
  __syncthreads();
  for (uint32_t k = threadIdx.x; k < ns; k += DY_T) {
    if (sF[k]) K[k].fail = 1u;
    if (sMin[k] == DY_NONE) continue;
    if (sT[k]) atomicMax(&K[k].T, sT[k]);
    atomicMin(&K[k].minx, sMin[k]);
    atomicMax(&K[k].maxx, sMax[k]);
  }
}

// C21: D2 (anchors and the |Y| bound) when pass == 0, D3 (collinearity) when pass == 1;
// C23: the second extreme addresses and the |Y| bound (2), the interior anchors (3), the records
// off the interior line (4)
__global__ void __launch_bounds__(DY_T) k_dy_check(const ve_record* r, uint64_t n, DevObjects o, uint32_t n_pcs,
                                                   DyKey* K, int pass, uint32_t tr) {
  DyObjCache oc;
  for (uint64_t i = (uint64_t)blockIdx.x * DY_T + threadIdx.x; i < n; i += (uint64_t)gridDim.x * DY_T) {
    DyRec d;
    if (!dy_load(r, i, o, n_pcs, d, oc)) continue;
    if (pass == 0) {                       // D2 needs only the records at a key's extreme address
      bool any = false;
      for (uint32_t j = 0; j < d.nk; ++j) {
        const DyKey& k = K[d.k[j]];
        any |= d.x == k.minx || d.x == k.maxx;
      }
      if (!any) continue;
    } else if (pass == 3) {                // C23 anchors: only the records at the interior anchors
      bool any = false;
      for (uint32_t j = 0; j < d.nk; ++j) {
        const DyKey& k = K[d.k[j]];
        any |= d.x == k.x2 || d.x == k.xl;
      }
      if (!any) continue;
    } else {                               // nothing left to check once every key of the record failed
      bool any = false;
      for (uint32_t j = 0; j < d.nk; ++j) any |= K[d.k[j]].fail == 0u;
      if (!any) continue;
    }
    long long M;
    int E;
    if (!dy_exact(dy_value(d.v, d.meta, tr), meta_kind(d.meta), meta_lg(d.meta), M, E)) continue;   // failed in D1
    for (uint32_t j = 0; j < d.nk; ++j) {
      DyKey& k = K[d.k[j]];
      if (k.fail) continue;                  // a stale 0 only costs the check below
      long long Y;
      if (!dy_scaled(M, E + (int)k.T, Y)) { k.fail = 1u; continue; }
      const unsigned long long yo = (unsigned long long)Y ^ (1ull << 63);
      if (pass == 0) {
        if (d.x == k.minx) atomicMin(&k.py, yo);
        if (d.x == k.maxx) atomicMin(&k.qy, yo);
        continue;
      }
      if (pass == 2) {                       // C23 step 2
        if (d.x > k.minx) atomicMin(&k.x2, (unsigned long long)d.x);
        if (d.x < k.maxx) atomicMax(&k.xl, (unsigned long long)d.x);
        continue;
      }
      if (pass == 3) {                       // C23 step 3 (py / qy hold the interior anchors' Y)
        if (d.x == k.x2) atomicMin(&k.py, yo);
        if (d.x == k.xl) atomicMin(&k.qy, yo);
        continue;
      }
      if (pass == 4) {                       // C23 step 4
        if (!(k.x2 != DY_NONE && k.x2 < k.xl)) continue;
        const long long ay = (long long)(k.py ^ (1ull << 63)), by = (long long)(k.qy ^ (1ull << 63));
        const __int128 dx = (__int128)(long long)(d.x - k.x2), bxa = (__int128)(long long)(k.xl - k.x2);
        if ((__int128)(Y - ay) * bxa != (__int128)(by - ay) * dx) atomicAdd(&k.n_off, 1ull);
        continue;
      }
      const long long py = (long long)(k.py ^ (1ull << 63)), qy = (long long)(k.qy ^ (1ull << 63));
      const __int128 dx = (__int128)(long long)(d.x - k.minx), qx = (__int128)(long long)(k.maxx - k.minx);
      bool ok = (__int128)(Y - py) * qx == (__int128)(qy - py) * dx;   // |Y - py| < 2^63, |dx| < 2^48
      ok = ok && !(d.x == k.minx && Y != py) && !(d.x == k.maxx && Y != qy);
      if (!ok) k.fail = 1u;
    }
  }
}

__global__ void k_dy_init(DyKey* K, uint32_t nk) {
  for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < nk; k += gridDim.x * blockDim.x) {
    K[k].T = 0; K[k].fail = 0;
    K[k].minx = DY_NONE; K[k].maxx = 0;
    K[k].py = DY_NONE; K[k].qy = DY_NONE;
    K[k].x2 = DY_NONE; K[k].xl = 0;
    K[k].n = 0; K[k].n_off = 0;
  }
}

}  // namespace ve

using namespace ve;

static ve_status dy_run(ve_ctx* c, const ve_record* d_records, uint64_t n, uint32_t tr, bool outlier,
                        std::vector<DyKey>& hk, cudaStream_t s) {
  const uint32_t nk = c->n_keys;
  if (n && (!d_records || ((uintptr_t)d_records & 7))) return fail(c, VE_ERR_INVALID, "fit: null or misaligned records");
  cudaSetDevice(c->device);
  DyKey* K = nullptr;
  cudaError_t e = cudaMallocAsync((void**)&K, sizeof(DyKey) * (size_t)nk, s);
  if (e != cudaSuccess) { cudaGetLastError(); return fail(c, VE_ERR_NOMEM, "fit: workspace"); }
  count_launch();
  k_dy_init<<<(nk + 255) / 256, 256, 0, s>>>(K, nk);
  if (n) {
    uint64_t b = (n + DY_T - 1) / DY_T;
    const uint64_t cap = (uint64_t)c->num_sms * 8;
    const unsigned grid = (unsigned)(b < cap ? b : cap);
    count_launch();
    k_dy_scan<<<grid, DY_T, 0, s>>>(d_records, n, c->o, c->cfg.n_pcs, nk, K, tr, outlier ? 1 : 0);
    const int passes[2][3] = {{0, 1, -1}, {2, 3, 4}};
    for (int p : passes[outlier ? 1 : 0]) {
      if (p < 0) continue;
      count_launch();
      k_dy_check<<<grid, DY_T, 0, s>>>(d_records, n, c->o, c->cfg.n_pcs, K, p, tr);
    }
  }
  hk.resize(nk);
  e = cudaMemcpyAsync(hk.data(), K, sizeof(DyKey) * (size_t)nk, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  cudaFreeAsync(K, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "fit");
  return VE_OK;
}

extern "C" ve_status ve_dyadic_fit_ex(ve_ctx* c, const ve_record* d_records, uint64_t n, uint32_t flags,
                                      ve_dyadic* h_out, cudaStream_t s) {
  if (!c || !h_out || (flags & ~VE_FIT_TRUNC)) return VE_ERR_INVALID;
  std::vector<DyKey> hk;
  ctx_begin(c, s);
  ve_status st = dy_run(c, d_records, n, (flags & VE_FIT_TRUNC) ? c->cfg.mant_bits : DY_NOTRUNC, false, hk, s);
  if (st != VE_OK) return st;
  for (uint32_t k = 0; k < c->n_keys; ++k) {
    ve_dyadic& o = h_out[k];
    o = ve_dyadic{};
    if (hk[k].fail) { o.state = VE_LINE_FAIL; continue; }
    if (hk[k].minx == DY_NONE) { o.state = VE_LINE_EMPTY; continue; }
    o.state = hk[k].minx == hk[k].maxx ? VE_LINE_POINT : VE_LINE_LINE;
    o.scale = hk[k].T;
    o.px = hk[k].minx;
    o.qx = hk[k].maxx;
    o.py = (int64_t)(hk[k].py ^ (1ull << 63));
    o.qy = (int64_t)(hk[k].qy ^ (1ull << 63));
  }
  return VE_OK;
}

extern "C" ve_status ve_dyadic_fit(ve_ctx* c, const ve_record* d_records, uint64_t n, ve_dyadic* h_out,
                                   cudaStream_t s) {
  return ve_dyadic_fit_ex(c, d_records, n, 0u, h_out, s);
}

extern "C" ve_status ve_outlier_fit(ve_ctx* c, const ve_record* d_records, uint64_t n, uint32_t flags,
                                    ve_outlier* h_out, cudaStream_t s) {
  if (!c || !h_out || (flags & ~VE_FIT_TRUNC)) return VE_ERR_INVALID;
  std::vector<DyKey> hk;
  ctx_begin(c, s);
  ve_status st = dy_run(c, d_records, n, (flags & VE_FIT_TRUNC) ? c->cfg.mant_bits : DY_NOTRUNC, true, hk, s);
  if (st != VE_OK) return st;
  for (uint32_t k = 0; k < c->n_keys; ++k) {
    ve_outlier& o = h_out[k];
    o = ve_outlier{};
    if (hk[k].fail) { o.state = VE_LINE_FAIL; continue; }
    if (hk[k].minx == DY_NONE) { o.state = VE_LINE_EMPTY; continue; }
    o.n = hk[k].n;
    o.scale = hk[k].T;
    if (!(hk[k].x2 != DY_NONE && hk[k].x2 < hk[k].xl)) { o.state = VE_LINE_POINT; o.scale = 0; continue; }
    o.state = VE_LINE_LINE;
    o.ax = hk[k].x2;
    o.bx = hk[k].xl;
    o.ay = (int64_t)(hk[k].py ^ (1ull << 63));
    o.by = (int64_t)(hk[k].qy ^ (1ull << 63));
    o.n_off = hk[k].n_off;
  }
  return VE_OK;
}
