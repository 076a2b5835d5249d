// k_analyze.cu -- K1: the fused record-analysis pass.
//
// One persistent CTA per SM streams 24-byte records (PC, address,
// size, raw value per access) in warp windows of 32 consecutive records.
// Per window each lane decodes one record, maps it to its data object
// (P:L230), gathers and compares the pre-snapshot bytes (Def 3.1),
// and derives the bit-level value tests of Defs 3.3-3.8.  Lanes
// are then grouped by key (PC, object) with __match_any_sync and every group
// is reduced with warp REDUX into per-CTA shared-memory stat rows, an
// open-addressing shared-memory value histogram (overflow to the exact HBM
// table), per-key line states (the (+) monoid) and the written / loaded
// element bitmaps.  At the end each CTA folds its shared state into the
// global tables.  All results are integer and order-free, hence identical for
// any grid, chunking or rank split (C12).
#include <cuda_runtime.h>

#include "ve_internal.cuh"

namespace ve {

struct AnalyzeParams {
  const ve_record* recs;
  uint64_t n;
  uint32_t n_pcs, n_obj;
  uint32_t sp, so;          // shared-memory stat rows for PCs [0,sp) and object keys [0,so)
  uint32_t mant_bits;
  uint32_t hs;              // shared histogram slots (power of 2)
  uint32_t objc;            // objects cached in shared memory (0 = use global table)
  DevObjects o;
  DevTables t;
};

struct Smem {
  uint32_t* ssum;           // [nsk][NSUM]
  unsigned long long* smin; // [nsk][NMM]
  unsigned long long* smax; // [nsk][NMM]
  LineState* sline;         // [nsk]
  HSlot* shs;               // [hs]
  uint32_t* shc;            // [hs]
  uint64_t* sob;            // [objc] base
  uint64_t* soe;            // [objc] end
  uint32_t* sctr;           // [4]: invalid, unmapped, hist fill
};

__host__ __device__ inline size_t align16(size_t x) { return (x + 15) & ~size_t(15); }

__host__ __device__ inline size_t smem_bytes(uint32_t nsk, uint32_t hs, uint32_t objc) {
  size_t b = 0;
  b += align16(sizeof(uint32_t) * nsk * NSUM);
  b += align16(sizeof(unsigned long long) * nsk * NMM) * 2;
  b += align16(sizeof(LineState) * nsk);
  b += align16(sizeof(HSlot) * hs);
  b += align16(sizeof(uint32_t) * hs);
  b += align16(sizeof(uint64_t) * objc) * 2;
  b += 16;
  return b;
}

__device__ inline Smem carve(uint8_t* base, uint32_t nsk, uint32_t hs, uint32_t objc) {
  Smem s;
  size_t off = 0;
  s.ssum = (uint32_t*)(base + off); off += align16(sizeof(uint32_t) * nsk * NSUM);
  s.smin = (unsigned long long*)(base + off); off += align16(sizeof(unsigned long long) * nsk * NMM);
  s.smax = (unsigned long long*)(base + off); off += align16(sizeof(unsigned long long) * nsk * NMM);
  s.sline = (LineState*)(base + off); off += align16(sizeof(LineState) * nsk);
  s.shs = (HSlot*)(base + off); off += align16(sizeof(HSlot) * hs);
  s.shc = (uint32_t*)(base + off); off += align16(sizeof(uint32_t) * hs);
  s.sob = (uint64_t*)(base + off); off += align16(sizeof(uint64_t) * objc);
  s.soe = (uint64_t*)(base + off); off += align16(sizeof(uint64_t) * objc);
  s.sctr = (uint32_t*)(base + off);
  return s;
}

// ---- warp helpers ------------------------------------------------------------
__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}
__device__ __forceinline__ uint64_t redmin64(unsigned gm, uint64_t v) {
  uint32_t hi = __reduce_min_sync(gm, (uint32_t)(v >> 32));
  uint32_t lo = __reduce_min_sync(gm, ((uint32_t)(v >> 32) == hi) ? (uint32_t)v : 0xFFFFFFFFu);
  return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ uint64_t redmax64(unsigned gm, uint64_t v) {
  uint32_t hi = __reduce_max_sync(gm, (uint32_t)(v >> 32));
  uint32_t lo = __reduce_max_sync(gm, ((uint32_t)(v >> 32) == hi) ? (uint32_t)v : 0u);
  return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ uint64_t shfl64(unsigned gm, uint64_t v, int src) {
  uint32_t lo = __shfl_sync(gm, (uint32_t)v, src);
  uint32_t hi = __shfl_sync(gm, (uint32_t)(v >> 32), src);
  return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ void atomic_min_u64(unsigned long long* p, unsigned long long v) {
  if (v < *(volatile unsigned long long*)p) atomicMin(p, v);
}
__device__ __forceinline__ void atomic_max_u64(unsigned long long* p, unsigned long long v) {
  if (v > *(volatile unsigned long long*)p) atomicMax(p, v);
}

// load w little-endian bytes of the pre snapshot (the gather of S3)
__device__ __forceinline__ uint64_t load_pre(uint64_t p, uint32_t lg) {
  uint32_t w = 1u << lg;
  if ((p & (w - 1)) == 0) {
    if (lg == 0) return *(const uint8_t*)p;
    if (lg == 1) return __ldg((const unsigned short*)p);
    if (lg == 2) return __ldg((const unsigned int*)p);
    return __ldg((const unsigned long long*)p);
  }
  uint64_t v = 0;
  for (uint32_t i = 0; i < w; ++i) v |= (uint64_t)__ldg((const unsigned char*)(p + i)) << (8 * i);
  return v;
}

// per-lane record facts shared by the PC-key and object-key groups
struct Facts {
  uint64_t addr, val, ordv, truncv;
  __int128 y;
  uint32_t tc;
  uint32_t packA, packB;    // 6-bit predicate fields for the packed REDUX sums
  bool nan, isf, pfail;
};

// Reduce one key group (all lanes in gm share the key) and fold it into the
// key's row: shared memory when slot >= 0, else the global table.
__device__ __forceinline__ void apply_group(const AnalyzeParams& P, const Smem& S, unsigned gm, int slot,
                                            uint32_t key, const Facts& f) {
  const int lane = threadIdx.x & 31;
  const unsigned gsize = __popc(gm);
  const int rank = __popc(gm & lanemask_lt());
  // C1/C2/C5 sums: 10 predicates packed 6 bits apart, two REDUX adds
  const uint32_t A = __reduce_add_sync(gm, f.packA);
  const uint32_t B = __reduce_add_sync(gm, f.packB);
  // n_type: one add per distinct type code in the group
  const unsigned tm = __match_any_sync(gm, f.tc);
  // C4/C5/C7 min/max
  const uint64_t rmin = redmin64(gm, f.val), rmax = redmax64(gm, f.val);
  const uint64_t omin = redmin64(gm, f.nan ? ~0ull : f.ordv), omax = redmax64(gm, f.nan ? 0ull : f.ordv);
  const bool tr = f.isf && !f.nan;
  const uint64_t tmin = redmin64(gm, tr ? f.truncv : ~0ull), tmax = redmax64(gm, tr ? f.truncv : 0ull);

  // distribute the 11 sum fields and 6 min/max fields over the group's lanes
  for (int j = rank; j < 17; j += gsize) {
    if (j < 11) {
      uint32_t v, field;
      if (j == 0) { v = gsize - (A & 63u); field = F_LD; }
      else if (j <= 5) { v = (A >> (6 * (j - 1))) & 63u; field = (uint32_t)j; }
      else { v = (B >> (6 * (j - 6))) & 63u; field = F_NAN + (uint32_t)(j - 6); }
      if (v) {
        if (slot >= 0) atomicAdd(&S.ssum[slot * NSUM + field], v);
        else atomicAdd(&P.t.sum[(uint64_t)key * NSUM + field], (unsigned long long)v);
      }
    } else {
      int m = j - 11;  // 0 raw_min 1 raw_max 2 ord_min 3 ord_max 4 trunc_min 5 trunc_max
      uint64_t v = (m == 0) ? rmin : (m == 1) ? rmax : (m == 2) ? omin : (m == 3) ? omax : (m == 4) ? tmin : tmax;
      unsigned long long* base = (m & 1) ? (slot >= 0 ? S.smax + slot * NMM : P.t.mx + (uint64_t)key * NMM)
                                         : (slot >= 0 ? S.smin + slot * NMM : P.t.mn + (uint64_t)key * NMM);
      if (m & 1) atomic_max_u64(base + (m >> 1), v);
      else atomic_min_u64(base + (m >> 1), v);
    }
  }
  if (lane == __ffs(tm) - 1) {
    uint32_t c = __popc(tm);
    if (slot >= 0) atomicAdd(&S.ssum[slot * NSUM + F_TYPE0 + f.tc], c);
    else atomicAdd(&P.t.sum[(uint64_t)key * NSUM + F_TYPE0 + f.tc], (unsigned long long)c);
  }

  // C8 structured: group line state, merged into the key's state unless it already FAILed
  LineState* ls = (slot >= 0) ? &S.sline[slot] : &P.t.line[key];
  // the state may change under us (other warps merge concurrently): decide group-uniformly
  const uint32_t cur = __shfl_sync(gm, *(volatile uint32_t*)&ls->state, __ffs(gm) - 1);
  if (cur == VE_LINE_FAIL) return;
  LinePts g;
  if (__any_sync(gm, f.pfail)) {
    g.state = VE_LINE_FAIL;
    g.px = g.qx = 0; g.py = g.qy = 0;
  } else {
    const uint64_t minx = redmin64(gm, f.addr), maxx = redmax64(gm, f.addr);
    const int pl = __ffs(__ballot_sync(gm, f.addr == minx)) - 1;
    const int ql = __ffs(__ballot_sync(gm, f.addr == maxx)) - 1;
    const uint64_t ylo = (uint64_t)f.y, yhi = (uint64_t)(f.y >> 64);
    const __int128 py = mk128(shfl64(gm, ylo, pl), (int64_t)shfl64(gm, yhi, pl));
    const __int128 qy = mk128(shfl64(gm, ylo, ql), (int64_t)shfl64(gm, yhi, ql));
    bool ok;
    if (minx == maxx) ok = (f.y == py);
    else ok = collinear(minx, py, maxx, qy, f.addr, f.y);
    ok = __all_sync(gm, ok);
    g.state = !ok ? VE_LINE_FAIL : (minx == maxx ? VE_LINE_POINT : VE_LINE_LINE);
    g.px = minx; g.py = py; g.qx = maxx; g.qy = qy;
  }
  if (rank == 0) line_merge_locked(ls, g);
}

// Insert a group of equal (tag, bits) with count c: shared table first, HBM table on miss/full.
__device__ __forceinline__ void hist_insert(const AnalyzeParams& P, const Smem& S, uint32_t tag, uint64_t bits,
                                            uint32_t c) {
  const uint32_t hmask = P.hs - 1;
  uint32_t h = (uint32_t)hist_hash(tag, bits) & hmask;
  for (int probe = 0; probe < 16; ++probe) {
    HSlot* s = &S.shs[h];
    uint64_t lo = *(volatile uint64_t*)&s->bits;
    uint32_t stag = *(volatile uint32_t*)&s->tag;
    if (stag == tag && lo == bits) { atomicAdd(&S.shc[h], c); return; }
    if (stag == EMPTY_TAG) {
      if (*(volatile uint32_t*)&S.sctr[2] >= (P.hs >> 1)) break;     // keep the table at most half full
      uint64_t ehi = ((uint64_t)(*(volatile uint32_t*)&s->pad) << 32) | EMPTY_TAG;
      uint64_t olo, ohi;
      cas128_shared(s, lo, ehi, bits, (uint64_t)tag, olo, ohi);
      if ((uint32_t)ohi == EMPTY_TAG && olo == lo) {
        atomicAdd(&S.sctr[2], 1u);
        atomicAdd(&S.shc[h], c);
        return;
      }
      if ((uint32_t)ohi == tag && olo == bits) { atomicAdd(&S.shc[h], c); return; }
    }
    h = (h + 1) & hmask;
  }
  hist_insert_global(P.t, tag, bits, c);
}

__device__ __forceinline__ int find_object(const AnalyzeParams& P, const Smem& S, uint64_t addr) {
  const uint64_t* base = P.objc ? S.sob : P.o.base;
  int lo = 0, hi = (int)P.o.n;  // first object with base > addr
  while (lo < hi) {
    int mid = (lo + hi) >> 1;
    if (base[mid] <= addr) lo = mid + 1; else hi = mid;
  }
  if (lo == 0) return -1;
  const uint64_t e = P.objc ? S.soe[lo - 1] : P.o.end[lo - 1];
  return addr < e ? lo - 1 : -1;
}

__device__ __forceinline__ void bitmap_or(uint32_t* bm, bool part, uint64_t word, uint32_t bits) {
  unsigned pm = __ballot_sync(0xFFFFFFFFu, part);
  if (part) {
    unsigned g = __match_any_sync(pm, word);
    uint32_t b = __reduce_or_sync(g, bits);
    if ((threadIdx.x & 31) == __ffs(g) - 1) atomicOr(&bm[word], b);
  }
}

__global__ void __launch_bounds__(512, 1) k_analyze(AnalyzeParams P) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  const uint32_t nsk = P.sp + P.so;
  Smem S = carve(smem_raw, nsk, P.hs, P.objc);
  const int tid = threadIdx.x, lane = tid & 31;

  for (uint32_t i = tid; i < nsk * NSUM; i += blockDim.x) S.ssum[i] = 0;
  for (uint32_t i = tid; i < nsk * NMM; i += blockDim.x) { S.smin[i] = ~0ull; S.smax[i] = 0; }
  for (uint32_t i = tid; i < nsk; i += blockDim.x) { S.sline[i].state = VE_LINE_EMPTY; S.sline[i].lock = 0; }
  for (uint32_t i = tid; i < P.hs; i += blockDim.x) {
    S.shs[i].bits = 0; S.shs[i].tag = EMPTY_TAG; S.shs[i].pad = 0; S.shc[i] = 0;
  }
  for (uint32_t i = tid; i < P.objc; i += blockDim.x) { S.sob[i] = P.o.base[i]; S.soe[i] = P.o.end[i]; }
  if (tid < 4) S.sctr[tid] = 0;
  __syncthreads();

  const uint64_t nwin = (P.n + 31) / 32;
  const uint64_t wstride = (uint64_t)gridDim.x * (blockDim.x / 32);
  int ocache = -1;  // warp-uniform last object
  uint32_t n_invalid = 0, n_unmapped = 0;

  for (uint64_t w = (uint64_t)blockIdx.x * (blockDim.x / 32) + (tid >> 5); w < nwin; w += wstride) {
    const uint64_t r = w * 32 + lane;
    const bool inrange = r < P.n;
    uint64_t addr = 0, val = 0;
    uint32_t pc = 0, meta = 0;
    if (inrange) {
      const unsigned long long* q = reinterpret_cast<const unsigned long long*>(&P.recs[r]);
      addr = __ldcs(q);
      val = __ldcs(q + 1);
      const unsigned long long pm = __ldcs(q + 2);
      pc = (uint32_t)pm;
      meta = (uint32_t)(pm >> 32);
    }
    // S1 decode + validate
    const bool valid = inrange && rec_valid(addr, val, pc, meta, P.n_pcs);
    const unsigned vmask = __ballot_sync(0xFFFFFFFFu, valid);
    const unsigned imask = __ballot_sync(0xFFFFFFFFu, inrange);
    if (lane == 0) n_invalid += (uint32_t)(__popc(imask) - __popc(vmask));
    if (vmask == 0) continue;
    const uint32_t lg = meta & 3u, kind = (meta >> 2) & 3u;
    const bool st = meta_store(meta), sh = meta_shared(meta);

    // S2 address -> object (warp-uniform cache, then binary search)
    const bool need = valid && !sh;
    int oi = -1;
    bool hit = false;
    if (ocache >= 0 && need) {
      const uint64_t b = P.objc ? S.sob[ocache] : P.o.base[ocache];
      const uint64_t e = P.objc ? S.soe[ocache] : P.o.end[ocache];
      hit = addr >= b && addr < e;
      if (hit) oi = ocache;
    }
    if (need && !hit) oi = find_object(P, S, addr);
    {
      const unsigned mm = __ballot_sync(0xFFFFFFFFu, need && oi >= 0);
      if (mm) ocache = __shfl_sync(0xFFFFFFFFu, oi, __ffs(mm) - 1);
    }
    const bool mapped = oi >= 0;
    const unsigned um = __ballot_sync(0xFFFFFFFFu, need && !mapped);
    if (lane == 0) n_unmapped += __popc(um);

    // S3 snapshot gather + eq_pre
    uint32_t ew_lg = 0, oid = 0;
    uint64_t off = 0, bmoff = 0;
    bool inside = false, eqdef = false, eq = false;
    if (mapped) {
      const uint64_t b = P.objc ? S.sob[oi] : P.o.base[oi];
      const uint64_t e = P.objc ? S.soe[oi] : P.o.end[oi];
      off = addr - b;
      inside = addr + (1u << lg) <= e;
      oid = P.o.id[oi];
      const uint32_t ew = P.o.ew[oi];
      ew_lg = (ew == 1) ? 0 : (ew == 2) ? 1 : (ew == 4) ? 2 : 3;
      bmoff = P.o.bmoff[oi];
      const uint64_t pre = P.o.pre[oi];
      if (inside && pre) {
        eqdef = true;
        eq = load_pre(pre + off, lg) == val;
      }
    }

    // W / L element bitmaps (C3, C10)
    {
      const bool wpart = inside && st;
      const uint64_t e0 = off >> ew_lg, e1 = (off + (1u << lg) - 1) >> ew_lg;
      const uint64_t w0 = bmoff + (e0 >> 5), w1 = bmoff + (e1 >> 5);
      uint32_t b0 = 0, b1 = 0;
      if (wpart) {
        for (uint64_t e = e0; e <= e1; ++e) {
          if (bmoff + (e >> 5) == w0) b0 |= 1u << (e & 31);
          else b1 |= 1u << (e & 31);
        }
      }
      bitmap_or(P.t.W, wpart, w0, b0);
      const bool spill = wpart && w1 != w0;
      if (__any_sync(0xFFFFFFFFu, spill)) bitmap_or(P.t.W, spill, w1, b1);
      const bool lpart = inside && !st && eq;
      bitmap_or(P.t.L, lpart, w0, 1u << (e0 & 31));
    }

    // per-record value tests (S4-S7)
    Facts f;
    f.addr = addr;
    f.val = val;
    f.tc = type_code(kind, lg);
    f.isf = kind >= 2u;
    int64_t ival = 0;
    const uint32_t ff = f.isf ? float_flags(val, kind, lg, ival) : 0u;
    f.nan = ff & 1u;
    f.pfail = f.isf && (ff & 2u);
    f.ordv = ord_key(val, kind, lg);
    f.truncv = f.isf ? trunc_bits(val, kind, lg, P.mant_bits) : 0ull;
    if (kind == 0u) f.y = (__int128)val;
    else if (kind == 1u) {
      const uint32_t sh64 = 64u - (8u << lg);
      f.y = (__int128)((int64_t)(val << sh64) >> sh64);
    } else f.y = (__int128)ival;
    f.packA = (uint32_t)st | ((uint32_t)(val == 0) << 6) | ((uint32_t)(eq && !st) << 12) |
              ((uint32_t)(eq && st) << 18) | ((uint32_t)(!eqdef) << 24);
    f.packB = (ff & 1u) | (((ff >> 1) & 1u) << 6) | (((ff >> 2) & 1u) << 12) | (((ff >> 3) & 1u) << 18) |
              (((ff >> 4) & 1u) << 24);

    // PC-key groups
    if (valid) {
      const unsigned gm = __match_any_sync(vmask, pc);
      apply_group(P, S, gm, pc < P.sp ? (int)pc : -1, pc, f);
    }
    // object-key groups (mapped global records, or the SHARED pseudo-object)
    const uint32_t koi = sh ? P.n_obj : (mapped ? oid : KO_NONE);
    const bool opart = valid && koi != KO_NONE;
    const unsigned omask = __ballot_sync(0xFFFFFFFFu, opart);
    if (opart) {
      const unsigned gm = __match_any_sync(omask, koi);
      apply_group(P, S, gm, koi < P.so ? (int)(P.sp + koi) : -1, P.n_pcs + koi, f);
    }
    // S8 exact histogram on the composite (pc, object key) tag
    if (valid) {
      const uint32_t tag = (pc << 16) | (koi & 0xFFFFu);
      const unsigned tg = __match_any_sync(vmask, tag);
      const unsigned vg = __match_any_sync(tg, val);
      if (lane == __ffs(vg) - 1) hist_insert(P, S, tag, val, __popc(vg));
    }
  }

  if (lane == 0) {
    if (n_invalid) atomicAdd(&S.sctr[0], n_invalid);
    if (n_unmapped) atomicAdd(&S.sctr[1], n_unmapped);
  }
  __syncthreads();

  // fold the CTA's shared state into the global tables
  for (uint32_t i = tid; i < nsk * NSUM; i += blockDim.x) {
    const uint32_t v = S.ssum[i];
    if (v) {
      const uint32_t s = i / NSUM, fld = i % NSUM;
      const uint32_t key = s < P.sp ? s : P.n_pcs + (s - P.sp);
      atomicAdd(&P.t.sum[(uint64_t)key * NSUM + fld], (unsigned long long)v);
    }
  }
  for (uint32_t i = tid; i < nsk * NMM; i += blockDim.x) {
    const uint32_t s = i / NMM, fld = i % NMM;
    const uint32_t key = s < P.sp ? s : P.n_pcs + (s - P.sp);
    if (S.smin[i] != ~0ull) atomic_min_u64(&P.t.mn[(uint64_t)key * NMM + fld], S.smin[i]);
    if (S.smax[i] != 0ull) atomic_max_u64(&P.t.mx[(uint64_t)key * NMM + fld], S.smax[i]);
  }
  for (uint32_t s = tid; s < nsk; s += blockDim.x) {
    if (S.sline[s].state != VE_LINE_EMPTY) {
      const uint32_t key = s < P.sp ? s : P.n_pcs + (s - P.sp);
      line_merge_locked(&P.t.line[key], line_load(S.sline[s]));
    }
  }
  for (uint32_t i = tid; i < P.hs; i += blockDim.x) {
    if (S.shs[i].tag != EMPTY_TAG) hist_insert_global(P.t, S.shs[i].tag, S.shs[i].bits, S.shc[i]);
  }
  if (tid == 0) {
    if (S.sctr[0]) atomicAdd(&P.t.glob[G_INVALID], (unsigned long long)S.sctr[0]);
    if (S.sctr[1]) atomicAdd(&P.t.glob[G_UNMAPPED], (unsigned long long)S.sctr[1]);
    if (blockIdx.x == 0) atomicAdd(&P.t.glob[G_RECORDS], (unsigned long long)P.n);
  }
}

ve_status launch_analyze(ve_ctx* c, const ve_record* d, uint64_t n, cudaStream_t s) {
  AnalyzeParams P;
  P.recs = d;
  P.n = n;
  P.n_pcs = c->cfg.n_pcs;
  P.n_obj = c->n_obj;
  P.mant_bits = c->cfg.mant_bits;
  // shared stat rows: up to 256 keys, PCs first then object keys (incl. SHARED)
  const uint32_t NSK_MAX = 256;
  uint32_t so = c->n_obj + 1 < 128 ? c->n_obj + 1 : 128;
  uint32_t sp = c->cfg.n_pcs < NSK_MAX - so ? c->cfg.n_pcs : NSK_MAX - so;
  so = (c->n_obj + 1 < NSK_MAX - sp) ? c->n_obj + 1 : NSK_MAX - sp;
  P.sp = sp;
  P.so = so;
  P.objc = c->n_obj <= 1024 ? c->n_obj : 0;
  P.o = c->o;
  P.t = c->t;
  int dev_smem = 0;
  cudaDeviceGetAttribute(&dev_smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, c->device);
  uint32_t hs = 8192;
  while (hs > 256 && smem_bytes(sp + so, hs, P.objc) > (size_t)dev_smem - 1024) hs >>= 1;
  P.hs = hs;
  const size_t sb = smem_bytes(sp + so, hs, P.objc);
  cudaError_t e = cudaFuncSetAttribute(k_analyze, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sb);
  if (e != cudaSuccess) return cuda_fail(c, e, "cudaFuncSetAttribute(k_analyze)");
  if (n == 0) return VE_OK;
  uint64_t windows = (n + 31) / 32;
  uint64_t blocks = (windows + 15) / 16;
  if (blocks > (uint64_t)c->num_sms) blocks = (uint64_t)c->num_sms;
  k_analyze<<<(unsigned)blocks, 512, sb, s>>>(P);
  e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "k_analyze launch");
  return VE_OK;
}

}  // namespace ve
