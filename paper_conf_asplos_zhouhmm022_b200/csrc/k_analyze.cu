// k_analyze.cu -- K1: the fused record-analysis pass.
//
// One persistent CTA per SM (16 warps).  Every warp streams its own
// CONTIGUOUS range of 24-byte records (PC, address, size, raw value per
// access) in windows of 32, with the next two windows' loads in flight.  Per
// window each lane decodes one record, maps it to its data object,
// gathers and compares the pre-snapshot bytes (Def 3.1) and derives
// the bit-level value tests of Defs 3.3-3.8.
//
//  * Fast path -- the valid lanes share (pc, access type, object), as a warp's
//    memory instruction does: one set of warp REDUX reductions serves both the
//    PC key and the object key, and is folded into lane-distributed register
//    accumulators (2 key slots per warp, 16 fields each); rows in shared memory
//    are only touched when a slot is evicted.
//  * Slow path -- mixed windows: lanes grouped per key with __match_any_sync,
//    each group reduced and folded into the shared rows directly.
//  * Both paths: exact (pc, object, value) histogram (shared open addressing,
//    overflow to HBM), per-key line states through a warp-private cache of the
//    (+) monoid, written / loaded element bitmaps.
// At exit each CTA folds its shared state into the global tables.  All results
// are integer and order-free, so any grid, chunking or rank split gives the
// same bits (C12).
#include <cuda_runtime.h>

#include "ve_internal.cuh"

namespace ve {

constexpr int K1_THREADS = 512;  // 16 warps x 128 registers
constexpr int K1_WARPS = K1_THREADS / 32;
constexpr int RING = 6;                      // record windows in flight per warp (TMA ring)
constexpr uint32_t WIN_BYTES = 32 * sizeof(ve_record);

struct AnalyzeParams {
  const ve_record* recs;
  uint64_t n;
  uint32_t n_pcs, n_obj;
  uint32_t sp, so;          // shared-memory stat rows for PCs [0,sp) and object keys [0,so)
  uint32_t mant_bits;
  uint32_t hs;              // shared histogram slots (power of 2)
  uint32_t objc;            // objects cached in shared memory (0 = use global table)
  uint32_t dense_ok;        // dense per-element counting enabled for this launch
  uint32_t ring;            // records 16-byte aligned: stream windows with cp.async.bulk
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
  uint8_t* ring;            // [K1_WARPS][RING][WIN_BYTES] TMA ring
  uint64_t* bars;           // [K1_WARPS][RING] mbarriers
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
  b += (size_t)K1_WARPS * RING * (WIN_BYTES + 8);
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
  s.sctr = (uint32_t*)(base + off); off += 16;
  s.ring = base + off; off += (size_t)K1_WARPS * RING * WIN_BYTES;
  s.bars = (uint64_t*)(base + off);
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
    if (lg == 0) return __ldg((const unsigned char*)p);
    if (lg == 1) return __ldg((const unsigned short*)p);
    if (lg == 2) return __ldg((const unsigned int*)p);
    return __ldg((const unsigned long long*)p);
  }
  uint64_t v = 0;
  for (uint32_t i = 0; i < w; ++i) v |= (uint64_t)__ldg((const unsigned char*)(p + i)) << (8 * i);
  return v;
}

// per-lane record facts shared by the key groups
struct Facts {
  uint64_t addr, val, ordv, truncv;
  __int128 y;
  uint32_t tc;
  uint32_t packA, packB;    // 6-bit predicate fields for the packed REDUX sums
  bool nan, isf, pfail;
};

// line state of the points of the lanes in gm (all valid, none pfail)
__device__ __noinline__ void group_line(unsigned gm, const Facts& f, LinePts& g) {
  if (__any_sync(gm, f.pfail)) {
    g.state = VE_LINE_FAIL;
    g.px = g.qx = 0; g.py = g.qy = 0;
    return;
  }
  const uint64_t minx = redmin64(gm, f.addr), maxx = redmax64(gm, f.addr);
  const int pl = __ffs(__ballot_sync(gm, f.addr == minx)) - 1;
  const int ql = __ffs(__ballot_sync(gm, f.addr == maxx)) - 1;
  const uint64_t ylo = (uint64_t)f.y, yhi = (uint64_t)(f.y >> 64);
  // |y| < 2^62 for every point: exact 64x64->128 products, else the generic 128-bit path
  const bool fits = (yhi == (uint64_t)((int64_t)ylo >> 63)) && (ylo + (1ull << 62)) < (1ull << 63);
  const bool small = __all_sync(gm, fits);
  bool ok;
  __int128 py, qy;
  if (small) {
    const int64_t py64 = (int64_t)__shfl_sync(gm, (unsigned long long)ylo, pl);
    const int64_t qy64 = (int64_t)__shfl_sync(gm, (unsigned long long)ylo, ql);
    py = (__int128)py64;
    qy = (__int128)qy64;
    if (minx == maxx) {
      ok = (int64_t)ylo == py64;
    } else {
      const int64_t dxq = (int64_t)(maxx - minx), dx = (int64_t)(f.addr - minx);
      const int64_t dy = (int64_t)ylo - py64, dq = qy64 - py64;
      ok = (dy * dxq == dq * dx) && (__mul64hi(dy, dxq) == __mul64hi(dq, dx));
    }
  } else {
    py = mk128(shfl64(gm, ylo, pl), (int64_t)shfl64(gm, yhi, pl));
    qy = mk128(shfl64(gm, ylo, ql), (int64_t)shfl64(gm, yhi, ql));
    if (minx == maxx) ok = (f.y == py);
    else ok = collinear(minx, py, maxx, qy, f.addr, f.y);
  }
  ok = __all_sync(gm, ok);
  g.state = !ok ? VE_LINE_FAIL : (minx == maxx ? VE_LINE_POINT : VE_LINE_LINE);
  g.px = minx; g.py = py; g.qx = maxx; g.qy = qy;
}

// Slow path: reduce one key group (all lanes in gm share the key) and fold it into
// the key's row: shared memory when slot >= 0, else the global table.
__device__ __noinline__ void apply_group(const AnalyzeParams& P, const Smem& S, unsigned gm, int slot,
                                            uint32_t key, const Facts& f, LinePts& g) {
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
  // C8: the group's line state unless the key's CTA state already FAILed
  g.state = VE_LINE_EMPTY;
  LineState* ls = (slot >= 0) ? &S.sline[slot] : &P.t.line[key];
  // the state may change under us (other warps merge concurrently): decide group-uniformly
  const uint32_t cur = __shfl_sync(gm, *(volatile uint32_t*)&ls->state, __ffs(gm) - 1);
  if (cur == VE_LINE_FAIL) return;
  group_line(gm, f, g);
}

// ---- warp-private line-state cache -------------------------------------------
// Line merges are the only read-modify-write of a wide state; doing them under a
// lock per window serialises warps on keys that stay collinear.  Each warp keeps
// the last WC keys' states privately and folds them into the CTA state only on
// eviction, on the first FAIL (so other warps skip the key early) and at exit.
constexpr int WC = 4;
struct WarpCache {
  uint32_t key1[WC];   // key + 1, 0 = empty
  int32_t slot[WC];
  uint32_t next, pad;
  LineState st[WC];
};

__device__ __forceinline__ LineState* line_target(const AnalyzeParams& P, const Smem& S, int slot, uint32_t key) {
  return (slot >= 0) ? &S.sline[slot] : &P.t.line[key];
}

// returns the key's merged (warp-local) state
__device__ __noinline__ uint32_t wcache_merge(const AnalyzeParams& P, const Smem& S, WarpCache& C, uint32_t key,
                                                 int slot, const LinePts& g) {
  for (int i = 0; i < WC; ++i) {
    if (C.key1[i] == key + 1) {
      const LinePts a = line_load(C.st[i]);
      const LinePts r = line_merge(a, g);
      line_store(C.st[i], r);
      if (r.state == VE_LINE_FAIL && a.state != VE_LINE_FAIL) line_merge_locked(line_target(P, S, slot, key), r);
      return r.state;
    }
  }
  int v = -1;
  for (int i = 0; i < WC; ++i)
    if (C.key1[i] == 0) { v = i; break; }
  if (v < 0) {
    v = (int)(C.next++ % WC);
    line_merge_locked(line_target(P, S, C.slot[v], C.key1[v] - 1), line_load(C.st[v]));
  }
  C.key1[v] = key + 1;
  C.slot[v] = slot;
  line_store(C.st[v], g);
  if (g.state == VE_LINE_FAIL) line_merge_locked(line_target(P, S, slot, key), g);
  return g.state;
}

__device__ __noinline__ void wcache_flush(const AnalyzeParams& P, const Smem& S, WarpCache& C) {
  for (int i = 0; i < WC; ++i) {
    if (C.key1[i]) {
      if (C.st[i].state != VE_LINE_FAIL) line_merge_locked(line_target(P, S, C.slot[i], C.key1[i] - 1), line_load(C.st[i]));
      C.key1[i] = 0;
    }
  }
}

// serialise the merges of this window's group leaders through the warp cache
__device__ __noinline__ void merge_lines(const AnalyzeParams& P, const Smem& S, WarpCache& C, bool lead,
                                            uint32_t key, int slot, const LinePts& g) {
  unsigned L = __ballot_sync(0xFFFFFFFFu, lead && g.state != VE_LINE_EMPTY);
  while (L) {
    const int l = __ffs(L) - 1;
    L &= L - 1;
    if ((int)(threadIdx.x & 31) == l) wcache_merge(P, S, C, key, slot, g);
    __syncwarp();
  }
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

__device__ __noinline__ int find_object(const AnalyzeParams& P, const Smem& S, uint64_t addr) {
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

// ---- fast path: lane-distributed register accumulators -----------------------
// Two key slots per warp; lane l holds field (l & 15) of slot (l >> 4):
//  0 n   1 n_zero   2 n_eq_pre   3 n_nosnap   4 nan   5 nonint   6 not_f16   7 not_bf16
//  8 not_f32   9 raw_min 10 raw_max 11 ord_min 12 ord_max 13 trunc_min 14 trunc_max
// For w <= 4 the ord fields of signed types hold sext32(b)^2^31 (order-isomorphic),
// converted to the 64-bit key at flush.
struct FastSlots {
  uint32_t pc[2], koi[2], meta[2];
  uint32_t used, mru;
  uint32_t lfail[2];     // bit0: PC key line FAIL, bit1: object key line FAIL (known to this warp)
  unsigned long long dense[2];  // per-element counters of this (pc, object), or 0
};

// claim (or find) a dense counter array of sorted object oi for pc (lane 0), broadcast
__device__ __noinline__ unsigned long long dense_lookup(const AnalyzeParams& P, int oi, uint32_t pc) {
  unsigned long long dp = 0;
  if ((threadIdx.x & 31) == 0) {
    for (int j = 0; j < DENSE_PER_OBJ; ++j) {
      uint32_t* slot = &P.o.dense_pc[DENSE_PER_OBJ * oi + j];
      uint32_t d = *(volatile uint32_t*)slot;
      if (d == DENSE_OFF) break;
      if (d == DENSE_FREE) {
        d = atomicCAS(slot, DENSE_FREE, pc);
        if (d == DENSE_FREE) d = pc;
      }
      if (d == pc) {
        dp = (unsigned long long)(P.o.dense_pool + P.o.dense_off[DENSE_PER_OBJ * oi + j]);
        break;
      }
    }
  }
  return __shfl_sync(0xFFFFFFFFu, dp, 0);
}

__device__ __forceinline__ uint64_t fast_identity(int f) {
  return (f >= 9 && (f & 1)) ? ~0ull : 0ull;
}

__device__ __forceinline__ void fold_row(const AnalyzeParams& P, const Smem& S, int slot, uint32_t key, int f,
                                         uint32_t field, uint64_t v) {
  if (f <= 8 || f == 15) {
    if (slot >= 0) atomicAdd(&S.ssum[slot * NSUM + field], (uint32_t)v);
    else atomicAdd(&P.t.sum[(uint64_t)key * NSUM + field], (unsigned long long)v);
  } else {
    const int m = (f - 9) >> 1;
    if (f & 1) atomic_min_u64(slot >= 0 ? &S.smin[slot * NMM + m] : &P.t.mn[(uint64_t)key * NMM + m], v);
    else atomic_max_u64(slot >= 0 ? &S.smax[slot * NMM + m] : &P.t.mx[(uint64_t)key * NMM + m], v);
  }
}

// fold slot s's accumulators into the PC-key row and the object-key row (lanes of half s)
__device__ __noinline__ void fast_flush(const AnalyzeParams& P, const Smem& S, uint32_t pc, uint32_t koi,
                                        uint32_t meta, int s, uint64_t acc) {
  const int lane = threadIdx.x & 31;
  const uint64_t nrec = __shfl_sync(0xFFFFFFFFu, acc, s * 16);   // field 0 of slot s
  if ((lane >> 4) != s) return;
  const int f = lane & 15;
  const uint32_t lg = meta & 3u, kind = (meta >> 2) & 3u;
  const bool st = meta_store(meta);
  uint64_t v = (f == 15) ? nrec : acc;
  if (v == fast_identity(f) && f != 15) return;
  if (f == 15 && v == 0) return;
  uint32_t field;
  if (f == 0) field = st ? F_ST : F_LD;
  else if (f == 1) field = F_ZERO;
  else if (f == 2) field = st ? F_STEQ : F_LDEQ;
  else if (f == 3) field = F_NOSNAP;
  else if (f <= 8) field = F_NAN + (uint32_t)(f - 4);
  else if (f == 15) field = F_TYPE0 + type_code(kind, lg);
  else field = 0;
  if ((f == 11 || f == 12) && kind == 1u && lg < 3u) {
    const int32_t sv = (int32_t)((uint32_t)v ^ 0x80000000u);
    v = (uint64_t)(int64_t)sv ^ (1ull << 63);
  }
  fold_row(P, S, pc < P.sp ? (int)pc : -1, pc, f, field, v);
  if (koi != KO_NONE) fold_row(P, S, koi < P.so ? (int)(P.sp + koi) : -1, P.n_pcs + koi, f, field, v);
}

// per-lane facts of a uniform window handed to its specialised fast path
struct WinCtx {
  uint64_t addr, val, off;
  uint64_t pv;            // pre-snapshot bytes (load in flight), valid iff eqdef
  uint64_t lw0;           // L bitmap word of the first element
  uint32_t lbit;
  uint32_t ew_lg;
  bool valid, eqdef, inside, st;
  unsigned vmask;
  int l0;
  uint32_t pc0, koi0;
};

// warp-uniform cache of the last object a window mapped to
struct ObjCache {
  int oi;
  uint64_t base, end, bmoff, pre;
  uint32_t id, ewlg;
};

// Fast path of a uniform window whose access type (KIND, LG = log2 width) is a
// compile-time constant: the bit tests of C5-C8 specialise to the type.
template <int KIND, int LG>
__device__ __forceinline__ void fast_window(const AnalyzeParams& P, const Smem& S, uint32_t& lfail_s,
                                            unsigned long long dense_s, int s, uint64_t& acc, WarpCache& wc,
                                            const WinCtx& x) {
  constexpr bool ISF = KIND >= 2;
  const int lane = threadIdx.x & 31;
  const uint64_t val = x.val;
  const bool valid = x.valid;
  int64_t ival = 0;
  const uint32_t ff = ISF ? float_flags(val, KIND, LG, ival) : 0u;
  const bool okv = valid && !(ff & 1u);       // contributes to ord / trunc (NaNs excluded)
  const uint32_t nv = __popc(x.vmask);
  uint32_t B = 0;
  if (ISF) {
    const uint32_t pB = valid ? ((ff & 1u) | (((ff >> 1) & 1u) << 6) | (((ff >> 2) & 1u) << 12) |
                                 (((ff >> 3) & 1u) << 18) | (((ff >> 4) & 1u) << 24)) : 0u;
    B = __reduce_add_sync(0xFFFFFFFFu, pB);
  }
  uint64_t rmin, rmax, omin, omax, tmin = ~0ull, tmax = 0;
  if (LG < 3) {
    // w <= 4 bytes: every key fits 32 bits -> one REDUX per min / max
    const uint32_t r32 = (uint32_t)val;
    rmin = __reduce_min_sync(0xFFFFFFFFu, valid ? r32 : 0xFFFFFFFFu);
    rmax = __reduce_max_sync(0xFFFFFFFFu, valid ? r32 : 0u);
    if (KIND == 0) {
      omin = rmin; omax = rmax;
    } else {
      uint32_t k32;
      if (KIND == 1) {                          // sext32(b) ^ 2^31: order-isomorphic to the 64-bit key
        constexpr uint32_t sh = 32 - (8 << LG);
        k32 = (uint32_t)(((int32_t)(r32 << sh)) >> sh) ^ 0x80000000u;
      } else {
        k32 = (uint32_t)ord_key(val, KIND, LG);
      }
      const unsigned okm = __ballot_sync(0xFFFFFFFFu, okv);
      omin = __reduce_min_sync(0xFFFFFFFFu, okv ? k32 : 0xFFFFFFFFu);
      omax = __reduce_max_sync(0xFFFFFFFFu, okv ? k32 : 0u);
      if (ISF) {
        const uint32_t t32 = (uint32_t)trunc_bits(val, KIND, LG, P.mant_bits);
        tmin = __reduce_min_sync(0xFFFFFFFFu, okv ? t32 : 0xFFFFFFFFu);
        tmax = __reduce_max_sync(0xFFFFFFFFu, okv ? t32 : 0u);
      }
      if (okm == 0) { omin = ~0ull; omax = 0; tmin = ~0ull; tmax = 0; }
    }
  } else {
    rmin = redmin64(0xFFFFFFFFu, valid ? val : ~0ull);
    rmax = redmax64(0xFFFFFFFFu, valid ? val : 0ull);
    if (KIND == 0) {
      omin = rmin; omax = rmax;
    } else {
      const uint64_t o = ord_key(val, KIND, LG);
      omin = redmin64(0xFFFFFFFFu, okv ? o : ~0ull);
      omax = redmax64(0xFFFFFFFFu, okv ? o : 0ull);
      if (ISF) {
        const uint64_t t = trunc_bits(val, KIND, LG, P.mant_bits);
        tmin = redmin64(0xFFFFFFFFu, okv ? t : ~0ull);
        tmax = redmax64(0xFFFFFFFFu, okv ? t : 0ull);
      }
    }
  }
  // the pre-snapshot gather is consumed only now
  const bool eq = x.eqdef && x.pv == val;
  const uint32_t pA = valid ? ((uint32_t)(val == 0) | ((uint32_t)eq << 6) | ((uint32_t)!x.eqdef << 12)) : 0u;
  const uint32_t A = __reduce_add_sync(0xFFFFFFFFu, pA);
  const bool lpart = x.inside && !x.st && eq;
  if (__any_sync(0xFFFFFFFFu, lpart)) bitmap_or(P.t.L, lpart, x.lw0, x.lbit);   // C3 loaded elements
  if ((lane >> 4) == s) {
    const int fl = lane & 15;
    if (fl == 0) acc += nv;
    else if (fl <= 3) acc += (A >> (6 * (fl - 1))) & 63u;
    else if (fl <= 8) acc += (B >> (6 * (fl - 4))) & 63u;
    else if (fl <= 14) {
      const int m = (fl - 9) >> 1;
      if (fl & 1) {
        const uint64_t v = m == 0 ? rmin : m == 1 ? omin : tmin;
        acc = v < acc ? v : acc;
      } else {
        const uint64_t v = m == 0 ? rmax : m == 1 ? omax : tmax;
        acc = v > acc ? v : acc;
      }
    }
  }
  // C8: one line state for the window, merged into each key not yet FAIL
  if (lfail_s != 3u) {
    Facts f;
    f.addr = x.addr;
    f.pfail = ISF && (ff & 2u);
    if (KIND == 0) f.y = (__int128)val;
    else if (KIND == 1) {
      constexpr uint32_t sh64 = 64u - (8u << LG);
      f.y = (__int128)((int64_t)(val << sh64) >> sh64);
    } else {
      f.y = (__int128)ival;
    }
    LinePts g;
    g.state = VE_LINE_EMPTY;
    if (valid) group_line(x.vmask, f, g);
    const int ps = x.pc0 < P.sp ? (int)x.pc0 : -1;
    const int os = x.koi0 < P.so ? (int)(P.sp + x.koi0) : -1;
    uint32_t lf = lfail_s;
    if (lane == x.l0) {
      if (!(lf & 1u) && wcache_merge(P, S, wc, x.pc0, ps, g) == VE_LINE_FAIL) lf |= 1u;
      if (!(lf & 2u) && wcache_merge(P, S, wc, P.n_pcs + x.koi0, os, g) == VE_LINE_FAIL) lf |= 2u;
    }
    __syncwarp();
    lfail_s = __shfl_sync(0xFFFFFFFFu, lf, x.l0);
  }
  // S8: exact histogram.  A load that reads an unchanged whole element carries the
  // pre-snapshot value of that element, so it is counted per element (a coalesced
  // counter increment) and mapped to its value at report time; every other record
  // is inserted per distinct value.
  const bool dl = dense_s != 0ull && eq && (uint32_t)LG == x.ew_lg && (x.off & ((1ull << LG) - 1)) == 0;
  if (dl) atomicAdd(reinterpret_cast<uint32_t*>(dense_s) + (x.off >> LG), 1u);
  const unsigned hmask = __ballot_sync(0xFFFFFFFFu, valid && !dl);
  if (valid && !dl) {
    const unsigned vg = (LG < 3) ? __match_any_sync(hmask, (uint32_t)val) : __match_any_sync(hmask, val);
    if (lane == __ffs(vg) - 1) hist_insert(P, S, (x.pc0 << 16) | (x.koi0 & 0xFFFFu), val, __popc(vg));
  }
}

struct Rec {
  uint64_t addr, val, pm;
};

// ---- per-warp TMA ring: cp.async.bulk of whole 768-byte windows into shared memory

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void ring_issue(uint8_t* dst, const void* src, uint64_t* bar) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(WIN_BYTES) : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(WIN_BYTES), "r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void ring_wait(uint64_t* bar, uint32_t phase) {
  uint32_t ok = 0;
  while (!ok) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(phase)
        : "memory");
  }
}

__device__ __forceinline__ Rec load_rec(const AnalyzeParams& P, uint64_t w, uint64_t wend, int lane) {
  Rec r{0, 0, 0};
  const uint64_t i = w * 32 + lane;
  if (w < wend && i < P.n) {
    const unsigned long long* q = reinterpret_cast<const unsigned long long*>(&P.recs[i]);
    r.addr = __ldcs(q);
    r.val = __ldcs(q + 1);
    r.pm = __ldcs(q + 2);
  }
  return r;
}

__global__ void __launch_bounds__(K1_THREADS, 1) k_analyze(AnalyzeParams P) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  const uint32_t nsk = P.sp + P.so;
  Smem S = carve(smem_raw, nsk, P.hs, P.objc);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;

  for (uint32_t i = tid; i < nsk * NSUM; i += blockDim.x) S.ssum[i] = 0;
  for (uint32_t i = tid; i < nsk * NMM; i += blockDim.x) { S.smin[i] = ~0ull; S.smax[i] = 0; }
  for (uint32_t i = tid; i < nsk; i += blockDim.x) { S.sline[i].state = VE_LINE_EMPTY; S.sline[i].lock = 0; }
  for (uint32_t i = tid; i < P.hs; i += blockDim.x) {
    S.shs[i].bits = 0; S.shs[i].tag = EMPTY_TAG; S.shs[i].pad = 0; S.shc[i] = 0;
  }
  for (uint32_t i = tid; i < P.objc; i += blockDim.x) { S.sob[i] = P.o.base[i]; S.soe[i] = P.o.end[i]; }
  if (tid < 4) S.sctr[tid] = 0;
  __shared__ WarpCache s_wc[K1_WARPS];
  WarpCache& wc = s_wc[warp];
  if (lane < WC) wc.key1[lane] = 0;
  if (lane == 0) wc.next = 0;

  // this warp's contiguous range of windows; full windows stream through a TMA ring
  const uint64_t nwin = (P.n + 31) / 32;
  const uint64_t tw = (uint64_t)gridDim.x * K1_WARPS, gw = (uint64_t)blockIdx.x * K1_WARPS + warp;
  const uint64_t wbeg = gw * nwin / tw, wend = (gw + 1) * nwin / tw;
  const uint64_t nfull = P.n / 32;
  const uint64_t rend = P.ring ? (wend < nfull ? wend : nfull) : wbeg;   // ring covers [wbeg, rend)
  uint8_t (*s_ring)[RING][WIN_BYTES] = reinterpret_cast<uint8_t (*)[RING][WIN_BYTES]>(S.ring);
  uint64_t (*s_bar)[RING] = reinterpret_cast<uint64_t (*)[RING]>(S.bars);
  if (lane == 0) {
    for (int d = 0; d < RING; ++d) mbar_init(&s_bar[warp][d], 1);
    fence_mbar_init();
    for (int d = 0; d < RING && wbeg + d < rend; ++d)
      ring_issue(s_ring[warp][d], P.recs + (wbeg + d) * 32, &s_bar[warp][d]);
  }
  __syncthreads();
  ObjCache oc;
  oc.oi = -1; oc.base = oc.end = oc.bmoff = oc.pre = 0; oc.id = 0; oc.ewlg = 0;
  uint32_t n_invalid = 0, n_unmapped = 0;
  FastSlots F;
  F.used = 0;
  F.mru = 0;
  uint64_t acc = 0;

  for (uint64_t w = wbeg; w < wend; ++w) {
    Rec cur;
    if (w < rend) {
      const uint64_t i = w - wbeg;
      const int d = (int)(i % RING);
      ring_wait(&s_bar[warp][d], (uint32_t)((i / RING) & 1));
      const unsigned long long* q = reinterpret_cast<const unsigned long long*>(s_ring[warp][d] + lane * 24);
      cur.addr = q[0];
      cur.val = q[1];
      cur.pm = q[2];
      __syncwarp();
      if (lane == 0 && w + RING < rend) {
        fence_proxy_async();   // our generic reads of the stage precede the next async write
        ring_issue(s_ring[warp][d], P.recs + (w + RING) * 32, &s_bar[warp][d]);
      }
    } else {
      cur = load_rec(P, w, wend, lane);
    }
    const uint64_t addr = cur.addr, val = cur.val;
    const uint32_t pc = (uint32_t)cur.pm, meta = (uint32_t)(cur.pm >> 32);
    const bool full = (w + 1) * 32 <= P.n;
    const bool inrange = full || (w * 32 + lane < P.n);

    // S1 decode + validate
    const bool valid = inrange && rec_valid(addr, val, pc, meta, P.n_pcs);
    const unsigned vmask = __ballot_sync(0xFFFFFFFFu, valid);
    if (lane == 0) n_invalid += (full ? 32u : (uint32_t)min((uint64_t)32, P.n - w * 32)) - (uint32_t)__popc(vmask);
    if (vmask == 0) continue;
    const uint32_t lg = meta & 3u, kind = (meta >> 2) & 3u;
    const bool st = meta_store(meta), sh = meta_shared(meta);

    // S2 address -> object: warp-uniform cached object, binary search only on a miss
    const bool need = valid && !sh;
    const bool hit = need && oc.oi >= 0 && addr >= oc.base && addr < oc.end;
    int oi = hit ? oc.oi : -1;
    uint64_t ob = oc.base, oe = oc.end, obm = oc.bmoff, opre = oc.pre;
    uint32_t oid = oc.id, oewlg = oc.ewlg;
    const unsigned missm = __ballot_sync(0xFFFFFFFFu, need && !hit);
    if (missm) {
      if (need && !hit) {
        oi = find_object(P, S, addr);
        if (oi >= 0) {
          ob = P.objc ? S.sob[oi] : P.o.base[oi];
          oe = P.objc ? S.soe[oi] : P.o.end[oi];
          obm = P.o.bmoff[oi];
          opre = P.o.pre[oi];
          oid = P.o.id[oi];
          const uint32_t ew = P.o.ew[oi];
          oewlg = (ew == 1) ? 0 : (ew == 2) ? 1 : (ew == 4) ? 2 : 3;
        }
      }
      const unsigned mm = __ballot_sync(0xFFFFFFFFu, need && !hit && oi >= 0);
      if (mm) {                                    // adopt the first newly found object
        const int src = __ffs(mm) - 1;
        oc.oi = __shfl_sync(0xFFFFFFFFu, oi, src);
        oc.base = __shfl_sync(0xFFFFFFFFu, ob, src);
        oc.end = __shfl_sync(0xFFFFFFFFu, oe, src);
        oc.bmoff = __shfl_sync(0xFFFFFFFFu, obm, src);
        oc.pre = __shfl_sync(0xFFFFFFFFu, opre, src);
        oc.id = __shfl_sync(0xFFFFFFFFu, oid, src);
        oc.ewlg = __shfl_sync(0xFFFFFFFFu, oewlg, src);
      }
      const unsigned um = __ballot_sync(0xFFFFFFFFu, need && oi < 0);
      if (lane == 0) n_unmapped += __popc(um);
    }
    const bool mapped = oi >= 0;

    // S3 snapshot gather + eq_pre
    const uint32_t ew_lg = mapped ? oewlg : 0u;
    const uint64_t off = mapped ? addr - ob : 0ull;
    const uint64_t bmoff = mapped ? obm : 0ull;
    const bool inside = mapped && addr + (1u << lg) <= oe;
    const bool eqdef = inside && opre != 0ull;
    // issue the pre-snapshot gather now, consume it as late as possible (latency hiding)
    const uint64_t pv = eqdef ? load_pre(opre + off, lg) : 0ull;
    const uint32_t koi = sh ? P.n_obj : (mapped ? oid : KO_NONE);
    const uint64_t lw0 = bmoff + ((off >> ew_lg) >> 5);        // L bitmap word / bit of the first element
    const uint32_t lbit = 1u << ((off >> ew_lg) & 31);

    // W element bitmap (C10); L is set once eq_pre is known
    {
      const bool wpart = inside && st;
      const uint64_t e0 = off >> ew_lg, e1 = (off + (1u << lg) - 1) >> ew_lg;
      const uint64_t w0 = bmoff + (e0 >> 5), w1 = bmoff + (e1 >> 5);
      const unsigned wany = __ballot_sync(0xFFFFFFFFu, wpart);
      if (wany) {
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
      }
    }

    // uniform window? (pc, access type and object shared by every valid lane)
    const int l0 = __ffs(vmask) - 1;
    const uint32_t pc0 = __shfl_sync(0xFFFFFFFFu, pc, l0);
    const uint32_t meta0 = __shfl_sync(0xFFFFFFFFu, meta, l0);
    const uint32_t koi0 = __shfl_sync(0xFFFFFFFFu, koi, l0);
    const bool uniform = __all_sync(0xFFFFFFFFu, !valid || (pc == pc0 && meta == meta0 && koi == koi0));

    if (uniform) {
      // ---------------- fast path ----------------
      // select / install the register slot for (pc, object key, access type)
      int s;
      if ((F.used & 1u) && F.pc[0] == pc0 && F.koi[0] == koi0 && F.meta[0] == meta0) s = 0;
      else if ((F.used & 2u) && F.pc[1] == pc0 && F.koi[1] == koi0 && F.meta[1] == meta0) s = 1;
      else {
        s = !(F.used & 1u) ? 0 : !(F.used & 2u) ? 1 : (int)(F.mru ^ 1u);
        if (F.used & (1u << s)) {
          if (s) fast_flush(P, S, F.pc[1], F.koi[1], F.meta[1], 1, acc);
          else fast_flush(P, S, F.pc[0], F.koi[0], F.meta[0], 0, acc);
        }
        F.used |= 1u << s;
        // constant indices only: the slot table stays in registers
        if (s) { F.pc[1] = pc0; F.koi[1] = koi0; F.meta[1] = meta0; }
        else { F.pc[0] = pc0; F.koi[0] = koi0; F.meta[0] = meta0; }
        if ((lane >> 4) == s) acc = fast_identity(lane & 15);
        // line states this warp can skip (already FAIL in the CTA state)
        const int ps = pc0 < P.sp ? (int)pc0 : -1;
        uint32_t lf = (line_target(P, S, ps, pc0)->state == VE_LINE_FAIL) ? 1u : 0u;
        if (koi0 == KO_NONE) lf |= 2u;
        else {
          const int os = koi0 < P.so ? (int)(P.sp + koi0) : -1;
          if (line_target(P, S, os, P.n_pcs + koi0)->state == VE_LINE_FAIL) lf |= 2u;
        }
        lf = __shfl_sync(0xFFFFFFFFu, lf, 0);
        // dense per-element counting for loads of a real object that read the pre value
        const int oi0 = __shfl_sync(0xFFFFFFFFu, oi, l0);
        const unsigned long long dn =
            (P.dense_ok && oi0 >= 0 && !meta_store(meta0)) ? dense_lookup(P, oi0, pc0) : 0ull;
        if (s) { F.lfail[1] = lf; F.dense[1] = dn; }
        else { F.lfail[0] = lf; F.dense[0] = dn; }
      }
      F.mru = (uint32_t)s;
      uint32_t lf_s = s ? F.lfail[1] : F.lfail[0];
      const unsigned long long dn_s = s ? F.dense[1] : F.dense[0];
      WinCtx x;
      x.addr = addr; x.val = val; x.off = off; x.ew_lg = ew_lg;
      x.valid = valid; x.eqdef = eqdef; x.inside = inside; x.st = st;
      x.pv = pv; x.lw0 = lw0; x.lbit = lbit;
      x.vmask = vmask; x.l0 = l0; x.pc0 = pc0; x.koi0 = koi0;
      // specialised on the window's access type (compile-time width / kind)
      switch (meta0 & 15u) {
        case 0: fast_window<0, 0>(P, S, lf_s, dn_s, s, acc, wc, x); break;
        case 1: fast_window<0, 1>(P, S, lf_s, dn_s, s, acc, wc, x); break;
        case 2: fast_window<0, 2>(P, S, lf_s, dn_s, s, acc, wc, x); break;
        case 3: fast_window<0, 3>(P, S, lf_s, dn_s, s, acc, wc, x); break;
        case 4: fast_window<1, 0>(P, S, lf_s, dn_s, s, acc, wc, x); break;
        case 5: fast_window<1, 1>(P, S, lf_s, dn_s, s, acc, wc, x); break;
        case 6: fast_window<1, 2>(P, S, lf_s, dn_s, s, acc, wc, x); break;
        case 7: fast_window<1, 3>(P, S, lf_s, dn_s, s, acc, wc, x); break;
        case 9: fast_window<2, 1>(P, S, lf_s, dn_s, s, acc, wc, x); break;
        case 10: fast_window<2, 2>(P, S, lf_s, dn_s, s, acc, wc, x); break;
        case 11: fast_window<2, 3>(P, S, lf_s, dn_s, s, acc, wc, x); break;
        default: fast_window<3, 1>(P, S, lf_s, dn_s, s, acc, wc, x); break;   // 13: bfloat16
      }
      if (s) F.lfail[1] = lf_s;
      else F.lfail[0] = lf_s;
    } else {
      // ---------------- slow path: per-key groups ----------------
      const bool eq = eqdef && pv == val;
      const bool lpart = inside && !st && eq;
      if (__any_sync(0xFFFFFFFFu, lpart)) bitmap_or(P.t.L, lpart, lw0, lbit);   // C3 loaded elements
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
      LinePts gp, go;
      gp.state = go.state = VE_LINE_EMPTY;
      bool leadp = false, leado = false;
      const int pslot = pc < P.sp ? (int)pc : -1;
      if (valid) {
        const unsigned gm = __match_any_sync(vmask, pc);
        apply_group(P, S, gm, pslot, pc, f, gp);
        leadp = lane == __ffs(gm) - 1;
      }
      const bool opart = valid && koi != KO_NONE;
      const unsigned omask = __ballot_sync(0xFFFFFFFFu, opart);
      const int oslot = koi < P.so ? (int)(P.sp + koi) : -1;
      if (opart) {
        const unsigned gm = __match_any_sync(omask, koi);
        apply_group(P, S, gm, oslot, P.n_pcs + koi, f, go);
        leado = lane == __ffs(gm) - 1;
      }
      merge_lines(P, S, wc, leadp, pc, pslot, gp);
      merge_lines(P, S, wc, leado, P.n_pcs + koi, oslot, go);
      if (valid) {
        const uint32_t tag = (pc << 16) | (koi & 0xFFFFu);
        const unsigned tg = __match_any_sync(vmask, tag);
        const unsigned vg = __match_any_sync(tg, val);
        if (lane == __ffs(vg) - 1) hist_insert(P, S, tag, val, __popc(vg));
      }
    }
  }

  // fold the warp's register slots and line cache, then the CTA's shared state
  if (F.used & 1u) fast_flush(P, S, F.pc[0], F.koi[0], F.meta[0], 0, acc);
  if (F.used & 2u) fast_flush(P, S, F.pc[1], F.koi[1], F.meta[1], 1, acc);
  if (lane == 0) {
    if (n_invalid) atomicAdd(&S.sctr[0], n_invalid);
    if (n_unmapped) atomicAdd(&S.sctr[1], n_unmapped);
    wcache_flush(P, S, wc);
  }
  __syncthreads();

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
  // u32 per-element counters cannot overflow while the ctx has seen < 2^32 records
  P.dense_ok = (c->dense_used > 0 && c->records_analyzed + n < (1ull << 32)) ? 1u : 0u;
  P.ring = ((uintptr_t)d % 16 == 0) ? 1u : 0u;
  c->records_analyzed += n;
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
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, k_analyze);
  const size_t budget = (size_t)dev_smem - fa.sharedSizeBytes - 1024;   // dynamic smem left after the TMA ring
  uint32_t hs = 8192;
  while (hs > 256 && smem_bytes(sp + so, hs, P.objc) > budget) hs >>= 1;
  P.hs = hs;
  const size_t sb = smem_bytes(sp + so, hs, P.objc);
  cudaError_t e = cudaFuncSetAttribute(k_analyze, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sb);
  if (e != cudaSuccess) return cuda_fail(c, e, "cudaFuncSetAttribute(k_analyze)");
  if (n == 0) return VE_OK;
  uint64_t windows = (n + 31) / 32;
  uint64_t blocks = (windows + K1_WARPS - 1) / K1_WARPS;
  if (blocks > (uint64_t)c->num_sms) blocks = (uint64_t)c->num_sms;
  count_launch();
  k_analyze<<<(unsigned)blocks, K1_THREADS, sb, s>>>(P);
  e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "k_analyze launch");
  return VE_OK;
}

}  // namespace ve
