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

#include <cstdlib>
#include <type_traits>

#include "ve_internal.cuh"

namespace ve {

#ifndef VE_K1_THREADS
#define VE_K1_THREADS 512
#endif
constexpr int K1_THREADS = VE_K1_THREADS;  // 16 warps x 128 registers
constexpr int K1_WARPS = K1_THREADS / 32;
#ifndef VE_RING
#define VE_RING 8
#endif
constexpr int RING = VE_RING;                // record windows per warp ring (2 stages)
constexpr uint32_t WIN_BYTES = 32 * sizeof(ve_record);
constexpr uint64_t STAGE_RS_MAX = 16384;      // S8 staging entries per warp (16 B each)

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
  uint64_t nring;           // full windows (streamed through the per-warp rings)
  uint32_t chunk;           // windows per static chunk (VE_CLAIM 2): CHUNK, or one stage for short traces
  uint32_t claim;           // 1: chunks claimed from the global counter *work (guided), 0: static interleave
  uint64_t nbig;            // claim mode: chunks of P.chunk windows before the one-stage tail chunks
  // units mode (ve_analyze_units, K1 v2 only): independent traces in one launch.  Unit u's records
  // are units[u].recs (16-byte aligned); its PCs are keys pcb .. pcb + npc - 1 (a record's pc is
  // local: pc >= npc is invalid) and its objects the sorted table entries [olo, ohi).  Chunk c of
  // the launch is chunk c - ucb[u] of the unit u with ucb[u] <= c < ucb[u + 1].
  const struct UnitDesc* units;
  const uint32_t* ucb;      // [n_units + 1] chunk prefix
  uint32_t n_units;
  unsigned long long* work; // chunk claim counter (zeroed before the launch)
  // S8 insert staging: a private region of stage_rs 16-byte entries per warp for the
  // (tag, bits, count) groups the shared table cannot take; k_hist_drain inserts them
  // into the HBM table after K1, at full occupancy, instead of K1's 16 warps/SM
  // waiting on one global CAS round trip per group
  uint4* stage;             // [grid * K1_WARPS][stage_rs]
  uint32_t* stage_cnt;      // [grid * K1_WARPS] entries written (<= stage_rs)
  uint32_t stage_rs;
  // byte offsets of the dynamic shared-memory regions (see carve_offsets)
  uint32_t o_ssum, o_smin, o_smax, o_sline, o_shs, o_shc, o_sob, o_soe, o_sctr, o_ring, o_bars;
  DevObjects o;
  DevTables t;
};

struct UnitDesc {
  const ve_record* recs;
  uint64_t n;
  uint32_t pcb, npc;        // key base and count of the unit's PCs
  uint32_t olo, ohi;        // the unit's objects in the sorted table
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

// region offsets, computed once on the host (kernel code reads them from the
// constant bank, so no pointer table lives in registers or on the stack)
inline void carve_offsets(AnalyzeParams& P, uint32_t nsk) {
  size_t off = 0;
  P.o_ssum = (uint32_t)off; off += align16(sizeof(uint32_t) * nsk * NSUM);
  P.o_smin = (uint32_t)off; off += align16(sizeof(unsigned long long) * nsk * NMM);
  P.o_smax = (uint32_t)off; off += align16(sizeof(unsigned long long) * nsk * NMM);
  P.o_sline = (uint32_t)off; off += align16(sizeof(LineState) * nsk);
  P.o_shs = (uint32_t)off; off += align16(sizeof(HSlot) * P.hs);
  P.o_shc = (uint32_t)off; off += align16(sizeof(uint32_t) * P.hs);
  P.o_sob = (uint32_t)off; off += align16(sizeof(uint64_t) * P.objc);
  P.o_soe = (uint32_t)off; off += align16(sizeof(uint64_t) * P.objc);
  P.o_sctr = (uint32_t)off; off += 16;
  P.o_ring = (uint32_t)off; off += (size_t)K1_WARPS * RING * WIN_BYTES;
  P.o_bars = (uint32_t)off;
}

extern __shared__ __align__(16) uint8_t ve_smem[];

__device__ __forceinline__ Smem smem_of(const AnalyzeParams& P) {
  Smem s;
  s.ssum = (uint32_t*)(ve_smem + P.o_ssum);
  s.smin = (unsigned long long*)(ve_smem + P.o_smin);
  s.smax = (unsigned long long*)(ve_smem + P.o_smax);
  s.sline = (LineState*)(ve_smem + P.o_sline);
  s.shs = (HSlot*)(ve_smem + P.o_shs);
  s.shc = (uint32_t*)(ve_smem + P.o_shc);
  s.sob = (uint64_t*)(ve_smem + P.o_sob);
  s.soe = (uint64_t*)(ve_smem + P.o_soe);
  s.sctr = (uint32_t*)(ve_smem + P.o_sctr);
  s.ring = ve_smem + P.o_ring;
  s.bars = (uint64_t*)(ve_smem + P.o_bars);
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
__device__ __noinline__ void apply_group(const AnalyzeParams& P, unsigned gm, int slot,
                                            uint32_t key, const Facts& f, LinePts& g) {
  const Smem S = smem_of(P);
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
#ifndef VE_WC
#define VE_WC 4
#endif
constexpr int WC = VE_WC;
struct WarpCache {
  uint32_t key1[WC];   // key + 1, 0 = empty
  int32_t slot[WC];
  uint32_t next, pad;
  LineState st[WC];
};

__device__ __forceinline__ LineState* line_target(const AnalyzeParams& P, int slot, uint32_t key) {
  const Smem S = smem_of(P);
  return (slot >= 0) ? &S.sline[slot] : &P.t.line[key];
}

// returns the key's merged (warp-local) state
__device__ __noinline__ uint32_t wcache_merge(const AnalyzeParams& P, WarpCache& C, uint32_t key,
                                                 int slot, const LinePts& g) {
  const Smem S = smem_of(P);
  for (int i = 0; i < WC; ++i) {
    if (C.key1[i] == key + 1) {
      const LinePts a = line_load(C.st[i]);
      const LinePts r = line_merge(a, g);
      line_store(C.st[i], r);
      if (r.state == VE_LINE_FAIL && a.state != VE_LINE_FAIL) line_merge_locked(line_target(P, slot, key), r);
      return r.state;
    }
  }
  int v = -1;
  for (int i = 0; i < WC; ++i)
    if (C.key1[i] == 0) { v = i; break; }
  if (v < 0) {
    v = (int)(C.next++ % WC);
    line_merge_locked(line_target(P, C.slot[v], C.key1[v] - 1), line_load(C.st[v]));
  }
  C.key1[v] = key + 1;
  C.slot[v] = slot;
  line_store(C.st[v], g);
  if (g.state == VE_LINE_FAIL) line_merge_locked(line_target(P, slot, key), g);
  return g.state;
}

__device__ __noinline__ void wcache_flush(const AnalyzeParams& P, WarpCache& C) {
  const Smem S = smem_of(P);
  for (int i = 0; i < WC; ++i) {
    if (C.key1[i]) {
      if (C.st[i].state != VE_LINE_FAIL) line_merge_locked(line_target(P, C.slot[i], C.key1[i] - 1), line_load(C.st[i]));
      C.key1[i] = 0;
    }
  }
}

// serialise the merges of this window's group leaders through the warp cache
__device__ __noinline__ void merge_lines(const AnalyzeParams& P, WarpCache& C, bool lead,
                                            uint32_t key, int slot, const LinePts& g) {
  const Smem S = smem_of(P);
  unsigned L = __ballot_sync(0xFFFFFFFFu, lead && g.state != VE_LINE_EMPTY);
  while (L) {
    const int l = __ffs(L) - 1;
    L &= L - 1;
    if ((int)(threadIdx.x & 31) == l) wcache_merge(P, C, key, slot, g);
    __syncwarp();
  }
}

__shared__ uint32_t s_stage_n[K1_WARPS];   // entries claimed in the warp's staging region
__shared__ uint32_t s_urange[K1_WARPS][2];  // units mode: the object range [lo, hi) of the warp's current unit

// Stage a (tag, bits, c) group for k_hist_drain; the HBM table directly once the
// warp's region is full.  A plain store: the warp does not wait on it.
__device__ __forceinline__ void hist_stage(const AnalyzeParams& P, uint32_t tag, uint64_t bits, uint32_t c) {
  const uint32_t w = threadIdx.x >> 5;
  const uint32_t pos = atomicAdd(&s_stage_n[w], 1u);
  if (pos < P.stage_rs) {
    uint4* q = P.stage + ((uint64_t)blockIdx.x * K1_WARPS + w) * P.stage_rs + pos;
    __stcg(q, make_uint4((uint32_t)bits, (uint32_t)(bits >> 32), tag, c));
  } else {
    hist_insert_global(P.t, tag, bits, c);
  }
}

// Shared-table part of an S8 insert: add count c to (tag, bits) in the CTA's table.
// Returns false if the group was not placed.  The table is kept at most half full;
// once it is, only the first two probe positions are searched for an existing entry.
// (Placing a group in the shared table, the staging region or the HBM table is
// equally exact: every part is summed into the HBM table in the end.)
__device__ __forceinline__ bool hist_insert_shared(const AnalyzeParams& P, uint32_t tag, uint64_t bits, uint32_t c) {
  const Smem S = smem_of(P);
  const uint32_t hmask = P.hs - 1;
  const bool full = *(volatile uint32_t*)&S.sctr[2] >= (P.hs >> 1);
  const int np = full ? 2 : 16;
  uint32_t h = (uint32_t)hist_hash(tag, bits) & hmask;
  for (int probe = 0; probe < np; ++probe) {
    HSlot* s = &S.shs[h];
    // one 16-byte read of the slot.  An empty slot is (bits 0, EMPTY_TAG, pad 0) and a claim
    // replaces both words by one 128-bit CAS; should a read ever combine the old bits with
    // the new tag, it would look like an entry of value 0 -- so a match of value 0 is
    // confirmed by the CAS, never taken from the read
    uint64_t lo, hi;
    asm volatile("ld.volatile.shared.v2.u64 {%0, %1}, [%2];"
                 : "=l"(lo), "=l"(hi) : "r"((uint32_t)__cvta_generic_to_shared(s)) : "memory");
    const uint32_t stag = (uint32_t)hi;
    if (stag == tag && lo == bits && bits != 0ull) { atomicAdd(&S.shc[h], c); return true; }
    if (stag == EMPTY_TAG || (stag == tag && lo == bits)) {
      if (stag == EMPTY_TAG && *(volatile uint32_t*)&S.sctr[2] >= (P.hs >> 1)) return false;   // at most half full
      uint64_t olo, ohi;
      cas128_shared(s, 0ull, (uint64_t)EMPTY_TAG, bits, (uint64_t)tag, olo, ohi);
      if ((uint32_t)ohi == EMPTY_TAG && olo == 0ull) {
        atomicAdd(&S.sctr[2], 1u);
        atomicAdd(&S.shc[h], c);
        return true;
      }
      if ((uint32_t)ohi == tag && olo == bits) { atomicAdd(&S.shc[h], c); return true; }
    }
    h = (h + 1) & hmask;
  }
  return false;
}

// Insert a group of equal (tag, bits) with count c: shared table first, then the
// warp's staging region (HBM table on miss/full, via k_hist_drain).
__device__ __forceinline__ void hist_insert(const AnalyzeParams& P, uint32_t tag, uint64_t bits,
                                            uint32_t c) {
  if (!hist_insert_shared(P, tag, bits, c)) hist_stage(P, tag, bits, c);
}

// Warp-collective insert of the groups led by the lanes with lead set (act = the
// lanes executing this call): shared table, then one staging claim for the warp.
__device__ __forceinline__ void hist_insert_warp(const AnalyzeParams& P, unsigned act, bool lead, uint32_t tag,
                                                 uint64_t bits, uint32_t c) {
  const bool need = lead && !hist_insert_shared(P, tag, bits, c);
  const unsigned F = __ballot_sync(act, need);
  if (!F) return;
  const int lane = threadIdx.x & 31, l0 = __ffs(act) - 1;
  const uint32_t w = threadIdx.x >> 5;
  uint32_t base = 0;
  if (lane == l0) base = atomicAdd(&s_stage_n[w], (uint32_t)__popc(F));
  base = __shfl_sync(act, base, l0);
  if (need) {
    const uint32_t pos = base + (uint32_t)__popc(F & ((1u << lane) - 1u));
    if (pos < P.stage_rs) {
      uint4* q = P.stage + ((uint64_t)blockIdx.x * K1_WARPS + w) * P.stage_rs + pos;
      __stcg(q, make_uint4((uint32_t)bits, (uint32_t)(bits >> 32), tag, c));
    } else {
      hist_insert_global(P.t, tag, bits, c);
    }
  }
}

__device__ __noinline__ int find_object(const AnalyzeParams& P, uint64_t addr) {
  const Smem S = smem_of(P);
  const uint64_t* base = P.objc ? S.sob : P.o.base;
  int lo = 0, hi = (int)P.o.n;  // first object with base > addr
  if (P.units) {                // units mode: only the current unit's objects
    lo = (int)s_urange[threadIdx.x >> 5][0];
    hi = (int)s_urange[threadIdx.x >> 5][1];
  }
  const int lo0 = lo;
  while (lo < hi) {
    int mid = (lo + hi) >> 1;
    if (base[mid] <= addr) lo = mid + 1; else hi = mid;
  }
  if (lo == lo0) return -1;
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

// ---- fast path key slots ------------------------------------------------------
// A fast window's statistics are warp-uniform REDUX results, accumulated into the
// totals of its key slot (pc, object, access type).  The active slot lives in
// registers inside run_fast; each warp keeps NSLOT slots in a private shared-memory
// cache and folds a slot into the PC-key and object-key rows only on eviction and
// at exit.  For w <= 4 the min / max totals are 32-bit forms: ord of signed types
// is sext32(b)^2^31 (order-isomorphic to the 64-bit key), and 0xFFFFFFFF is the min
// identity of ord / trunc of floats (no non-NaN key has that value).
#ifndef VE_NSLOT
#define VE_NSLOT 8
#endif
constexpr int NSLOT = VE_NSLOT;          // slots of the multi-key kernel (cfg4 rotates 8 PCs)
#ifndef VE_NSLOT_SINGLE
#define VE_NSLOT_SINGLE 4
#endif
constexpr int NSLOT_SINGLE = VE_NSLOT_SINGLE;   // slots of the single-key kernel (few-PC traces)
struct __align__(16) SlotE {
  uint64_t key;                 // meta << 32 | object id << 16 | pc; ~0 = free
  unsigned long long dense;     // per-element counters of (pc, object), or 0
  uint64_t mm[6];               // raw min, raw max, ord min, ord max, trunc min, trunc max
  uint32_t nwin;                // windows (32 records each)
  uint32_t lfail;               // bit0: PC key line FAIL, bit1: object key line FAIL (known to this warp)
  uint32_t nosnap;              // the object has no pre snapshot
  uint32_t pad;
  uint32_t sum[8];              // zero, eq_pre, nan, nonint, not_f16, not_bf16, not_f32, -
  // C8 of constant runs, deferred: while the key's line is live, consecutive runs of
  // one value cy only widen [cx0, cx1]; the horizontal segment is merged once (the
  // (+) monoid keeps only the extreme points, so this equals merging every run)
  uint64_t cy, cx0, cx1;
  uint32_t cpend;               // a deferred constant segment is held
  uint32_t pad2;
};
static_assert(sizeof(SlotE) == 144, "SlotE layout");

__device__ __noinline__ uint32_t const_line(const AnalyzeParams& P, WarpCache& wc, uint64_t xmin, uint64_t xmax,
                                            uint64_t cy, uint32_t meta0, uint32_t pc0, uint32_t koi0, uint32_t lf);

// merge a slot's deferred constant segment into the line states (all lanes)
__device__ __noinline__ void slot_line_flush(const AnalyzeParams& P, WarpCache& wc, SlotE* e) {
  if (!e->cpend) return;
  const uint64_t key = e->key;
  const uint32_t lf = const_line(P, wc, e->cx0, e->cx1, e->cy, (uint32_t)(key >> 32), (uint32_t)key & 0xFFFFu,
                                 (uint32_t)(key >> 16) & 0xFFFFu, e->lfail);
  __syncwarp();
  if ((threadIdx.x & 31) == 0) { e->lfail = lf; e->cpend = 0; }
  __syncwarp();
}

// claim (or find) a dense counter array of sorted object oi for the loads of one
// (pc, access type): claim key ck = meta << 16 | pc (lane 0), broadcast.  The claimer
// takes the array from the pool (bump allocation) and publishes its offset; a warp
// finding the slot already claimed by ck waits for that offset (a few cycles).
__device__ __noinline__ unsigned long long dense_lookup(const AnalyzeParams& P, int oi, uint32_t ck) {
  unsigned long long dp = 0;
  if ((threadIdx.x & 31) == 0) {
    const uint64_t ne = (P.o.end[oi] - P.o.base[oi] + P.o.ew[oi] - 1) / P.o.ew[oi];
    for (int j = 0; j < DENSE_PER_OBJ; ++j) {
      const int si = DENSE_PER_OBJ * oi + j;
      uint32_t* slot = &P.o.dense_pc[si];
      uint32_t d = *(volatile uint32_t*)slot;
      if (d == DENSE_OFF) break;
      if (d == DENSE_FREE) {
        d = atomicCAS(slot, DENSE_FREE, ck);
        if (d == DENSE_FREE) {                       // ours: allocate and publish
          const unsigned long long off = atomicAdd(P.o.dense_next, (unsigned long long)ne);
          atomicExch(&P.o.dense_off[si], off + ne <= P.o.dense_cap ? off : DENSE_NONE);
          d = ck;
        }
      }
      if (d == ck) {
        unsigned long long off;
        while ((off = *(volatile unsigned long long*)&P.o.dense_off[si]) == DENSE_NOT_READY) {
        }
        if (off != DENSE_NONE) dp = (unsigned long long)(P.o.dense_pool + off);
        break;
      }
    }
  }
  return __shfl_sync(0xFFFFFFFFu, dp, 0);
}

// line states of (pc, object id) this warp can skip (already FAIL in the CTA state)
__device__ __noinline__ uint32_t slot_lfail(const AnalyzeParams& P, uint32_t pc, uint32_t koi) {
  const Smem S = smem_of(P);
  const int ps = pc < P.sp ? (int)pc : -1;
  const int os = koi < P.so ? (int)(P.sp + koi) : -1;
  uint32_t lf = (line_target(P, ps, pc)->state == VE_LINE_FAIL) ? 1u : 0u;
  if (line_target(P, os, P.n_pcs + koi)->state == VE_LINE_FAIL) lf |= 2u;
  return __shfl_sync(0xFFFFFFFFu, lf, 0);
}

// field f of a key row: f <= 8 or 15 a sum, f = 9..14 min (odd) / max (even)
__device__ __forceinline__ void fold_row(const AnalyzeParams& P, int slot, uint32_t key, int f, uint32_t field,
                                         uint64_t v) {
  const Smem S = smem_of(P);
  if (f <= 8 || f == 15) {
    if (slot >= 0) atomicAdd(&S.ssum[slot * NSUM + field], (uint32_t)v);
    else atomicAdd(&P.t.sum[(uint64_t)key * NSUM + field], (unsigned long long)v);
  } else {
    const int m = (f - 9) >> 1;
    if (f & 1) atomic_min_u64(slot >= 0 ? &S.smin[slot * NMM + m] : &P.t.mn[(uint64_t)key * NMM + m], v);
    else atomic_max_u64(slot >= 0 ? &S.smax[slot * NMM + m] : &P.t.mx[(uint64_t)key * NMM + m], v);
  }
}

// fold a slot into its PC-key row (lanes 0-15) and object-key row (lanes 16-31);
// lane field f: 0 n  1 zero  2 eq_pre  3 nosnap  4-8 float flags  9-14 min / max  15 n_type
__device__ __noinline__ void slot_flush(const AnalyzeParams& P, const SlotE* e) {
  const int lane = threadIdx.x & 31, f = lane & 15;
  const uint64_t key = e->key;
  const uint32_t pc = (uint32_t)key & 0xFFFFu, koi = (uint32_t)(key >> 16) & 0xFFFFu;
  const uint32_t meta = (uint32_t)(key >> 32), lg = meta & 3u, kind = (meta >> 2) & 3u;
  const bool st = meta_store(meta);
  const uint64_t n = (uint64_t)e->nwin * 32u;
  uint64_t v = 0;
  uint32_t field = 0;
  bool skip;
  if (f == 0) { v = n; field = st ? F_ST : F_LD; }
  else if (f == 1) { v = e->sum[0]; field = F_ZERO; }
  else if (f == 2) { v = e->sum[1]; field = st ? F_STEQ : F_LDEQ; }
  else if (f == 3) { v = e->nosnap ? n : 0; field = F_NOSNAP; }
  else if (f <= 8) { v = e->sum[f - 2]; field = F_NAN + (uint32_t)(f - 4); }
  else if (f == 15) { v = n; field = F_TYPE0 + type_code(kind, lg); }
  else v = e->mm[f - 9];
  if (f <= 8 || f == 15) {
    skip = v == 0;
  } else {
    const int m = f - 9;                       // 0 raw min 1 raw max 2 ord min 3 ord max 4 trunc min 5 trunc max
    if (m >= 4 && kind < 2u) v = (m & 1) ? 0ull : ~0ull;        // no trunc for integers
    else if (lg < 3u) {
      if (kind == 1u && (m == 2 || m == 3)) {  // sext32(b)^2^31 -> 64-bit ord key
        const int32_t sv = (int32_t)((uint32_t)v ^ 0x80000000u);
        v = (uint64_t)(int64_t)sv ^ (1ull << 63);
      } else if (kind >= 2u && (m == 2 || m == 4) && v == 0xFFFFFFFFull) {
        v = ~0ull;                             // 32-bit min identity (all NaN)
      }
    }
    skip = (m & 1) ? v == 0ull : v == ~0ull;
  }
  if (skip) return;
  if (lane < 16) fold_row(P, pc < P.sp ? (int)pc : -1, pc, f, field, v);
  else fold_row(P, koi < P.so ? (int)(P.sp + koi) : -1, P.n_pcs + koi, f, field, v);
}

// index of key's slot in the warp's cache; a miss evicts round-robin (folding the
// victim) and initialises the slot for key's access type
template <int NS>
__device__ __noinline__ int slot_acquire(const AnalyzeParams& P, WarpCache& wc, SlotE* slots, uint32_t* next,
                                         uint64_t key, int oi, bool nosnap) {
  for (int i = 0; i < NS; ++i)
    if (slots[i].key == key) return i;
  int v = -1;
  for (int i = 0; i < NS; ++i)
    if (slots[i].key == ~0ull) { v = i; break; }
  if (v < 0) {
    v = (int)(*next % NS);
    __syncwarp();
    if ((threadIdx.x & 31) == 0) *next = *next + 1;
    slot_line_flush(P, wc, &slots[v]);
    slot_flush(P, &slots[v]);
  }
  const uint32_t pc = (uint32_t)key & 0xFFFFu, koi = (uint32_t)(key >> 16) & 0xFFFFu;
  const uint32_t meta = (uint32_t)(key >> 32);
  const uint32_t lf = slot_lfail(P, pc, koi);
  const unsigned long long dn = (P.dense_ok && !meta_store(meta) && !nosnap) ? dense_lookup(P, oi, (meta << 16) | pc) : 0ull;
  __syncwarp();
  if ((threadIdx.x & 31) == 0) {
    SlotE& e = slots[v];
    e.key = key;
    e.dense = dn;
    const uint64_t mid = (meta & 3u) < 3u ? 0xFFFFFFFFull : ~0ull;
    for (int m = 0; m < 6; ++m) e.mm[m] = (m & 1) ? 0ull : mid;
    e.nwin = 0;
    e.lfail = lf;
    e.nosnap = nosnap ? 1u : 0u;
    e.cpend = 0;
    for (int i = 0; i < 8; ++i) e.sum[i] = 0;
  }
  __syncwarp();
  return v;
}

struct Rec {
  uint64_t addr, val, pm;
};

// ---- per-warp TMA ring: cp.async.bulk of 2-window stages into shared memory ----
// Each warp streams its own contiguous range of full windows.  The ring state is
// warp-uniform (every lane computes it; lane 0 alone issues the copies), so no
// per-window broadcast is needed.  Records are read once: the copies carry an
// L2 evict-first policy so the stream does not push snapshots and counters out.
#ifndef VE_STAGE_WIN
#define VE_STAGE_WIN 4
#endif
constexpr int STAGE_WIN = VE_STAGE_WIN;
constexpr int NSTAGE = RING / STAGE_WIN;
constexpr uint32_t STAGE_BYTES = STAGE_WIN * WIN_BYTES;

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void ring_issue(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar, uint64_t pol) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          dst),
      "l"(src), "r"(bytes), "r"(bar), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void ring_wait(uint32_t bar, uint32_t phase) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tRW_LOOP:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra RW_LOOP;\n\t}" ::"r"(bar), "r"(phase)
      : "memory");
}
// non-blocking: has the phase with this parity completed?
__device__ __forceinline__ bool mbar_test(uint32_t bar, uint32_t phase) {
  uint32_t r;
  asm volatile(
      "{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(r) : "r"(bar), "r"(phase) : "memory");
  return r != 0u;
}
#ifndef VE_APFAST
#define VE_APFAST 1           // K1 v2: structured windows that are arithmetic progressions held per slot
#endif
#ifndef VE_PF_NEXT
#define VE_PF_NEXT 0
#endif
// fire-and-forget global atomics under a predicate (no branch, no compiler-generated
// warp aggregation around them)
__device__ __forceinline__ void red_or(uint32_t* p, uint32_t v, bool on = true) {
  asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q red.relaxed.gpu.global.or.b32 [%0], %1;\n\t}" ::"l"(p),
               "r"(v), "r"((uint32_t)on)
               : "memory");
}
__device__ __forceinline__ void red_add(uint32_t* p, uint32_t v, bool on = true) {
  asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q red.relaxed.gpu.global.add.u32 [%0], %1;\n\t}" ::"l"(p),
               "r"(v), "r"((uint32_t)on)
               : "memory");
}
// the same, with an L2 evict-last policy (per-element counters that are re-hit)
__device__ __forceinline__ void red_add_keep(uint32_t* p, uint32_t v, bool on = true) {
  asm volatile(
      "{\n\t.reg .pred q;\n\t.reg .b64 pol;\n\tsetp.ne.u32 q, %2, 0;\n\t"
      "createpolicy.fractional.L2::evict_last.b64 pol, 1.0;\n\t"
      "@q red.relaxed.gpu.global.add.L2::cache_hint.u32 [%0], %1, pol;\n\t}" ::"l"(p),
      "r"(v), "r"((uint32_t)on)
      : "memory");
}
// lane predicate `on`: order the warp's generic reads of the stage before the async
// write, arm the stage's mbarrier and start its bulk copy (branch-free)
__device__ __forceinline__ void ring_issue_pred(bool on, uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile(
      "{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %4, 0;\n\t"
      "@q fence.proxy.async.shared::cta;\n\t"
      "@q mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n\t"
      "@q cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%2], [%3], %1, [%0], %5;\n\t}" ::"r"(
          bar),
      "r"(bytes), "r"(dst), "l"(src), "r"((uint32_t)on), "l"(policy_evict_first())
      : "memory");
}

// A warp's ring: NSTAGE (= 2) stages of STAGE_WIN windows.  The state is warp-
// uniform; lane 0 alone issues the copies.  A consumed stage is refilled at the
// start of the following ring_next, once the window read last has been fully
// processed, so the proxy fence before the refill finds no loads outstanding.
// Work split (VE_CLAIM): 2 (default) = static interleave of CHUNK-window chunks (chunk c
// to warp c mod all warps: every warp sees the same mix of the trace, so warps whose
// share holds costly windows -- e.g. Darknet's C rows with random stored values -- no
// longer finish last; measured 2.05 -> 1.82 ms on the cfg2 gemm epoch with 16-window
// chunks vs one contiguous range per warp); 1 = dynamic claims from a global counter;
// 0 = one static contiguous range per warp.
static_assert(NSTAGE * STAGE_WIN == RING, "whole stages");
#ifndef VE_WCLK
#define VE_WCLK 0
#endif
#if VE_WCLK
__shared__ uint32_t s_dbg[K1_WARPS][6];   // dense stages, dense singles, fast windows, hist inserts, dense exits nd, dense exits fit
#define VE_DBG(i, n) do { if ((threadIdx.x & 31) == 0) s_dbg[threadIdx.x >> 5][i] += (n); } while (0)
__shared__ unsigned long long s_dbgc[K1_WARPS][6];   // cycles: run_fast, run_dense, line, slot_acquire, refill, slow
#define VE_TBEG(v) const long long v = clock64()
#define VE_TEND(i, v) do { if ((threadIdx.x & 31) == 0) s_dbgc[threadIdx.x >> 5][i] += clock64() - (v); } while (0)
#else
#define VE_TBEG(v) do { } while (0)
#define VE_TEND(i, v) do { } while (0)
#define VE_DBG(i, n) do { } while (0)
#endif
#ifndef VE_CLAIM
#define VE_CLAIM 2
#endif
#ifndef VE_CHUNK_STAGES
#define VE_CHUNK_STAGES 4
#endif
constexpr uint32_t CHUNK = VE_CHUNK_STAGES * STAGE_WIN;   // windows per claim (whole stages)
struct Ring {
  const ve_record* src;   // next window to issue
  uint32_t iss;           // windows of the current range / chunk not yet issued
  uint32_t left;          // windows issued and not yet consumed
  uint32_t o, o0;         // shared address of this lane's record in the current slot / in slot 0
  uint32_t bar0;          // shared address of stage 0's mbarrier
  uint32_t dst0;          // shared address of stage 0
  uint32_t d, sw, ph;     // stage and window within it of the next read, phase parity of the current pass
  uint32_t pend;          // stage + 1 to refill at the next read, 0 = none
  uint64_t nextc;         // VE_CLAIM == 2: the warp's next static chunk (gw, gw + warps, ...)
  uint32_t cstride;       // warps of the grid (the static interleave's stride)
  uint32_t cu;            // units mode: unit of the chunk being issued
  uint32_t su;            // units mode: unit of the windows in stage d: bits [16d, 16d + 16)
  uint32_t snw;           // windows issued into stage d: bits [4d, 4d + 4) (< STAGE_WIN only for a chunk's end)
};

// claim the next chunk of full windows (all lanes; lane 0 does the atomic).  Guided:
// CHUNK-window chunks cover the first 7/8 of the trace, then chunks of one stage, so
// the warps finish together even where windows differ much in cost.
constexpr uint32_t CHUNK_TAIL = STAGE_WIN;
// MODE: 0 any split (v1: P.claim / P.units at run time), 1 dynamic claims only (v2), 2 units only
// (v2 units mode) -- the v2 instantiations carry no code or registers of the splits they never use
template <int MODE = 0>
__device__ __forceinline__ void ring_claim(const AnalyzeParams& P, Ring& R) {
  uint64_t w0, len;
  if (MODE == 2 || (MODE == 0 && P.units)) {
    // a dynamic claim; its unit by binary search over the chunk prefix (warp-uniform)
    unsigned long long c = 0;
    if ((threadIdx.x & 31) == 0) c = atomicAdd(P.work, 1ull);
    c = __shfl_sync(0xFFFFFFFFu, c, 0);
    if (c >= P.ucb[P.n_units]) { R.iss = 0; return; }
    uint32_t lo = 0, hi = P.n_units;          // last u with ucb[u] <= c
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (P.ucb[mid] <= c) lo = mid; else hi = mid;
    }
    const UnitDesc& U = P.units[lo];
    const uint64_t fw = U.n / 32;
    w0 = (c - P.ucb[lo]) * (uint64_t)P.chunk;
    R.src = U.recs + w0 * 32;
    R.iss = (uint32_t)(fw - w0 < P.chunk ? fw - w0 : P.chunk);
    R.cu = lo;
    return;
  }
  if (MODE == 0 && !P.claim) {
    // static interleave: chunk c goes to warp c mod (all warps); no atomics, and every
    // warp sees the same mix of the trace
    w0 = R.nextc * P.chunk;
    len = P.chunk;
    R.nextc += R.cstride;
  } else {
    // dynamic (K1 v2): chunks from a global counter, the last 1/8 of the trace in one-stage
    // chunks, so warps whose windows cost more (line keys, slot misses) do not set the end
    // of the launch (cfg4: the exit barrier held 9.5% of v2's stall samples under the static split)
    unsigned long long c = 0;
    if ((threadIdx.x & 31) == 0) c = atomicAdd(P.work, 1ull);
    c = __shfl_sync(0xFFFFFFFFu, c, 0);
    const uint64_t nbig = P.nbig;           // (host-computed: a 64-bit division per claim cost ~12
    if (c < nbig) { w0 = (uint64_t)c * P.chunk; len = P.chunk; }   //  instructions per window on cfg4)
    else { w0 = nbig * P.chunk + (uint64_t)(c - nbig) * CHUNK_TAIL; len = CHUNK_TAIL; }
  }
  if (w0 < P.nring) {
    R.src = P.recs + w0 * 32;
    R.iss = (uint32_t)(P.nring - w0 < len ? P.nring - w0 : len);
  } else {
    R.iss = 0;
  }
}

template <int MODE = 0>
__device__ __forceinline__ void ring_issue_stage(const AnalyzeParams& P, Ring& R, uint32_t d) {
  const uint32_t nw = R.iss < (uint32_t)STAGE_WIN ? R.iss : (uint32_t)STAGE_WIN;
  if (nw == 0u) return;
  ring_issue_pred((threadIdx.x & 31) == 0, R.dst0 + d * STAGE_BYTES, R.src, nw * WIN_BYTES, R.bar0 + d * 8u);
  R.su = (R.su & ~(0xFFFFu << (16u * d))) | (R.cu << (16u * d));
  R.snw = (R.snw & ~(0xFu << (4u * d))) | (nw << (4u * d));
  R.src += nw * 32;
  R.iss -= nw;
  R.left += nw;
#if VE_CLAIM
  if (R.iss == 0u) ring_claim<MODE>(P, R);
#endif
}

// take the next window out of the ring (R.left > 0)
__device__ __forceinline__ void ring_next(const AnalyzeParams& P, Ring& R, uint64_t& addr, uint64_t& val,
                                          uint64_t& pm) {
  if (R.pend) {
    __syncwarp();
    ring_issue_stage(P, R, R.pend - 1u);
    R.pend = 0;
  }
  const uint32_t d = R.d;
  ring_wait(R.bar0 + d * 8u, R.ph);
  asm volatile("ld.shared.u64 %0, [%3];\n\tld.shared.u64 %1, [%3+8];\n\tld.shared.u64 %2, [%3+16];"
               : "=l"(addr), "=l"(val), "=l"(pm)
               : "r"(R.o)
               : "memory");
  --R.left;
  R.o += WIN_BYTES;
  if (++R.sw == ((R.snw >> (4u * d)) & 0xFu)) {   // stage consumed (whole, or a chunk's short last stage)
    R.sw = 0;
    R.pend = R.iss ? d + 1u : 0u;
    if (++R.d == (uint32_t)NSTAGE) { R.d = 0; R.ph ^= 1u; }
    R.o = R.o0 + R.d * STAGE_BYTES;
  }
}

// whole-stage access (the dense batch path): refill a pending stage, wait for the
// current stage (the next read is its first window), read window j of it, and
// consume the stage
__device__ __forceinline__ bool ring_stage_full(const Ring& R) { return R.sw == 0u && R.left >= (uint32_t)STAGE_WIN; }
__device__ __forceinline__ void ring_stage_wait(const AnalyzeParams& P, Ring& R) {
  if (R.pend) {
    __syncwarp();
    ring_issue_stage(P, R, R.pend - 1u);
    R.pend = 0;
  }
  ring_wait(R.bar0 + R.d * 8u, R.ph);
}
__device__ __forceinline__ void ring_stage_read(const Ring& R, uint32_t j, uint64_t& addr, uint64_t& val,
                                                uint64_t& pm) {
  asm volatile("ld.shared.u64 %0, [%3];\n\tld.shared.u64 %1, [%3+8];\n\tld.shared.u64 %2, [%3+16];"
               : "=l"(addr), "=l"(val), "=l"(pm)
               : "r"(R.o + j * WIN_BYTES)
               : "memory");
}
__device__ __forceinline__ void ring_stage_consume(Ring& R) {
  R.left -= STAGE_WIN;
  R.o += STAGE_WIN * WIN_BYTES;
  R.pend = R.iss ? R.d + 1u : 0u;
  if (++R.d == (uint32_t)NSTAGE) { R.d = 0; R.o = R.o0; R.ph ^= 1u; }
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

// ---- slow path: any window (mixed keys, invalid / shared / unmapped / straddling
// records, tails).  Returns this lane's (invalid | unmapped << 16) counts.
__device__ __noinline__ uint32_t slow_window(const AnalyzeParams& P, WarpCache& wc, uint64_t addr,
                                             uint64_t val, uint64_t pm, bool inrange) {
  const Smem S = smem_of(P);
  const int lane = threadIdx.x & 31;
  __syncwarp();
  const uint32_t pc = (uint32_t)pm, meta = (uint32_t)(pm >> 32);
  // S1 decode + validate
  const bool valid = inrange && rec_valid(addr, val, pc, meta, P.n_pcs);
  const unsigned vmask = __ballot_sync(0xFFFFFFFFu, valid);
  const uint32_t inv = (inrange && !valid) ? 1u : 0u;
  if (vmask == 0) return inv;
  const uint32_t lg = meta & 3u, kind = (meta >> 2) & 3u;
  const bool st = meta_store(meta), sh = meta_shared(meta);

  // S2 address -> object (binary search)
  const bool need = valid && !sh;
  const int oi = need ? find_object(P, addr) : -1;
  const bool mapped = oi >= 0;
  uint64_t ob = 0, oe = 0, bmoff = 0, opre = 0;
  uint32_t oid = 0, ew_lg = 0;
  if (mapped) {
    ob = P.objc ? S.sob[oi] : P.o.base[oi];
    oe = P.objc ? S.soe[oi] : P.o.end[oi];
    bmoff = P.o.bmoff[oi];
    opre = P.o.pre[oi];
    oid = P.o.id[oi];
    const uint32_t ew = P.o.ew[oi];
    ew_lg = (ew == 1) ? 0 : (ew == 2) ? 1 : (ew == 4) ? 2 : 3;
  }
  const uint32_t unm = (need && !mapped) ? 1u : 0u;

  // S3 snapshot gather + eq_pre
  const uint64_t off = mapped ? addr - ob : 0ull;
  const bool inside = mapped && addr + (1u << lg) <= oe;
  const bool eqdef = inside && opre != 0ull;
  const uint64_t pv = eqdef ? load_pre(opre + off, lg) : 0ull;
  const uint32_t koi = sh ? P.n_obj : (mapped ? oid : KO_NONE);

  // W element bitmap (C10) and L start-element bitmap (C3)
  const uint64_t e0 = off >> ew_lg, e1 = (off + (1u << lg) - 1) >> ew_lg;
  const uint64_t w0 = bmoff + (e0 >> 5), w1 = bmoff + (e1 >> 5);
  {
    const bool wpart = inside && st;
    if (__any_sync(0xFFFFFFFFu, wpart)) {
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
  const bool eq = eqdef && pv == val;
  const bool lpart = inside && !st && eq;
  if (__any_sync(0xFFFFFFFFu, lpart)) bitmap_or(P.t.L, lpart, w0, 1u << (e0 & 31));

  // per-key groups
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
    apply_group(P, gm, pslot, pc, f, gp);
    leadp = lane == __ffs(gm) - 1;
  }
  const bool opart = valid && koi != KO_NONE;
  const unsigned omask = __ballot_sync(0xFFFFFFFFu, opart);
  const int oslot = koi < P.so ? (int)(P.sp + koi) : -1;
  if (opart) {
    const unsigned gm = __match_any_sync(omask, koi);
    apply_group(P, gm, oslot, P.n_pcs + koi, f, go);
    leado = lane == __ffs(gm) - 1;
  }
  merge_lines(P, wc, leadp, pc, pslot, gp);
  merge_lines(P, wc, leado, P.n_pcs + koi, oslot, go);
  if (valid) {
    const uint32_t tag = (pc << 16) | (koi & 0xFFFFu);
    const unsigned tg = __match_any_sync(vmask, tag);
    const unsigned vg = __match_any_sync(tg, val);
    if (lane == __ffs(vg) - 1) hist_insert(P, tag, val, __popc(vg));
  }
  __syncwarp();
  return inv | (unm << 16);
}

// ---- fast path ---------------------------------------------------------------
// A fast window: all 32 lanes valid, one (pc, access type), global space, every
// access aligned inside the warp's cached object whose element width equals the
// access width.  Its type is a compile-time constant of run_fast below.

// warp-uniform cache of the last object windows mapped to
struct ObjCache {
  uint64_t base, lim;      // offsets [0, lim] hold a whole element
  uint64_t bmoff, pre;
  int oi;
  uint32_t id, fastlg;     // fastlg: log2 element width, 0xFF = no fast windows
};

__device__ __noinline__ ObjCache obj_refill(const AnalyzeParams& P, uint64_t a) {
  const Smem S = smem_of(P);
  ObjCache oc;
  oc.oi = find_object(P, a);
  oc.base = 0; oc.lim = 0; oc.bmoff = 0; oc.pre = 0; oc.id = 0; oc.fastlg = 0xFFu;
  if (oc.oi >= 0) {
    const int i = oc.oi;
    oc.base = P.objc ? S.sob[i] : P.o.base[i];
    const uint64_t e = P.objc ? S.soe[i] : P.o.end[i];
    oc.bmoff = P.o.bmoff[i];
    oc.pre = P.o.pre[i];
    oc.id = P.o.id[i];
    const uint32_t ew = P.o.ew[i];
    const uint32_t lg = (ew == 1) ? 0 : (ew == 2) ? 1 : (ew == 4) ? 2 : 3;
    // pre must be aligned for element-wide gathers
    if (e - oc.base >= ew && (oc.pre & (ew - 1)) == 0) {
      oc.lim = e - oc.base - ew;
      oc.fastlg = lg;
    }
  }
  return oc;
}

constexpr uint32_t VALID_KL = 0x2EFFu;  // valid (kind << 2 | log2 w) pairs of include/ve.h
// a window whose lanes all carry (pc0, meta0): global space, valid type, pc in range
__device__ __forceinline__ bool meta_fast(uint32_t meta0, uint32_t pc0, uint32_t n_pcs) {
  return (meta0 >> 5) == 0u && ((VALID_KL >> (meta0 & 15u)) & 1u) && pc0 < n_pcs;
}

__device__ const unsigned long long ve_zero_word = 0ull;

// The pre-snapshot gather of a window is prefetched into L1 when the window is read
// ahead (VE_PREFETCH) instead of being loaded into a register there: a register in
// flight would stall the register rotation of the read-ahead pipeline.
#ifndef VE_PREFETCH
#define VE_PREFETCH 0
#endif
__device__ __forceinline__ void prefetch_l1(uint64_t p) { asm volatile("prefetch.global.L1 [%0];" ::"l"(p)); }
// L2 policy of the data K1 re-reads (snapshot gathers, per-element counters): keep it
// over the record stream (evict-first) and the histogram
#ifndef VE_KEEP_HINT
#define VE_KEEP_HINT 1
#endif
__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
template <int LG>
__device__ __forceinline__ uint64_t ld_pre(uint64_t p) {
#if VE_KEEP_HINT
  const uint64_t pol = policy_evict_last();
  if (LG == 0) { uint16_t v; asm("ld.global.nc.L2::cache_hint.u8 %0, [%1], %2;" : "=h"(v) : "l"(p), "l"(pol)); return v & 0xFFu; }
  if (LG == 1) { uint16_t v; asm("ld.global.nc.L2::cache_hint.u16 %0, [%1], %2;" : "=h"(v) : "l"(p), "l"(pol)); return v; }
  if (LG == 2) { uint32_t v; asm("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol)); return v; }
  uint64_t v;
  asm("ld.global.nc.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol));
  return v;
#else
  if (LG == 0) return __ldg((const unsigned char*)p);
  if (LG == 1) return __ldg((const unsigned short*)p);
  if (LG == 2) return __ldg((const unsigned int*)p);
  return __ldg((const unsigned long long*)p);
#endif
}

// C5 float flags of a <= 32-bit float (same definition as float_flags, 32-bit
// arithmetic, branch-free)
template <int KIND, int LG>
__device__ __forceinline__ uint32_t fflags32(uint32_t b) {
  constexpr int EB = KIND == 3 ? 8 : (LG == 1 ? 5 : 8);
  constexpr int MB = KIND == 3 ? 7 : (LG == 1 ? 10 : 23);
  constexpr int NB = 8 << LG;
  constexpr uint32_t EMAX = (1u << EB) - 1u;
  constexpr int BIAS = (1 << (EB - 1)) - 1;
  const uint32_t E = (b >> MB) & EMAX, M = b & ((1u << MB) - 1u);
  const bool sign = (b >> (NB - 1)) & 1u;
  const uint32_t sig = E ? (M | (1u << MB)) : M;
  const int ex = (E ? (int)E : 1) - BIAS - MB;
  const int low = ex + __ffs((int)sig) - 1;
  const int top = ex + 31 - __clz((int)sig);
  uint32_t f = (top >= 63 || low < 0) ? 2u : 0u;
  if (!(top <= 15 && low >= max(top - 10, -24))) f |= 4u;
  if (!(top <= 127 && low >= max(top - 7, -133))) f |= 8u;
  f = sig == 0u ? (sign ? 2u : 0u) : f;                 // +-0.0 (-0.0 is nonint)
  return E == EMAX ? (M ? 15u : 2u) : f;                // NaN fails everything, +-Inf nonint only
}

// one window's OR into an element bitmap; lanes' words are usually one or two
// consecutive words from lane 0's
__device__ __forceinline__ void bitmap_or_win(uint32_t* bm, bool part, uint64_t word, uint32_t bit) {
  const int lane = threadIdx.x & 31;
  const uint64_t w0 = shfl64(0xFFFFFFFFu, word, 0);
  const uint64_t d = word - w0;
  if (__all_sync(0xFFFFFFFFu, !part || d <= 1ull)) {
    const uint32_t b0 = __reduce_or_sync(0xFFFFFFFFu, (part && d == 0ull) ? bit : 0u);
    const uint32_t b1 = __reduce_or_sync(0xFFFFFFFFu, (part && d == 1ull) ? bit : 0u);
    const uint32_t bv = lane ? b1 : b0;
    red_or(&bm[w0 + lane], bv, lane < 2 && bv != 0u);
  } else {
    bitmap_or(bm, part, word, bit);
  }
}

// C8 point of a value: y = the integer the bits denote (uint, sint, or an integral
// float); pfail = a float that is not a finite integer below 2^63 (no point)
__device__ __forceinline__ __int128 line_y(uint64_t val, uint32_t kind, uint32_t lg, bool& pfail) {
  int64_t ival = 0;
  const uint32_t ff = kind >= 2u ? float_flags(val, kind, lg, ival) : 0u;
  pfail = kind >= 2u && (ff & 2u);
  if (kind == 0u) return (__int128)val;
  if (kind == 1u) {
    const uint32_t sh64 = 64u - (8u << lg);
    return (__int128)((int64_t)(val << sh64) >> sh64);
  }
  return (__int128)ival;
}

// merge a window's line state into the keys of its slot not yet FAIL (lane 0);
// returns the updated FAIL bits (warp-uniform)
__device__ __forceinline__ uint32_t line_apply(const AnalyzeParams& P, WarpCache& wc, const LinePts& g,
                                               uint32_t pc0, uint32_t koi0, uint32_t lf) {
  const int lane = threadIdx.x & 31;
  const int ps = pc0 < P.sp ? (int)pc0 : -1;
  const int os = koi0 < P.so ? (int)(P.sp + koi0) : -1;
  if (lane == 0) {
    if (!(lf & 1u) && wcache_merge(P, wc, pc0, ps, g) == VE_LINE_FAIL) lf |= 1u;
    if (!(lf & 2u) && wcache_merge(P, wc, P.n_pcs + koi0, os, g) == VE_LINE_FAIL) lf |= 2u;
  }
  __syncwarp();
  return __shfl_sync(0xFFFFFFFFu, lf, 0);
}

// C8 for a fast window: one line state over its 32 points
__device__ __noinline__ uint32_t fast_line(const AnalyzeParams& P, WarpCache& wc, uint64_t addr,
                                           uint64_t val, uint32_t meta0, uint32_t pc0, uint32_t koi0, uint32_t lf) {
  Facts f;
  f.addr = addr;
  f.y = line_y(val, (meta0 >> 2) & 3u, meta0 & 3u, f.pfail);
  LinePts g;
  group_line(0xFFFFFFFFu, f, g);
  return line_apply(P, wc, g, pc0, koi0, lf);
}

// C8 for a run of windows that all carry the one value cy: its points (x, y(cy))
// span [xmin, xmax], so the run is POINT or a slope-0 LINE between its extremes
__device__ __noinline__ uint32_t const_line(const AnalyzeParams& P, WarpCache& wc, uint64_t xmin, uint64_t xmax,
                                            uint64_t cy, uint32_t meta0, uint32_t pc0, uint32_t koi0, uint32_t lf) {
  bool pfail;
  const __int128 y = line_y(cy, (meta0 >> 2) & 3u, meta0 & 3u, pfail);
  LinePts g;
  g.state = pfail ? VE_LINE_FAIL : (xmin == xmax ? VE_LINE_POINT : VE_LINE_LINE);
  g.px = xmin; g.qx = xmax;
  g.py = g.qy = y;
  return line_apply(P, wc, g, pc0, koi0, lf);
}

// Dense batch path for a key whose loads are counted per element (C3 / S8 dense
// counters): such a window's statistics are its record count, its eq_pre count and
// one counter increment per element -- every value statistic is taken from the
// pre snapshot at report time (k_dense_flush).  Whole ring stages are consumed at
// once (one barrier wait, STAGE_WIN gathers in flight together).  Stops at a key
// change (returns true, window left in addr / val / pm), at the end of the ring
// (false), or at a window that is not entirely dense: then nd is set and that
// window, unprocessed, is left in addr / val / pm for run_fast.
template <int LG>
__device__ __forceinline__ bool run_dense(const AnalyzeParams& P, const ObjCache& oc, SlotE* se, Ring& R,
                                          uint64_t& addr, uint64_t& val, uint64_t& pm, bool& nd) {
  using MT = typename std::conditional<(LG < 3), uint32_t, uint64_t>::type;
  constexpr uint32_t W = 1u << LG;
  const unsigned FULL = 0xFFFFFFFFu;
  const uint64_t pm0 = shfl64(FULL, pm, 0);
  uint32_t* const dn = reinterpret_cast<uint32_t*>(se->dense);
  uint32_t ndw = 0;                                  // dense windows processed
  auto fits = [&](uint64_t a, uint64_t v, uint64_t p, uint64_t& o) -> bool {
    o = a - oc.base;
    bool ok = o <= oc.lim && (o & (W - 1)) == 0 && p == pm0;
    if constexpr (LG < 3) ok = ok && (v >> (8 * W)) == 0ull;
    return ok;
  };
  auto done = [&]() {
    __syncwarp();
    if ((threadIdx.x & 31) == 0) { se->nwin += ndw; se->sum[1] += ndw * 32u; }
    __syncwarp();
  };
  nd = false;
  // the current window (already read from the ring)
  {
    const uint64_t o = addr - oc.base;
    const MT pv = (MT)ld_pre<LG>(oc.pre + o);
    if (!__all_sync(FULL, pv == (MT)val)) { nd = true; done(); return true; }
    red_add_keep(dn + (o >> LG), 1u, true);
    ++ndw;
  }
  while (true) {
    if (ring_stage_full(R)) {
      ring_stage_wait(P, R);
      uint64_t a[STAGE_WIN], v[STAGE_WIN], p[STAGE_WIN], o[STAGE_WIN];
      bool ok = true;
#pragma unroll
      for (int j = 0; j < STAGE_WIN; ++j) {
        ring_stage_read(R, (uint32_t)j, a[j], v[j], p[j]);
        ok = ok && fits(a[j], v[j], p[j], o[j]);
      }
#if VE_PF_NEXT
      // the following stage, if already landed: pull its pre elements into L1 now, so
      // its gathers hit L1 instead of waiting on L2 one stage later
      if (NSTAGE >= 3 && R.left >= 2u * STAGE_WIN) {
        const uint32_t dn = R.d + 1u == (uint32_t)NSTAGE ? 0u : R.d + 1u;
        const uint32_t phn = R.d + 1u == (uint32_t)NSTAGE ? (R.ph ^ 1u) : R.ph;
        if (mbar_test(R.bar0 + dn * 8u, phn)) {
#pragma unroll
          for (int j = 0; j < STAGE_WIN; ++j) {
            uint64_t an;
            asm volatile("ld.shared.u64 %0, [%1];" : "=l"(an) : "r"(R.o0 + dn * STAGE_BYTES + (uint32_t)j * WIN_BYTES)
                         : "memory");
            const uint64_t on = an - oc.base;
            if (on <= oc.lim) prefetch_l1(oc.pre + on);
          }
        }
      }
#endif
      if (__all_sync(FULL, ok)) {
        MT pv[STAGE_WIN];
#pragma unroll
        for (int j = 0; j < STAGE_WIN; ++j) pv[j] = (MT)ld_pre<LG>(oc.pre + o[j]);
        bool eq = true;
#pragma unroll
        for (int j = 0; j < STAGE_WIN; ++j) eq = eq && pv[j] == (MT)v[j];
        if (__all_sync(FULL, eq)) {
#pragma unroll
          for (int j = 0; j < STAGE_WIN; ++j) red_add_keep(dn + (o[j] >> LG), 1u, true);
          ndw += STAGE_WIN;
          VE_DBG(0, 1);
          ring_stage_consume(R);
          continue;
        }
      }
      // not a whole dense stage of this key: go on window by window
    }
    if (R.left == 0u) { done(); return false; }
    ring_next(P, R, addr, val, pm);
    uint64_t o;
    if (!__all_sync(FULL, fits(addr, val, pm, o))) { VE_DBG(5, 1); done(); return true; }
    const MT pv = (MT)ld_pre<LG>(oc.pre + o);
    if (!__all_sync(FULL, pv == (MT)val)) { VE_DBG(4, 1); nd = true; done(); return true; }
    red_add_keep(dn + (o >> LG), 1u, true);
    VE_DBG(1, 1);
    ++ndw;
  }
}

// Multi-key dense path (VE_MULTI_DENSE): like run_dense, but a following window may
// belong to ANY key of the warp's slot cache that counts its loads densely and has no
// live line state (loads of one object by several PCs interleaved window by window:
// stencil neighbours, Darknet's C rows).  Whole stages are taken up to the first
// window that does not qualify, their STAGE_WIN gathers in flight together; each
// window's record count and eq count go to its own slot.  Stops (returns true, window
// left in addr / val / pm for the main loop) at a window that does not qualify; nd is
// set only when the entry window itself is not entirely dense.
#ifndef VE_MULTI_DENSE
#define VE_MULTI_DENSE 1
#endif
#ifndef VE_MULTI_MIN_PCS
#define VE_MULTI_MIN_PCS 8
#endif
template <int LG>
__device__ __forceinline__ bool run_dense_multi(const AnalyzeParams& P, const ObjCache& oc, SlotE* slots, SlotE* se,
                                                Ring& R, uint64_t& addr, uint64_t& val, uint64_t& pm, bool& nd) {
  using MT = typename std::conditional<(LG < 3), uint32_t, uint64_t>::type;
  constexpr uint32_t W = 1u << LG;
  const unsigned FULL = 0xFFFFFFFFu;
  const int lane = threadIdx.x & 31;
  uint64_t lastp = shfl64(FULL, pm, 0);      // the key seen last, its slot, and the windows
  SlotE* lasts = se;                          // counted for it but not yet added to the slot
  uint32_t nlast = 0;
  auto settle = [&]() {
    __syncwarp();
    if (lane == 0 && nlast) { lasts->nwin += nlast; lasts->sum[1] += nlast * 32u; }
    __syncwarp();
    nlast = 0;
  };
  // the slot of a window (warp-uniform pm) if it is a dense load key of this object
  // without live line state, else nullptr; it becomes the "last" slot
  auto slot_of = [&](uint64_t p) -> SlotE* {
    if (__all_sync(FULL, p == lastp)) return lasts;
    const uint64_t p0 = shfl64(FULL, p, 0);
    if (!__all_sync(FULL, p == p0)) return nullptr;
    const uint32_t meta = (uint32_t)(p0 >> 32), pc = (uint32_t)p0;
    if ((meta & 3u) != (uint32_t)LG || meta_store(meta) || meta_shared(meta)) return nullptr;
    const uint64_t key = ((uint64_t)meta << 32) | ((uint64_t)oc.id << 16) | pc;
#pragma unroll
    for (int i = 0; i < NSLOT; ++i)
      if (slots[i].key == key) {
        if (slots[i].dense == 0ull || slots[i].lfail != 3u) return nullptr;
        settle();
        lastp = p0;
        lasts = &slots[i];
        return lasts;
      }
    return nullptr;
  };
  auto lane_fits = [&](uint64_t a, uint64_t v, uint64_t& o) -> bool {
    o = a - oc.base;
    bool ok = o <= oc.lim && (o & (W - 1)) == 0;
    if constexpr (LG < 3) ok = ok && (v >> (8 * W)) == 0ull;
    return ok;
  };
  nd = false;
  {   // the entry window (its slot is se)
    const uint64_t o = addr - oc.base;
    const MT pv = (MT)ld_pre<LG>(oc.pre + o);
    if (!__all_sync(FULL, pv == (MT)val)) { nd = true; return true; }
    red_add_keep(reinterpret_cast<uint32_t*>(se->dense) + (o >> LG), 1u, true);
    ++nlast;
  }
  while (true) {
    if (ring_stage_full(R)) {
      ring_stage_wait(P, R);
      uint64_t a[STAGE_WIN], v[STAGE_WIN], p[STAGE_WIN], o[STAGE_WIN];
      bool same = true;
#pragma unroll
      for (int j = 0; j < STAGE_WIN; ++j) {
        ring_stage_read(R, (uint32_t)j, a[j], v[j], p[j]);
        same = same && p[j] == lastp && lane_fits(a[j], v[j], o[j]);
      }
      if (__all_sync(FULL, same)) {           // a whole stage of the last key: as run_dense
        MT pv[STAGE_WIN];
#pragma unroll
        for (int j = 0; j < STAGE_WIN; ++j) pv[j] = (MT)ld_pre<LG>(oc.pre + o[j]);
        bool eq = true;
#pragma unroll
        for (int j = 0; j < STAGE_WIN; ++j) eq = eq && pv[j] == (MT)v[j];
        if (__all_sync(FULL, eq)) {
          uint32_t* const dn = reinterpret_cast<uint32_t*>(lasts->dense);
#pragma unroll
          for (int j = 0; j < STAGE_WIN; ++j) red_add_keep(dn + (o[j] >> LG), 1u, true);
          nlast += STAGE_WIN;
          VE_DBG(0, 1);
          ring_stage_consume(R);
          continue;
        }
      } else {                                 // several keys: each window's own slot
        SlotE* es[STAGE_WIN];
        bool ok = true;
#pragma unroll
        for (int j = 0; j < STAGE_WIN; ++j) {
          es[j] = ok ? slot_of(p[j]) : nullptr;
          ok = ok && es[j] != nullptr && __all_sync(FULL, lane_fits(a[j], v[j], o[j]));
        }
        if (ok) {
          MT pv[STAGE_WIN];
#pragma unroll
          for (int j = 0; j < STAGE_WIN; ++j) pv[j] = (MT)ld_pre<LG>(oc.pre + o[j]);
          bool eq = true;
#pragma unroll
          for (int j = 0; j < STAGE_WIN; ++j) eq = eq && pv[j] == (MT)v[j];
          if (__all_sync(FULL, eq)) {
            settle();
#pragma unroll
            for (int j = 0; j < STAGE_WIN; ++j) {
              red_add_keep(reinterpret_cast<uint32_t*>(es[j]->dense) + (o[j] >> LG), 1u, true);
              if (lane == 0) { es[j]->nwin += 1u; es[j]->sum[1] += 32u; }
            }
            __syncwarp();
            VE_DBG(0, 1);
            ring_stage_consume(R);
            continue;
          }
        }
      }
      // not a whole stage of qualifying windows: go on window by window
    }
    if (R.left == 0u) { settle(); return false; }
    ring_next(P, R, addr, val, pm);
    SlotE* e = slot_of(pm);
    uint64_t o;
    if (e == nullptr || !__all_sync(FULL, lane_fits(addr, val, o))) { VE_DBG(5, 1); settle(); return true; }
    const MT pv = (MT)ld_pre<LG>(oc.pre + o);
    if (!__all_sync(FULL, pv == (MT)val)) { VE_DBG(4, 1); settle(); return true; }   // re-dispatched by the main loop
    red_add_keep(reinterpret_cast<uint32_t*>(e->dense) + (o >> LG), 1u, true);
    ++nlast;
    VE_DBG(1, 1);
  }
}

// Consume fast windows of access type (KIND, LG) from the ring, starting with the
// current one (addr, val, pm; known fast).  Returns true when it stopped at a
// window it has not consumed (left in addr, val, pm), false when the ring is empty.
//
// Every lane folds its own record of each window into per-lane accumulators of the
// active slot (counts in 16-bit fields, min / max in MT); the warp reduces them
// only when the slot is switched out, so a window costs no warp reductions.
template <typename MT>
__device__ __forceinline__ MT wmin(MT v) {
  if constexpr (sizeof(MT) == 4) return __reduce_min_sync(0xFFFFFFFFu, v);
  else return redmin64(0xFFFFFFFFu, v);
}
template <typename MT>
__device__ __forceinline__ MT wmax(MT v) {
  if constexpr (sizeof(MT) == 4) return __reduce_max_sync(0xFFFFFFFFu, v);
  else return redmax64(0xFFFFFFFFu, v);
}
__device__ __forceinline__ uint32_t wsum16(uint32_t v, int hi) {
  return __reduce_add_sync(0xFFFFFFFFu, hi ? (v >> 16) : (v & 0xFFFFu));
}

template <int KIND, int LG>
__device__ __forceinline__ bool run_fast(const AnalyzeParams& P, const ObjCache& oc, SlotE* se, bool one, bool cmode,
                                         uint64_t cy, uint64_t& xmin, uint64_t& xmax, Ring& R, uint64_t& addr,
                                         uint64_t& val, uint64_t& pm) {
  using MT = typename std::conditional<(LG < 3), uint32_t, uint64_t>::type;   // min / max accumulators
  constexpr bool ISF = KIND >= 2;
  constexpr uint32_t W = 1u << LG;
  constexpr int MB = KIND == 3 ? 7 : (LG == 1 ? 10 : LG == 2 ? 23 : 52);
  constexpr MT MID = (MT)~0ull;                                                 // min identity
  const unsigned FULL = 0xFFFFFFFFu;
  const int lane = threadIdx.x & 31;
  const MT tmask = (MT)(P.mant_bits >= (uint32_t)MB ? ~0ull : ~((1ull << (MB - P.mant_bits)) - 1ull));
  const bool eqdef = oc.pre != 0ull;
  const uint64_t pm0 = shfl64(FULL, pm, 0);
  const uint32_t pc0 = (uint32_t)pm0, meta0 = (uint32_t)(pm0 >> 32);
  const bool st = meta_store(meta0);
  const unsigned long long dn = se->dense;
  const uint32_t tag = (pc0 << 16) | (oc.id & 0xFFFFu);
  // per-lane accumulators
  uint32_t nwin = 0;
  uint32_t cz = 0, cf0 = 0, cf1 = 0, cf2 = 0;   // zero | eq_pre<<16, nan | nonint<<16, not_f16 | not_bf16<<16, not_f32
  MT m0 = MID, m1 = 0, m2 = MID, m3 = 0, m4 = MID, m5 = 0;
  auto save = [&]() {   // fold the accumulators into the slot and reset them
    const uint32_t s0 = wsum16(cz, 0), s1 = wsum16(cz, 1);
    uint32_t s2 = 0, s3 = 0, s4 = 0, s5 = 0, s6 = 0;
    if constexpr (ISF) {
      s2 = wsum16(cf0, 0); s3 = wsum16(cf0, 1); s4 = wsum16(cf1, 0); s5 = wsum16(cf1, 1);
      if constexpr (LG == 3) s6 = __reduce_add_sync(FULL, cf2);
    }
    const MT r0 = wmin(m0), r1 = wmax(m1);
    MT r2 = r0, r3 = r1, r4 = MID, r5 = 0;
    if constexpr (KIND != 0) { r2 = wmin(m2); r3 = wmax(m3); }
    if constexpr (ISF) { r4 = wmin(m4); r5 = wmax(m5); }
    __syncwarp();
    if (lane == 0) {
      SlotE& e = *se;
      e.nwin += nwin;
      e.sum[0] += s0; e.sum[1] += s1; e.sum[2] += s2; e.sum[3] += s3; e.sum[4] += s4; e.sum[5] += s5; e.sum[6] += s6;
      e.mm[0] = min(e.mm[0], (uint64_t)r0); e.mm[1] = max(e.mm[1], (uint64_t)r1);
      e.mm[2] = min(e.mm[2], (uint64_t)r2); e.mm[3] = max(e.mm[3], (uint64_t)r3);
      e.mm[4] = min(e.mm[4], (uint64_t)r4); e.mm[5] = max(e.mm[5], (uint64_t)r5);
    }
    __syncwarp();
    cz = cf0 = cf1 = cf2 = 0;
    m0 = MID; m1 = 0; m2 = MID; m3 = 0; m4 = MID; m5 = 0;
    nwin = 0;
  };
  // S3 gather of a window's pre-snapshot elements (a zero word when the object has
  // no snapshot).  Software-pipelined: the next window is read from the ring and its
  // gather issued before the current window is processed.
  auto gather = [&](uint64_t o) -> MT { return (MT)ld_pre<LG>(eqdef ? oc.pre + o : (uint64_t)&ve_zero_word); };
  // window i+1 read ahead: a continuing window's record is in (a1, v1) with its
  // gather pv1 in flight; a window that does not continue is left in (a1, v1, p1)
  auto peek = [&](uint64_t& a, uint64_t& v, uint64_t& p, uint64_t& o, MT& g, bool& c) {
    ring_next(P, R, a, v, p);
    o = a - oc.base;
    bool ok = o <= oc.lim && (o & (W - 1)) == 0;
    if constexpr (LG < 3) ok = ok && (v >> (8 * W)) == 0ull;
    c = __all_sync(FULL, ok && p == pm0 && (!cmode || v == cy));
#if VE_PREFETCH
    if (c && eqdef) prefetch_l1(oc.pre + o);
#else
    if (c) g = gather(o);
#endif
  };
  VE_TBEG(tf0);
  uint64_t off = addr - oc.base;
  MT pv = gather(off);
  uint64_t a1 = 0, v1 = 0, p1 = 0, off1 = 0;
  MT pv1 = 0;
  bool more1 = !one && R.left != 0u, cont1 = false;
  if (more1) peek(a1, v1, p1, off1, pv1, cont1);
#if VE_WCLK
  { volatile MT sink = pv; (void)sink; }
#endif
  VE_TEND(1, tf0);
  while (true) {
    VE_TBEG(tw0);
    // window i+2, two windows ahead of the one processed now
    uint64_t a2 = 0, v2 = 0, p2 = 0, off2 = 0;
    MT pv2 = 0;
    const bool more2 = cont1 && R.left != 0u;
    bool cont2 = false;
    if (more2) peek(a2, v2, p2, off2, pv2, cont2);

#if VE_PREFETCH
    pv = gather(off);                     // prefetched into L1 two windows ago
#endif
#ifndef VE_EXP
#define VE_EXP 0   // timing experiments only (wrong results): 1 stream only, 2 + gather/eq, 3 + dense counts
#endif
#if VE_EXP == 1
    cz += 1u;
#elif VE_EXP == 2
    cz += ((MT)val == pv) ? 1u : 0u;
#elif VE_EXP == 3
    {
      const bool eq = (MT)val == pv;
      cz += eq ? 1u : 0u;
      red_add_keep(reinterpret_cast<uint32_t*>(dn) + (off >> LG), 1u, eq && dn != 0ull);
    }
#else
    // element, written bitmap
    const uint64_t e = off >> LG;
    const uint64_t word = oc.bmoff + (e >> 5);
    const uint32_t bit = 1u << ((uint32_t)e & 31u);
    if (st) bitmap_or_win(P.t.W, true, word, bit);
    if (cmode) {                          // C8 of a constant run: the extreme addresses
      xmin = addr < xmin ? addr : xmin;
      xmax = addr > xmax ? addr : xmax;
    }

    const MT b = (MT)val;
    const bool eq = eqdef && pv == b;
    const bool dl = dn != 0ull && eq;
    if (dn != 0ull && __all_sync(FULL, dl)) {
      // a dense window: every load reads its element's unchanged pre value, so its
      // value statistics (C1 zero, C4-C7, C9) are those of the pre snapshot at the
      // counted elements, taken once per element at report time (k_dense_flush)
      cz += 0x10000u;
      red_add_keep(reinterpret_cast<uint32_t*>(dn) + e, 1u, true);
    } else {
    // C1/C4-C7: per-lane folds of the records not counted per element
    const bool fo = !dl;
    m0 = min(m0, fo ? b : MID);
    m1 = max(m1, fo ? b : (MT)0);
    if constexpr (KIND == 1) {
      MT k;
      if constexpr (LG < 3) {               // sext32(b) ^ 2^31 (order-isomorphic to the 64-bit key)
        constexpr uint32_t sh = 32 - (8 << LG);
        k = (uint32_t)(((int32_t)(b << sh)) >> sh) ^ 0x80000000u;
      } else {
        k = b ^ (1ull << 63);
      }
      m2 = min(m2, fo ? k : MID);
      m3 = max(m3, fo ? k : (MT)0);
    } else if constexpr (ISF) {
      uint32_t ff;
      if constexpr (KIND == 2 && LG == 2) ff = fflags_f32((uint32_t)b);
      else if constexpr (LG < 3) ff = fflags32<KIND, LG>((uint32_t)b);
      else { int64_t ival; ff = float_flags(val, 2u, 3u, ival); }
      ff = fo ? ff : 1u;                    // counted elements: as NaN below, then masked out
      const bool okv = !(ff & 1u);          // NaNs excluded from ord / trunc
      constexpr MT SIGN = (MT)1 << ((8 << LG) - 1);
      constexpr MT MASK = (MT)((8 << LG) == 64 ? ~0ull : ((1ull << (8 << LG)) - 1ull));
      const MT k = (b & SIGN) ? (~b & MASK) : (b | SIGN);
      const MT t = b & tmask;
      m2 = min(m2, okv ? k : MID);
      m3 = max(m3, okv ? k : (MT)0);
      m4 = min(m4, okv ? t : MID);
      m5 = max(m5, okv ? t : (MT)0);
      ff = fo ? ff : 0u;
      cf0 += (ff & 1u) | ((ff & 2u) << 15);
      cf1 += ((ff >> 2) & 1u) | ((ff & 8u) << 13);
      if constexpr (LG == 3) cf2 += (ff >> 4) & 1u;
    }
    cz += (fo && b == (MT)0 ? 1u : 0u) + (eq ? 0x10000u : 0u);

    // C3 loaded elements; loads counted per element below get their bits from the
    // dense counters at report time
    if (!st && dn == 0ull) {
      if (__any_sync(FULL, eq)) bitmap_or_win(P.t.L, eq, word, bit);
    }

    // S8: exact histogram.  A load that reads an unchanged element carries that
    // element's pre value, so it is counted per element (mapped to its value at
    // report time); every other record is inserted per distinct value.
    red_add_keep(reinterpret_cast<uint32_t*>(dn) + e, 1u, dl);
    const unsigned hm = __ballot_sync(FULL, !dl);
    VE_TBEG(th0);
    if (hm) {
      const int l = __ffs(hm) - 1;
      const uint64_t v0 = (LG < 3) ? (uint64_t)__shfl_sync(FULL, (uint32_t)val, l) : shfl64(FULL, val, l);
      if (__all_sync(FULL, dl || val == v0)) {
        VE_DBG(3, 1);
        if (lane == l) hist_insert(P, tag, val, __popc(hm));
      } else if (!dl) {
        const unsigned vg = (LG < 3) ? __match_any_sync(hm, (uint32_t)val) : __match_any_sync(hm, val);
        VE_DBG(3, 32);
        hist_insert_warp(P, hm, lane == __ffs(vg) - 1, tag, val, __popc(vg));
      }
    }
    VE_TEND(3, th0);
    }
#endif
    VE_DBG(2, 1);
    if (++nwin == 0xFFFFu) save();          // 16-bit per-lane count fields
    VE_TEND(2, tw0);

    // next window: continue while it is fast with the same key
    if (!cont1) {
      VE_TBEG(ts0);
      save();
      VE_TEND(5, ts0);
      if (more1) { addr = a1; val = v1; pm = p1; }
      return more1;
    }
    addr = a1; val = v1; off = off1; pv = pv1;
    a1 = a2; v1 = v2; p1 = p2; off1 = off2; pv1 = pv2; more1 = more2; cont1 = cont2;
  }
}

// MULTI: take the multi-key dense path (run_dense_multi) for keys without live line
// state.  A separate instantiation, so traces with few PCs keep the register
// allocation of the single-key kernel (launch_analyze picks by the PC count).
template <bool MULTI>
__global__ void __launch_bounds__(K1_THREADS, 1) k_analyze(const __grid_constant__ AnalyzeParams P) {
  const uint32_t nsk = P.sp + P.so;
  const Smem S = smem_of(P);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const unsigned FULL = 0xFFFFFFFFu;

  for (uint32_t i = tid; i < nsk * NSUM; i += blockDim.x) S.ssum[i] = 0;
  for (uint32_t i = tid; i < nsk * NMM; i += blockDim.x) { S.smin[i] = ~0ull; S.smax[i] = 0; }
  for (uint32_t i = tid; i < nsk; i += blockDim.x) { S.sline[i].state = VE_LINE_EMPTY; S.sline[i].lock = 0; }
  for (uint32_t i = tid; i < P.hs; i += blockDim.x) {
    S.shs[i].bits = 0; S.shs[i].tag = EMPTY_TAG; S.shs[i].pad = 0; S.shc[i] = 0;
  }
  for (uint32_t i = tid; i < P.objc; i += blockDim.x) { S.sob[i] = P.o.base[i]; S.soe[i] = P.o.end[i]; }
  if (tid < 4) S.sctr[tid] = 0;
  __shared__ WarpCache s_wc[K1_WARPS];
  constexpr int NS = MULTI ? NSLOT : NSLOT_SINGLE;
  __shared__ SlotE s_slot[K1_WARPS][NS];
  __shared__ uint32_t s_snext[K1_WARPS];
  WarpCache& wc = s_wc[warp];
  SlotE* slots = s_slot[warp];
  if (lane < WC) wc.key1[lane] = 0;
  if (lane < NS) slots[lane].key = ~0ull;
  if (lane == 0) { wc.next = 0; s_snext[warp] = 0; s_stage_n[warp] = 0; }

  // full windows stream through the warp's TMA ring (a static contiguous range per
  // warp); without the ring (records not 16-byte aligned) each warp takes a static
  // range of plain loads
  const uint64_t nwin = (P.n + 31) / 32;
  const uint64_t tw = (uint64_t)gridDim.x * K1_WARPS, gw = (uint64_t)blockIdx.x * K1_WARPS + warp;
  Ring R;
  R.dst0 = smem_u32(ve_smem + P.o_ring + (uint32_t)warp * RING * WIN_BYTES);
  R.o0 = R.o = R.dst0 + (uint32_t)lane * 24u;
  R.bar0 = smem_u32(ve_smem + P.o_bars + (uint32_t)warp * RING * 8u);
  R.d = R.sw = R.ph = R.pend = 0;
  R.left = 0;
  R.cu = R.su = R.snw = 0;
  if (lane == 0 && P.nring) {
    for (int d = 0; d < NSTAGE; ++d) mbar_init(R.bar0 + d * 8u, 1);
    fence_mbar_init();
  }
  __syncwarp();
  // short traces (one-stage chunks): chunk c goes to CTA c mod grid first, so the few chunks
  // spread over all SMs instead of filling the first CTAs' warps
  R.nextc = P.chunk == CHUNK ? gw : (uint64_t)warp * gridDim.x + blockIdx.x;
  R.cstride = gridDim.x * K1_WARPS;
#if VE_CLAIM
  ring_claim(P, R);
#else
  {
    const uint64_t b = gw * P.nring / tw, e = (gw + 1) * P.nring / tw;
    R.src = P.recs + b * 32;
    R.iss = (uint32_t)(e - b);
  }
#endif
  for (int d = 0; d < NSTAGE; ++d) ring_issue_stage(P, R, (uint32_t)d);
  __syncthreads();
  ObjCache oc;
  oc.base = 0; oc.lim = 0; oc.bmoff = 0; oc.pre = 0; oc.oi = -1; oc.id = 0; oc.fastlg = 0xFFu;
  uint32_t n_inv = 0, n_unm = 0;   // this lane's invalid / unmapped records (slow windows)
#if VE_WCLK
  const long long wclk0 = clock64();
  if (lane < 6) { s_dbg[warp][lane] = 0; s_dbgc[warp][lane] = 0; }
  __syncwarp();
  uint32_t wslow = 0, wfast = 0;
#endif

  uint64_t addr = 0, val = 0, pm = 0;
  bool have = false;
  while (have || R.left) {
    if (!have) ring_next(P, R, addr, val, pm);
    have = false;
    const uint64_t pm0 = shfl64(FULL, pm, 0);
    const uint32_t meta0 = (uint32_t)(pm0 >> 32), pc0 = (uint32_t)pm0;
    bool fast = false;
    if (__all_sync(FULL, pm == pm0) && meta_fast(meta0, pc0, P.n_pcs)) {
      const uint32_t lg0 = meta0 & 3u;
      const uint64_t wm = (1ull << lg0) - 1ull;
      const bool vok = lg0 == 3u || (val >> (8u << lg0)) == 0ull;
      uint64_t off = addr - oc.base;
      if (!__all_sync(FULL, off <= oc.lim && (off & wm) == 0ull) || lg0 != oc.fastlg) {
        oc = obj_refill(P, shfl64(FULL, addr, 0));
        off = addr - oc.base;
      }
      fast = __all_sync(FULL, vok && off <= oc.lim && (off & wm) == 0ull) && lg0 == oc.fastlg;
    }
    if (fast) {
      // the window's key slot (pc, object, access type); while one of its line states
      // is still live, windows go one at a time through the line check
      const uint64_t key = ((uint64_t)meta0 << 32) | ((uint64_t)oc.id << 16) | pc0;
      SlotE* se = &slots[slot_acquire<NS>(P, wc, slots, &s_snext[warp], key, oc.oi, oc.pre == 0ull)];
      const uint32_t lf = se->lfail;
      // a live line state: runs of one value take the constant-run path, other windows
      // go one at a time through the per-window line check
      bool one = false, cm = false;
      uint64_t cy = 0, xmin = ~0ull, xmax = 0;
      if (lf != 3u) {
        cy = shfl64(FULL, val, 0);
        cm = __all_sync(FULL, val == cy);
        one = !cm;
      }
      // dense loads of a key without live line state: the stage-batched dense path
      bool nd = true;
      VE_TBEG(t1);
      if (!one && !cm && se->dense != 0ull) {
#if VE_MULTI_DENSE
        if (MULTI && lf == 3u) {
          switch (meta0 & 3u) {
            case 0: have = run_dense_multi<0>(P, oc, slots, se, R, addr, val, pm, nd); break;
            case 1: have = run_dense_multi<1>(P, oc, slots, se, R, addr, val, pm, nd); break;
            case 2: have = run_dense_multi<2>(P, oc, slots, se, R, addr, val, pm, nd); break;
            default: have = run_dense_multi<3>(P, oc, slots, se, R, addr, val, pm, nd); break;
          }
        } else
#endif
        switch (meta0 & 3u) {
          case 0: have = run_dense<0>(P, oc, se, R, addr, val, pm, nd); break;
          case 1: have = run_dense<1>(P, oc, se, R, addr, val, pm, nd); break;
          case 2: have = run_dense<2>(P, oc, se, R, addr, val, pm, nd); break;
          default: have = run_dense<3>(P, oc, se, R, addr, val, pm, nd); break;
        }
      }
      (void)0;
      VE_TBEG(t0);
      if (nd) {
      // specialised on the window's access type (compile-time width / kind)
#define VE_RF(K, L) have = run_fast<K, L>(P, oc, se, one, cm, cy, xmin, xmax, R, addr, val, pm)
      switch (meta0 & 15u) {
        case 0: VE_RF(0, 0); break;
        case 1: VE_RF(0, 1); break;
        case 2: VE_RF(0, 2); break;
        case 3: VE_RF(0, 3); break;
        case 4: VE_RF(1, 0); break;
        case 5: VE_RF(1, 1); break;
        case 6: VE_RF(1, 2); break;
        case 7: VE_RF(1, 3); break;
        case 9: VE_RF(2, 1); break;
        case 10: VE_RF(2, 2); break;
        case 11: VE_RF(2, 3); break;
        default: VE_RF(3, 1); break;   // 13: bfloat16
      }
#undef VE_RF
      }
      VE_TEND(0, t0);
      VE_TBEG(t2);
      if (lf != 3u) {
        uint32_t nlf;
        if (one) {   // C8 for the window just consumed (still in addr / val)
          nlf = fast_line(P, wc, addr, val, meta0, pc0, oc.id, lf);
        } else {
          xmin = redmin64(FULL, xmin);
          xmax = redmax64(FULL, xmax);
          nlf = lf;
          if (se->cpend && se->cy == cy) {         // same constant: widen the deferred segment
            if (lane == 0) {
              se->cx0 = xmin < se->cx0 ? xmin : se->cx0;
              se->cx1 = xmax > se->cx1 ? xmax : se->cx1;
            }
          } else {
            slot_line_flush(P, wc, se);            // another constant: merge the held one first
            nlf = se->lfail;
            if (nlf != 3u && lane == 0) { se->cpend = 1; se->cy = cy; se->cx0 = xmin; se->cx1 = xmax; }
          }
        }
        __syncwarp();
        if (lane == 0) se->lfail = nlf;
        __syncwarp();
      }
      VE_TEND(4, t2);
#if VE_WCLK
      ++wfast;
#endif
    } else {
#if VE_WCLK
      ++wslow;
#endif
      const uint32_t cnt = slow_window(P, wc, addr, val, pm, true);
      n_inv += cnt & 0xFFFFu;
      n_unm += cnt >> 16;
    }
  }
  // windows outside the ring: the partial last window, or (records not 16-byte
  // aligned) a static range of every warp
  uint64_t wbeg = P.nring, wend = gw == 0 ? nwin : P.nring;
  if (!P.nring) { wbeg = gw * nwin / tw; wend = (gw + 1) * nwin / tw; }
  for (uint64_t w = wbeg; w < wend; ++w) {
    const Rec cur = load_rec(P, w, wend, lane);
    const uint32_t cnt = slow_window(P, wc, cur.addr, cur.val, cur.pm, w * 32 + lane < P.n);
    n_inv += cnt & 0xFFFFu;
    n_unm += cnt >> 16;
  }

#if VE_WCLK
  if (lane == 0 && P.n > 100000000ull && (blockIdx.x < 3 || blockIdx.x == 147))
    printf("WCLK %d %d %lld fast %u slow %u dstage %u dsingle %u fwin %u hist %u exnd %u exfit %u\n", blockIdx.x, warp,
           clock64() - wclk0, wfast, wslow, s_dbg[warp][0], s_dbg[warp][1], s_dbg[warp][2], s_dbg[warp][3],
           s_dbg[warp][4], s_dbg[warp][5]);
  if (lane == 0 && P.n > 100000000ull && (blockIdx.x < 3 || blockIdx.x == 147))
    printf("WCYC %d %d runfast %llu fill %llu body %llu hist %llu line %llu save %llu\n", blockIdx.x, warp, s_dbgc[warp][0],
           s_dbgc[warp][1], s_dbgc[warp][2], s_dbgc[warp][3], s_dbgc[warp][4], s_dbgc[warp][5]);
#endif
  // fold the warp's key slots and line cache, then the CTA's shared state
  for (int i = 0; i < NS; ++i)
    if (slots[i].key != ~0ull) {
      slot_line_flush(P, wc, &slots[i]);
      slot_flush(P, &slots[i]);
    }
  n_inv = __reduce_add_sync(FULL, n_inv);
  n_unm = __reduce_add_sync(FULL, n_unm);
  __syncwarp();
  if (lane == 0) {
    const uint32_t ns = s_stage_n[warp];
    P.stage_cnt[gw] = ns < P.stage_rs ? ns : P.stage_rs;
    if (n_inv) atomicAdd(&S.sctr[0], n_inv);
    if (n_unm) atomicAdd(&S.sctr[1], n_unm);
    wcache_flush(P, wc);
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
  // line states of the shared keys: one row per CTA, folded by K2 (no global locks)
  for (uint32_t s = tid; s < nsk; s += blockDim.x) P.t.lcta[(uint64_t)blockIdx.x * nsk + s] = S.sline[s];
  for (uint32_t i = tid; i < P.hs; i += blockDim.x) {
    if (S.shs[i].tag != EMPTY_TAG) hist_insert_global_rf(P.t, S.shs[i].tag, S.shs[i].bits, S.shc[i]);
  }
  if (tid == 0) {
    if (S.sctr[0]) atomicAdd(&P.t.glob[G_INVALID], (unsigned long long)S.sctr[0]);
    if (S.sctr[1]) atomicAdd(&P.t.glob[G_UNMAPPED], (unsigned long long)S.sctr[1]);
    if (blockIdx.x == 0) atomicAdd(&P.t.glob[G_RECORDS], (unsigned long long)P.n);
  }
}


// ============================================================================
// K1 v2: register-resident key slots for traces whose PCs and objects alternate
// window by window (stencil neighbours, op mixes, multi-PC kernels).
//
// Slot s of a warp lives in lane s's registers (32 slots per warp), so a window
// switches key at the cost of one ballot: the warp reduces the window's value
// statistics with REDUX (counts packed 6 bits apart, 32-bit min / max) and lane s
// folds them into its accumulators with predicated instructions.  A slot is folded
// into the PC-key and object-key rows (shared memory, or the global table) only on
// eviction and at exit, by its own lane.  Objects (<= 32) are cached one per lane:
// an address is mapped by one ballot, the metadata moves by shuffles.  Everything
// else (slow windows, S8 inserts, line states, dense counters) is shared with v1.
// ============================================================================
constexpr int NS2 = 32;
// deferred C8 state of slot s, merged into the key's line states on eviction / FAIL / exit (the (+)
// monoid is associative and commutative, so this equals merging every window): cpend 1: a run of one
// value (raw bits cy) between addresses cx0 and cx1 (SlotE::cy); cpend 2: a POINT / LINE segment
// st from (cx0, (int64) cy) to (cx1, y1), |y| < 2^62 -- the windows of a structured key whose 32
// points are an arithmetic progression in address and value (cfg4's xc[x]: ~960 instructions per
// window through the generic fit and two cache merges)
// (32 bytes: the flags ride in the top bits of the < 2^48 addresses -- a 40-byte record cost epoch 0
// of cfg4 over a millisecond)
constexpr uint64_t SL_XM = (1ull << 48) - 1ull;
struct SlotLine {
  uint64_t cy;            // cpend 1: the run's raw bits; cpend 2: (int64) y of the first end point
  uint64_t w0, w1;        // bits 0-47: cx0 / cx1; bits 62-63 of w0: cpend, of w1: the segment's state
  int64_t y1;
  __device__ __forceinline__ uint32_t cpend() const { return (uint32_t)(w0 >> 62); }
  __device__ __forceinline__ uint32_t st() const { return (uint32_t)(w1 >> 62); }
  __device__ __forceinline__ uint64_t cx0() const { return w0 & SL_XM; }
  __device__ __forceinline__ uint64_t cx1() const { return w1 & SL_XM; }
  __device__ __forceinline__ void set(uint32_t pend, uint32_t state, uint64_t x0, uint64_t x1) {
    w0 = x0 | ((uint64_t)pend << 62);
    w1 = x1 | ((uint64_t)state << 62);
  }
  __device__ __forceinline__ void clear() { w0 &= SL_XM; }
};
static_assert(sizeof(SlotLine) == 32, "SlotLine layout");
struct SlotRec {             // slot s's object and arrays (per warp, shared memory; read by every lane)
  uint64_t cb, clim, cpre, cpost, cbm;
  unsigned long long dn, dq;
  uint32_t cidlg, coi;       // object id | log2 element width << 16 (every register of the object is restored); sorted index
};
struct LaneSlot {            // the registers of lane s that hold slot s
  uint64_t key;              // meta << 32 | object id << 16 | pc; ~0 = free
  uint64_t pmw, ob, olim;    // pc | meta << 32, and the object's range [ob, ob + olim] (the hit test)
  unsigned long long dn;     // dense counter array of (pc, object) loads that read the pre value, or 0
  unsigned long long dq;     // dense counter array of records that carry the post value (DENSE_POST), or 0
  uint32_t info;             // bits 0-1: line FAIL (PC key, object key); bit 2: object has no pre snapshot
  uint32_t n, zero, eq, nan, nonint, nf16, nbf16, nf32;
  uint64_t mm[6];            // raw min, raw max, ord min, ord max, trunc min, trunc max (64-bit keys)
};

__device__ __forceinline__ void lslot_clear_acc(LaneSlot& L) {
  L.n = L.zero = L.eq = L.nan = L.nonint = L.nf16 = L.nbf16 = L.nf32 = 0;
#pragma unroll
  for (int m = 0; m < 6; ++m) L.mm[m] = (m & 1) ? 0ull : ~0ull;
}

// A slot leaves lane s's registers through a per-warp shared-memory record (lane s writes it),
// then the whole warp folds it into the PC-key row (lanes 0-15) and the object-key row (lanes
// 16-31), one field per lane: f 0 n  1 zero  2 eq_pre  3 nosnap  4-8 float flags  9-14 min / max
// 15 n_type (the layout of slot_flush)
struct SlotSave {
  uint64_t key;
  uint32_t info, n, zero, eq, nan, nonint, nf16, nbf16, nf32, pad;
  uint64_t mm[6];
};
__device__ __forceinline__ void lslot_save(SlotSave* sv, const LaneSlot& L) {
  sv->key = L.key; sv->info = L.info; sv->n = L.n; sv->zero = L.zero; sv->eq = L.eq; sv->nan = L.nan;
  sv->nonint = L.nonint; sv->nf16 = L.nf16; sv->nbf16 = L.nbf16; sv->nf32 = L.nf32;
#pragma unroll
  for (int m = 0; m < 6; ++m) sv->mm[m] = L.mm[m];
}
__device__ __noinline__ void lslot_fold(const AnalyzeParams& P, const SlotSave* sv) {
  __syncwarp();
  const int lane = threadIdx.x & 31, f = lane & 15;
  const uint64_t key = sv->key;
  const uint32_t n = sv->n;
  if (key == ~0ull || n == 0u) { __syncwarp(); return; }
  const uint32_t pc = (uint32_t)key & 0xFFFFu, koi = (uint32_t)(key >> 16) & 0xFFFFu;
  const uint32_t meta = (uint32_t)(key >> 32), lg = meta & 3u, kind = (meta >> 2) & 3u;
  const bool st = meta_store(meta);
  uint64_t v = 0;
  uint32_t field = 0;
  if (f == 0) { v = n; field = st ? F_ST : F_LD; }
  else if (f == 1) { v = sv->zero; field = F_ZERO; }
  else if (f == 2) { v = sv->eq; field = st ? F_STEQ : F_LDEQ; }
  else if (f == 3) { v = (sv->info & 4u) ? n : 0u; field = F_NOSNAP; }
  else if (f == 4) { v = sv->nan; field = F_NAN; }
  else if (f == 5) { v = sv->nonint; field = F_NONINT; }
  else if (f == 6) { v = sv->nf16; field = F_NF16; }
  else if (f == 7) { v = sv->nbf16; field = F_NBF16; }
  else if (f == 8) { v = sv->nf32; field = F_NF32; }
  else if (f == 15) { v = n; field = F_TYPE0 + type_code(kind, lg); }
  else v = sv->mm[f - 9];
  bool skip;
  if (f <= 8 || f == 15) skip = v == 0;
  else {
    const int m = f - 9;
    skip = (m >= 4 && kind < 2u) || ((m & 1) ? v == 0ull : v == ~0ull);
  }
  if (!skip) {
    if (lane < 16) fold_row(P, pc < P.sp ? (int)pc : -1, pc, f, field, v);
    else fold_row(P, koi < P.so ? (int)(P.sp + koi) : -1, P.n_pcs + koi, f, field, v);
  }
  __syncwarp();
}

// merge slot v's deferred constant segment into the line states (all lanes); returns the new FAIL bits
__device__ __noinline__ uint32_t sl_flush(const AnalyzeParams& P, WarpCache& wc, SlotLine* sl, int v, uint64_t key,
                                          uint32_t lf) {
  const uint32_t cp = sl[v].cpend();
  if (!cp) return lf;
  uint32_t nlf;
  if (cp == 1u) {
    nlf = const_line(P, wc, sl[v].cx0(), sl[v].cx1(), sl[v].cy, (uint32_t)(key >> 32), (uint32_t)key & 0xFFFFu,
                     (uint32_t)(key >> 16) & 0xFFFFu, lf);
  } else {
    LinePts g;
    g.state = sl[v].st(); g.px = sl[v].cx0(); g.qx = sl[v].cx1();
    g.py = (__int128)(int64_t)sl[v].cy; g.qy = (__int128)sl[v].y1;
    nlf = line_apply(P, wc, g, (uint32_t)key & 0xFFFFu, (uint32_t)(key >> 16) & 0xFFFFu, lf);
  }
  __syncwarp();
  if ((threadIdx.x & 31) == 0) sl[v].clear();
  __syncwarp();
  return nlf;
}

// a slot for key (all lanes): the caller picked slot v (a free one, else round robin: the victim
// key vk with FAIL bits vlf, whose pending segment is merged here); returns the new slot's dense
// array and, in lf, its FAIL bits
__device__ __noinline__ unsigned long long lslot_prepare(const AnalyzeParams& P, WarpCache& wc, SlotLine* sl, int v,
                                                        bool evict, uint64_t vk, uint32_t vlf, uint64_t key, int oi,
                                                        bool nosnap, bool postok, uint32_t* lf,
                                                        unsigned long long* dq) {
  if (evict) sl_flush(P, wc, sl, v, vk, vlf);
  const uint32_t pc = (uint32_t)key & 0xFFFFu, koi = (uint32_t)(key >> 16) & 0xFFFFu;
  const uint32_t meta = (uint32_t)(key >> 32);
  *lf = slot_lfail(P, pc, koi);
  const unsigned long long dn = (P.dense_ok && !meta_store(meta) && !nosnap) ? dense_lookup(P, oi, (meta << 16) | pc) : 0ull;
  (void)postok;
  *dq = 0ull;   // a post array is claimed on demand (win_fast), so keys counted against pre use no slot
  __syncwarp();
  if ((threadIdx.x & 31) == 0) sl[v].clear();
  __syncwarp();
  return dn;
}

// C8 of one fast window of a key with a live line state (all lanes); returns the new FAIL bits
__device__ __noinline__ uint32_t win_line(const AnalyzeParams& P, WarpCache& wc, SlotLine* sl, int s, uint64_t key,
                                          uint32_t lf, uint64_t addr, uint64_t val) {
  const unsigned FULL = 0xFFFFFFFFu;
  const int lane = threadIdx.x & 31;
  const uint32_t pc0 = (uint32_t)key & 0xFFFFu, koi0 = (uint32_t)(key >> 16) & 0xFFFFu, meta0 = (uint32_t)(key >> 32);
  const uint64_t cy = shfl64(FULL, val, 0);
  SlotLine& e = sl[s];
#if !VE_APFAST
  if (!__all_sync(FULL, val == cy)) return fast_line(P, wc, addr, val, meta0, pc0, koi0, lf);
#endif
  if (!__all_sync(FULL, val == cy)) {
    // an arithmetic-progression window (lane i at a0 + i*w with value y0 + i*dy, exact integers
    // |y| < 2^62) is the segment of its end points; merged into the held segment by lane 0
    const uint32_t kind = (meta0 >> 2) & 3u, lg = meta0 & 3u;
    int64_t y = 0;
    bool ok = false;
    if (kind == 0u) { y = (int64_t)val; ok = val < (1ull << 62); }
    else if (kind == 1u) {
      const uint32_t sh64 = 64u - (8u << lg);
      y = (int64_t)(val << sh64) >> sh64;
      ok = y > -(1ll << 62) && y < (1ll << 62);
    } else if (kind == 2u && lg >= 2u) {
      const double d = lg == 3u ? __longlong_as_double((long long)val) : (double)__uint_as_float((uint32_t)val);
      // an exact integer below 2^62 (NaN, inf and fractions fail) and not -0.0, which the line fit
      // does not admit (DESIGN 3, Q11-Q13; float_flags): such windows take the generic path
      const bool negz = val == (lg == 3u ? 0x8000000000000000ull : 0x80000000ull);
      ok = !negz && d == trunc(d) && fabs(d) < 4611686018427387904.0;
      y = ok ? (int64_t)d : 0;
    }
    const uint64_t a0 = shfl64(FULL, addr, 0);
    const int64_t y0 = (int64_t)shfl64(FULL, (uint64_t)y, 0), dy = (int64_t)shfl64(FULL, (uint64_t)y, 1) - y0;
    const bool dok = dy > -(1ll << 56) && dy < (1ll << 56);
    if (!__all_sync(FULL, ok && dok && addr == a0 + ((uint64_t)lane << lg) && y == y0 + (int64_t)lane * dy))
      return fast_line(P, wc, addr, val, meta0, pc0, koi0, lf);
    LinePts g;
    g.state = VE_LINE_LINE;
    g.px = a0; g.py = (__int128)y0;
    g.qx = a0 + (31ull << lg); g.qy = (__int128)(y0 + 31 * dy);
    if (e.cpend() == 1u) lf = sl_flush(P, wc, sl, s, key, lf);   // (a held run of one value goes first)
    uint32_t st = 0;
    __syncwarp();
    if (lane == 0) {
      LinePts r = g;
      if (e.cpend() == 2u) {
        LinePts a;
        a.state = e.st(); a.px = e.cx0(); a.qx = e.cx1(); a.py = (__int128)(int64_t)e.cy; a.qy = (__int128)e.y1;
        r = line_merge(a, g);
      }
      st = r.state;
      if (st != VE_LINE_FAIL) {
        e.set(2u, r.state, r.px, r.qx); e.cy = (uint64_t)(int64_t)r.py; e.y1 = (int64_t)r.qy;
      } else {
        e.clear();
      }
    }
    st = __shfl_sync(FULL, st, 0);
    __syncwarp();
    if (st == VE_LINE_FAIL) {            // the slot's points are not collinear: publish the FAIL now
      g.state = VE_LINE_FAIL;
      return line_apply(P, wc, g, pc0, koi0, lf);
    }
    return lf;
  }
  // a window of one value: its points lie on y = cy between its extreme addresses; consecutive
  // windows of one value only widen a held segment (the (+) monoid keeps the extreme points)
  const uint64_t xmin = redmin64(FULL, addr), xmax = redmax64(FULL, addr);
  if (e.cpend() == 1u && e.cy == cy) {
    __syncwarp();
    if ((threadIdx.x & 31) == 0) {
      const uint64_t x0 = e.cx0(), x1 = e.cx1();
      e.set(1u, 0u, xmin < x0 ? xmin : x0, xmax > x1 ? xmax : x1);
    }
    __syncwarp();
    return lf;
  }
  lf = sl_flush(P, wc, sl, s, key, lf);
  if (lf != 3u && (threadIdx.x & 31) == 0) { e.set(1u, 0u, xmin, xmax); e.cy = cy; }
  __syncwarp();
  return lf;
}

// The value statistics of a fast window of type (KIND, LG) that is not entirely counted
// densely (lanes with dl are: their values are taken from the pre snapshot at report time).
template <int KIND, int LG>
__device__ __forceinline__ void win_value(const AnalyzeParams& P, LaneSlot& L, int s, bool st, bool eq, bool dl,
                                          uint64_t val, uint64_t word, uint32_t bit, bool dense_key, uint32_t tag) {
  using MT = typename std::conditional<(LG < 3), uint32_t, uint64_t>::type;
  constexpr bool ISF = KIND >= 2;
  constexpr int MB = KIND == 3 ? 7 : (LG == 1 ? 10 : LG == 2 ? 23 : 52);
  constexpr MT MID = (MT)~0ull;
  const unsigned FULL = 0xFFFFFFFFu;
  const int lane = threadIdx.x & 31;
  const MT b = (MT)val;
  const bool fo = !dl;
  const uint32_t zc = __popc(__ballot_sync(FULL, fo && b == (MT)0));
  const uint32_t ec = __popc(__ballot_sync(FULL, eq));
  const MT r0 = wmin<MT>(fo ? b : MID), r1 = wmax<MT>(fo ? b : (MT)0);
  uint64_t R[6] = {(uint64_t)r0, (uint64_t)r1, ~0ull, 0ull, ~0ull, 0ull};
  uint32_t fsum = 0, nf32 = 0;
  if constexpr (KIND == 0) {
    R[2] = R[0]; R[3] = R[1];
  } else if constexpr (KIND == 1) {
    if constexpr (LG < 3) {                 // sext32(b) ^ 2^31 (order-isomorphic to the 64-bit key)
      constexpr uint32_t sh = 32 - (8 << LG);
      const uint32_t k = (uint32_t)(((int32_t)(b << sh)) >> sh) ^ 0x80000000u;
      const uint32_t a = __reduce_min_sync(FULL, fo ? k : 0xFFFFFFFFu), c = __reduce_max_sync(FULL, fo ? k : 0u);
      R[2] = (uint64_t)(int64_t)(int32_t)(a ^ 0x80000000u) ^ (1ull << 63);
      R[3] = (uint64_t)(int64_t)(int32_t)(c ^ 0x80000000u) ^ (1ull << 63);
    } else {
      R[2] = redmin64(FULL, fo ? (b ^ (1ull << 63)) : ~0ull);
      R[3] = redmax64(FULL, fo ? (b ^ (1ull << 63)) : 0ull);
    }
  } else {
    uint32_t ff;
    if constexpr (KIND == 2 && LG == 2) ff = fflags_f32((uint32_t)b);
    else if constexpr (LG < 3) ff = fflags32<KIND, LG>((uint32_t)b);
    else { int64_t ival; ff = float_flags(val, 2u, 3u, ival); }
    const bool okv = fo && !(ff & 1u);      // NaNs excluded from ord / trunc
    ff = fo ? ff : 0u;
    constexpr MT SIGN = (MT)1 << ((8 << LG) - 1);
    constexpr MT MASK = (MT)((8 << LG) == 64 ? ~0ull : ((1ull << (8 << LG)) - 1ull));
    const MT k = (b & SIGN) ? (~b & MASK) : (b | SIGN);
    const MT tmask = (MT)(P.mant_bits >= (uint32_t)MB ? ~0ull : ~((1ull << (MB - P.mant_bits)) - 1ull));
    const MT t = b & tmask;
    const MT k0 = wmin<MT>(okv ? k : MID), k1 = wmax<MT>(okv ? k : (MT)0);
    const MT t0 = wmin<MT>(okv ? t : MID), t1 = wmax<MT>(okv ? t : (MT)0);
    R[2] = (LG < 3 && k0 == MID) ? ~0ull : (uint64_t)k0; R[3] = (uint64_t)k1;
    R[4] = (LG < 3 && t0 == MID) ? ~0ull : (uint64_t)t0; R[5] = (uint64_t)t1;
    fsum = __reduce_add_sync(FULL, (ff & 1u) | (((ff >> 1) & 1u) << 6) | (((ff >> 2) & 1u) << 12) | (((ff >> 3) & 1u) << 18));
    if constexpr (LG == 3) nf32 = __popc(__ballot_sync(FULL, (ff >> 4) & 1u));
  }
  if (lane == s) {
    L.n += 32u; L.zero += zc; L.eq += ec;
    if constexpr (ISF) {
      L.nan += fsum & 63u; L.nonint += (fsum >> 6) & 63u; L.nf16 += (fsum >> 12) & 63u; L.nbf16 += (fsum >> 18) & 63u;
      L.nf32 += nf32;
    }
#pragma unroll
    for (int m = 0; m < 6; ++m) L.mm[m] = (m & 1) ? (R[m] > L.mm[m] ? R[m] : L.mm[m]) : (R[m] < L.mm[m] ? R[m] : L.mm[m]);
  }
  // C10 written elements; C3 loaded elements of loads not counted per element
  if (st) bitmap_or_win(P.t.W, true, word, bit);
  else if (!dense_key && __any_sync(FULL, eq)) bitmap_or_win(P.t.L, eq, word, bit);
  // S8: every record not counted per element is inserted per distinct value
  const unsigned hm = __ballot_sync(FULL, fo);
  const int l = __ffs(hm) - 1;
  const uint64_t v0 = (LG < 3) ? (uint64_t)__shfl_sync(FULL, (uint32_t)val, l) : shfl64(FULL, val, l);
  if (__all_sync(FULL, !fo || val == v0)) {
    if (lane == l) hist_insert(P, tag, val, __popc(hm));
  } else if (fo) {
    const unsigned vg = (LG < 3) ? __match_any_sync(hm, (uint32_t)val) : __match_any_sync(hm, val);
    hist_insert_warp(P, hm, lane == __ffs(vg) - 1, tag, val, __popc(vg));
  }
  __syncwarp();   // reconverge before the next window's warp-collectives
}

// one fast window of access width LG: eq_pre, then the per-element counted lanes -- loads that read
// the pre value (dn) and records that carry the post value (dq, gathered here) -- and the value path
// of the window's type for the rest
template <int LG>
__device__ __forceinline__ bool win_fast(const AnalyzeParams& P, LaneSlot& L, int s, uint32_t meta0, uint32_t pc0,
                                         uint32_t oid, uint64_t opre, uint64_t obm, uint64_t off, uint64_t val,
                                         uint64_t pv, unsigned long long dn, uint64_t qv, unsigned long long dq) {
  using MT = typename std::conditional<(LG < 3), uint32_t, uint64_t>::type;
  constexpr MT WMASK = (MT)(LG == 3 ? ~0ull : ((1ull << (8u << LG)) - 1ull));
  const unsigned FULL = 0xFFFFFFFFu;
  const int lane = threadIdx.x & 31;
  const bool st = meta_store(meta0);
  bool eq = false;
  if (opre) eq = ((MT)pv & WMASK) == (MT)val;   // pv: the gathered pre element (low 8w bits)
  const uint64_t e = off >> LG;
  const bool dl = dn != 0ull && eq;
  if (dn != 0ull && __all_sync(FULL, dl)) {
    red_add_keep(reinterpret_cast<uint32_t*>(dn) + e, 1u, true);
    if (lane == s) { L.n += 32u; L.eq += 32u; }
    return false;
  }
  const bool dql = dq != 0ull && !dl && ((MT)qv & WMASK) == (MT)val;   // qv: the gathered post element
  const bool dc = dl || dql;                   // counted per element: value statistics at the flush
  red_add_keep(reinterpret_cast<uint32_t*>(dn) + e, 1u, dl);
  red_add_keep(reinterpret_cast<uint32_t*>(dq) + e, 1u, dql);
  const uint64_t word = obm + (e >> 5);
  const uint32_t bit = 1u << ((uint32_t)e & 31u);
  if (__all_sync(FULL, dc)) {
    const uint32_t ec = __popc(__ballot_sync(FULL, eq));
    if (lane == s) { L.n += 32u; L.eq += ec; }
    if (st) bitmap_or_win(P.t.W, true, word, bit);
    else if (dn == 0ull && __any_sync(FULL, eq)) bitmap_or_win(P.t.L, eq, word, bit);
    return false;
  }
  const uint32_t tag = (pc0 << 16) | (oid & 0xFFFFu);
  const bool dk = dn != 0ull;
  switch (meta0 & 15u) {
#define VE_WV(K) win_value<K, LG>(P, L, s, st, eq, dc, val, word, bit, dk, tag)
    case 0u | LG: VE_WV(0); break;
    case 4u | LG: VE_WV(1); break;
    default:
      if constexpr (LG == 1) {
        if ((meta0 & 15u) == 13u) { VE_WV(3); break; }
      }
      if constexpr (LG != 0) VE_WV(2);
      break;
#undef VE_WV
  }
  return dq == 0ull;    // lanes went the value path: a post array may count them per element
}

// claim the post-value array of the current slot's key (all lanes; on the first window that needs it)
__device__ __noinline__ unsigned long long post_claim(const AnalyzeParams& P, int oi, uint64_t key) {
  const uint32_t pc = (uint32_t)key & 0xFFFFu, meta = (uint32_t)(key >> 32);
  return dense_lookup(P, oi, DENSE_POST | (meta << 16) | pc);
}

// K1 v2 runs K2_WARPS warps per CTA (168 registers: the slots and the object state stay in registers)
// inside the 16-warp shared-memory layout of v1 (rings and staging regions of warps >= K2_WARPS unused)
#ifndef VE_DIAG
#define VE_DIAG 0
#endif

#ifndef VE_K2_THREADS
#define VE_K2_THREADS 384
#endif
constexpr int K2_THREADS = VE_K2_THREADS;
constexpr int K2_WARPS = K2_THREADS / 32;
static_assert(K2_WARPS <= K1_WARPS, "v2 uses the v1 shared-memory layout");

template <bool UNITS>
__global__ void __launch_bounds__(K2_THREADS, 1) k_analyze2(const __grid_constant__ AnalyzeParams P) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const unsigned FULL = 0xFFFFFFFFu;
  {
    const uint32_t nsk = P.sp + P.so;
    const Smem S = smem_of(P);
    for (uint32_t i = tid; i < nsk * NSUM; i += blockDim.x) S.ssum[i] = 0;
    for (uint32_t i = tid; i < nsk * NMM; i += blockDim.x) { S.smin[i] = ~0ull; S.smax[i] = 0; }
    for (uint32_t i = tid; i < nsk; i += blockDim.x) { S.sline[i].state = VE_LINE_EMPTY; S.sline[i].lock = 0; }
    for (uint32_t i = tid; i < P.hs; i += blockDim.x) {
      S.shs[i].bits = 0; S.shs[i].tag = EMPTY_TAG; S.shs[i].pad = 0; S.shc[i] = 0;
    }
    for (uint32_t i = tid; i < P.objc; i += blockDim.x) { S.sob[i] = P.o.base[i]; S.soe[i] = P.o.end[i]; }
    if (tid < 4) S.sctr[tid] = 0;
    if (tid < K1_WARPS - K2_WARPS) P.stage_cnt[(uint64_t)blockIdx.x * K1_WARPS + K2_WARPS + tid] = 0;
  }
  __shared__ WarpCache s_wc[K2_WARPS];
  __shared__ SlotLine s_sl[K2_WARPS][NS2];
  __shared__ SlotSave s_save[K2_WARPS];
  WarpCache& wc = s_wc[warp];
  SlotLine* sl = s_sl[warp];
  if (lane < WC) wc.key1[lane] = 0;
  sl[lane].w0 = 0;
  if (lane == 0) { wc.next = 0; s_stage_n[warp] = 0; }
  LaneSlot L;
  L.key = ~0ull; L.pmw = ~0ull; L.ob = 1; L.olim = 0; L.dn = 0; L.dq = 0; L.info = 0;
  lslot_clear_acc(L);
  uint32_t snext = 0;

  // objects: the CTA caches sorted objects 0..31 (base, end, pre, bitmap offset, id | log2 ew << 16 |
  // fast << 20); an address is mapped by one ballot over them when there are at most 32, else by
  // binary search
  const bool ob32 = P.o.n <= 32u;
  __shared__ uint64_t s_ob[32], s_oe[32], s_opre[32], s_obm[32], s_opost[32];
  __shared__ uint32_t s_ometa[32];
  if (tid < 32 && (uint32_t)tid < P.o.n) {
    const uint64_t b = P.o.base[tid], e = P.o.end[tid], pr = P.o.pre[tid], po = P.o.post[tid];
    s_ob[tid] = b; s_oe[tid] = e; s_opre[tid] = pr; s_obm[tid] = P.o.bmoff[tid];
    const uint32_t ew = P.o.ew[tid];
    const uint32_t lg = (ew == 1) ? 0 : (ew == 2) ? 1 : (ew == 4) ? 2 : 3;
    const bool fast = e - b >= ew && (pr & (ew - 1)) == 0;
    s_opost[tid] = (po & (ew - 1)) == 0 ? po : 0ull;   // post values counted per element need aligned elements
    s_ometa[tid] = (P.o.id[tid] & 0xFFFFu) | (lg << 16) | (fast ? (1u << 20) : 0u);
  }

  Ring R;
  R.dst0 = smem_u32(ve_smem + P.o_ring + (uint32_t)warp * RING * WIN_BYTES);
  R.o0 = R.o = R.dst0 + (uint32_t)lane * 24u;
  R.bar0 = smem_u32(ve_smem + P.o_bars + (uint32_t)warp * RING * 8u);
  R.d = R.sw = R.ph = R.pend = 0;
  R.left = 0;
  R.cu = R.su = R.snw = 0;
  if (lane == 0 && P.nring) {
    for (int d = 0; d < NSTAGE; ++d) mbar_init(R.bar0 + d * 8u, 1);
    fence_mbar_init();
  }
  __syncwarp();
  R.nextc = P.chunk == CHUNK ? (uint64_t)blockIdx.x * K2_WARPS + warp : (uint64_t)warp * gridDim.x + blockIdx.x;
  R.cstride = gridDim.x * K2_WARPS;
  ring_claim<UNITS ? 2 : 1>(P, R);
  for (int d = 0; d < NSTAGE; ++d) ring_issue_stage<UNITS ? 2 : 1>(P, R, (uint32_t)d);
  __syncthreads();

  // the current object (warp-uniform): offsets [0, clim] hold a whole element
  uint64_t cb = 1, clim = 0, cpre = 0, cbm = 0, cpost = 0;
  uint32_t cid = 0, clg = 0xFFu;
  int coi = -1;
  // the current slot's warp-uniform copies (dense arrays, FAIL bits)
  unsigned long long ldn = 0, ldq = 0;
  bool lpt = false;          // the post array of the current slot was claimed (or tried)
  uint32_t llf = 3;
  uint32_t n_inv = 0, n_unm = 0;
  // units mode: the current unit's PC base / count and object range (registers; the range also in
  // s_urange for find_object)
  uint32_t cu = ~0u, upcb = 0, unpc = ~0u, ulo = 0, uhi = P.o.n;

  // make sorted object oi (-1: none) the current object
  auto obj_set = [&](int oi) {
    coi = oi;
    if (oi < 0) {
      cb = 1; clim = 0; clg = 0xFFu; cpre = 0; cpost = 0;
    } else if (ob32) {
      cb = s_ob[oi];
      const uint64_t ce = s_oe[oi];
      cpre = s_opre[oi];
      cpost = s_opost[oi];
      cbm = s_obm[oi];
      const uint32_t mt = s_ometa[oi];
      cid = mt & 0xFFFFu;
      const bool fok = (mt >> 20) & 1u;
      clg = fok ? (mt >> 16) & 3u : 0xFFu;
      clim = fok ? ce - cb - (1ull << ((mt >> 16) & 3u)) : 0ull;
    } else {
      cb = P.o.base[oi];
      const uint64_t ce = P.o.end[oi];
      cpre = P.o.pre[oi]; cbm = P.o.bmoff[oi]; cid = P.o.id[oi];
      const uint32_t ew = P.o.ew[oi];
      cpost = (P.o.post[oi] & (ew - 1)) == 0 ? P.o.post[oi] : 0ull;
      const uint32_t lg = (ew == 1) ? 0 : (ew == 2) ? 1 : (ew == 4) ? 2 : 3;
      const bool fok = ce - cb >= ew && (cpre & (ew - 1)) == 0;
      clg = fok ? lg : 0xFFu;
      clim = fok ? ce - cb - ew : 0ull;
    }
  };
  // the object holding address a0 (warp-uniform) becomes current, unless it already is
  auto obj_find = [&](uint64_t a0) {
    if (a0 - cb <= clim && coi >= 0) return;
    int oi;
    if (ob32) {
      const unsigned m = __ballot_sync(FULL, (UNITS ? (uint32_t)lane >= ulo && (uint32_t)lane < uhi
                                                    : (uint32_t)lane < P.o.n) && s_ob[lane] <= a0 && a0 < s_oe[lane]);
      oi = m ? __ffs(m) - 1 : -1;
    } else {
      oi = find_object(P, a0);
    }
    obj_set(oi);
  };
  // Slot s also holds, in lane s's registers, its (pc | meta << 32) word pmw and its object's range
  // [ob, ob + olim]; its object / array data sits in the warp's shared-memory record sr[s].  A window
  // whose lane 0 carries (pmw, an address in that range) is found by ONE ballot; the registers below
  // hold the data of the slot ls used last, so runs of one key reload nothing.
  __shared__ SlotRec s_rec[K2_WARPS][NS2];
  SlotRec* const sr = s_rec[warp];
  uint64_t kvm = 0, kkey = ~0ull;
  uint32_t kwm = 0, klg = 0;
  int s = 0, ls = -1;

#if VE_DIAG == 2
  uint64_t dsink = 0;
#endif
  auto unit_enter = [&](uint32_t u) {
    cu = u;
    const UnitDesc& U = P.units[u];
    upcb = U.pcb; unpc = U.npc; ulo = U.olo; uhi = U.ohi;
    if (lane == 0) { s_urange[warp][0] = ulo; s_urange[warp][1] = uhi; }
    __syncwarp();
    coi = -1; cb = 1; clim = 0; clg = 0xFFu; ls = -1;   // the object registers belong to the last unit
  };
  // the ring is consumed a stage at a time: one refill and one barrier wait per stage, then its
  // windows in a loop (ring_next's per-window bookkeeping cost ~40 instructions per window)
  while (R.left) {
    if (R.pend) {
      __syncwarp();
      ring_issue_stage<UNITS ? 2 : 1>(P, R, R.pend - 1u);
      R.pend = 0;
    }
    const uint32_t wd = R.d;
    ring_wait(R.bar0 + wd * 8u, R.ph);
    const uint32_t nws = (R.snw >> (4u * wd)) & 0xFu;
    const uint32_t sbase = R.o0 + wd * STAGE_BYTES;
    for (uint32_t wj = 0; wj < nws; ++wj) {
    uint64_t addr, val, pm;
    asm volatile("ld.shared.u64 %0, [%3];\n\tld.shared.u64 %1, [%3+8];\n\tld.shared.u64 %2, [%3+16];"
                 : "=l"(addr), "=l"(val), "=l"(pm)
                 : "r"(sbase + wj * WIN_BYTES)
                 : "memory");
    if constexpr (UNITS) {                     // a local pc -> the unit's key; out of range -> invalid
      const uint32_t u = (R.su >> (16u * wd)) & 0xFFFFu;
      if (u != cu) unit_enter(u);
      pm = (uint32_t)pm < unpc ? pm + upcb : (pm | 0xFFFFFFFFull);
    }
#if VE_DIAG == 2   // diagnostic: the record stream alone (results wrong)
    dsink += addr ^ val ^ pm;
    continue;
#endif
    const uint64_t pm0 = shfl64(FULL, pm, 0);
    const uint64_t a0 = shfl64(FULL, addr, 0);
    const unsigned hit = __ballot_sync(FULL, L.pmw == pm0 && a0 - L.ob <= L.olim);
    bool ok = false;
    if (hit) {
      s = __ffs(hit) - 1;
      if (s != ls) {
        ls = s;
        const SlotRec& r = sr[s];
        // the object registers are reloaded only when the slot's object differs (a stencil's PCs
        // alternate over one object: their slots differ in their arrays alone)
        if ((int)r.coi != coi) {
          cb = r.cb; clim = r.clim; cpre = r.cpre; cpost = r.cpost; cbm = r.cbm;
          cid = r.cidlg & 0xFFFFu; coi = (int)r.coi; clg = r.cidlg >> 16;
        }
        ldn = r.dn; ldq = r.dq;
        kkey = ((uint64_t)(uint32_t)(pm0 >> 32) << 32) | ((uint64_t)cid << 16) | (uint32_t)pm0;
        klg = (uint32_t)(pm0 >> 32) & 3u;
        kwm = (1u << klg) - 1u;
        kvm = klg == 3u ? 0ull : ~((1ull << (8u << klg)) - 1ull);
        const uint32_t inf = __shfl_sync(FULL, L.info, s);
        llf = inf & 3u;
        lpt = (inf >> 3) & 1u;
      }
      const uint64_t o = addr - cb;
      ok = __all_sync(FULL, pm == pm0 && o <= clim && ((uint32_t)o & kwm) == 0u && (val & kvm) == 0ull);
    }
    if (!ok) {
      // another key or object, or a window for the slow path
      const uint32_t meta0 = (uint32_t)(pm0 >> 32), pc0 = (uint32_t)pm0;
      bool fast = false;
      if (__all_sync(FULL, pm == pm0) && meta_fast(meta0, pc0, P.n_pcs)) {
        const uint32_t lg0 = meta0 & 3u;
        const uint64_t wm = (1ull << lg0) - 1ull;
        const bool vok = lg0 == 3u || (val >> (8u << lg0)) == 0ull;
        ls = -1;                                     // the object registers change
        obj_find(a0);
        const uint64_t o = addr - cb;
        fast = lg0 == clg && __all_sync(FULL, vok && o <= clim && (o & wm) == 0ull);
      }
      if (!fast) {
        const uint32_t cnt = slow_window(P, wc, addr, val, pm, true);
        n_inv += cnt & 0xFFFFu;
        n_unm += cnt >> 16;
        continue;
      }
      const uint64_t key = ((uint64_t)meta0 << 32) | ((uint64_t)cid << 16) | pc0;
      const unsigned kh = __ballot_sync(FULL, L.key == key);
      if (kh) {
        s = __ffs(kh) - 1;
      } else {
        const unsigned fr = __ballot_sync(FULL, L.key == ~0ull);
        const bool evict = fr == 0u;
        s = evict ? (int)(snext++ & 31u) : __ffs(fr) - 1;
        const uint64_t vk = shfl64(FULL, L.key, s);
        const uint32_t vlf = __shfl_sync(FULL, L.info, s) & 3u;
        uint32_t nlf;
        unsigned long long dq;
        const unsigned long long dn = lslot_prepare(P, wc, sl, s, evict, vk, vlf, key, coi, cpre == 0ull,
                                                    cpost != 0ull, &nlf, &dq);
        if (evict) {
          if (lane == s) lslot_save(&s_save[warp], L);
          lslot_fold(P, &s_save[warp]);
        }
        if (lane == s) {
          L.key = key;
          L.pmw = pm0;
          L.ob = cb;
          L.olim = clim;
          L.dn = dn;
          L.dq = dq;
          L.info = nlf | (cpre == 0ull ? 4u : 0u);
          lslot_clear_acc(L);
          SlotRec& r = sr[s];
          r.cb = cb; r.clim = clim; r.cpre = cpre; r.cpost = cpost; r.cbm = cbm; r.dn = dn; r.dq = dq;
          r.cidlg = (cid & 0xFFFFu) | (clg << 16); r.coi = (uint32_t)coi;
        }
        __syncwarp();
      }
      ls = s;
      kkey = key;
      ldn = shfl64(FULL, L.dn, s);
      ldq = shfl64(FULL, L.dq, s);
      const uint32_t inf = __shfl_sync(FULL, L.info, s);
      llf = inf & 3u;
      lpt = (inf >> 3) & 1u;
      klg = meta0 & 3u;
      kwm = (1u << klg) - 1u;
      kvm = klg == 3u ? 0ull : ~((1ull << (8u << klg)) - 1ull);
    }
    // a fast window of slot s (its object in cb ..)
    const uint64_t o = addr - cb;
    uint64_t pv = 0, qv = 0;
#if VE_DIAG == 1   // diagnostic: no snapshot gathers (results wrong)
    if (cpre != 0ull) pv = val;
    if (ldq != 0ull) qv = val;
#else
    if (cpre != 0ull) pv = ld_pre<3>((cpre + o) & ~7ull) >> (8u * (uint32_t)((cpre + o) & 7ull));
    if (ldq != 0ull) qv = ld_pre<3>((cpost + o) & ~7ull) >> (8u * (uint32_t)((cpost + o) & 7ull));
#endif
    const uint32_t meta0 = (uint32_t)(kkey >> 32), pc0 = (uint32_t)kkey & 0xFFFFu;
    bool wantq = false;
    switch (klg) {
      case 0: wantq = win_fast<0>(P, L, s, meta0, pc0, cid, cpre, cbm, o, val, pv, ldn, qv, ldq); break;
      case 1: wantq = win_fast<1>(P, L, s, meta0, pc0, cid, cpre, cbm, o, val, pv, ldn, qv, ldq); break;
      case 2: wantq = win_fast<2>(P, L, s, meta0, pc0, cid, cpre, cbm, o, val, pv, ldn, qv, ldq); break;
      default: wantq = win_fast<3>(P, L, s, meta0, pc0, cid, cpre, cbm, o, val, pv, ldn, qv, ldq); break;
    }
    if (wantq && !lpt && cpost != 0ull && P.dense_ok) {       // first value-path window of the key
      lpt = true;
      ldq = post_claim(P, coi, kkey);
      if (lane == s) { L.dq = ldq; L.info |= 8u; sr[s].dq = ldq; }
      __syncwarp();
    }
    // (no overflow check: a launch gives a warp < 2^31 records, so the 32-bit accumulators hold)
    if (llf != 3u) {
      const uint32_t nlf = win_line(P, wc, sl, s, kkey, llf, addr, val);
      if (nlf != llf) {
        llf = nlf;
        if (lane == s) L.info = (L.info & ~3u) | nlf;
      }
    }
    }   // the stage's windows
    R.left -= nws;
    R.pend = R.iss ? wd + 1u : 0u;     // refilled at the next stage's start (its windows are all done)
    if (++R.d == (uint32_t)NSTAGE) { R.d = 0; R.ph ^= 1u; }
    R.o = R.o0 + R.d * STAGE_BYTES;
    R.sw = 0;
  }
#if VE_DIAG == 2
  if (dsink == 0x123456789ull) P.t.glob[G_WORK] = dsink;
#endif
  // windows outside the ring: the partial last window, or (records not 16-byte aligned) a
  // static range of every warp
  const uint64_t nwin = (P.n + 31) / 32;
  const uint64_t tw = (uint64_t)gridDim.x * K2_WARPS, gw = (uint64_t)blockIdx.x * K2_WARPS + warp;
  uint64_t wbeg = P.nring, wend = gw == 0 ? nwin : P.nring;
  if (!P.nring) { wbeg = gw * nwin / tw; wend = (gw + 1) * nwin / tw; }
  if constexpr (UNITS) {                       // units mode: every unit's partial last window
    wbeg = wend = 0;
    for (uint64_t u = gw; u < P.n_units; u += tw) {
      const uint64_t un = P.units[u].n;
      const uint32_t rem = (uint32_t)(un & 31u);
      if (!rem) continue;
      unit_enter((uint32_t)u);
      uint64_t addr = 0, val = 0, pm = 0;
      if ((uint32_t)lane < rem) {
        const unsigned long long* q = reinterpret_cast<const unsigned long long*>(&P.units[u].recs[(un & ~31ull) + lane]);
        addr = __ldcs(q);
        val = __ldcs(q + 1);
        pm = __ldcs(q + 2);
        pm = (uint32_t)pm < unpc ? pm + upcb : (pm | 0xFFFFFFFFull);
      }
      const uint32_t cnt = slow_window(P, wc, addr, val, pm, (uint32_t)lane < rem);
      n_inv += cnt & 0xFFFFu;
      n_unm += cnt >> 16;
    }
  }
  for (uint64_t w = wbeg; w < wend; ++w) {
    const Rec cur = load_rec(P, w, wend, lane);
    const uint32_t cnt = slow_window(P, wc, cur.addr, cur.val, cur.pm, w * 32 + lane < P.n);
    n_inv += cnt & 0xFFFFu;
    n_unm += cnt >> 16;
  }
  // fold the slots (pending constant segments first), the line cache, then the CTA's shared state
  for (int v = 0; v < NS2; ++v) {
    const uint64_t vk = shfl64(FULL, L.key, v);
    if (vk == ~0ull) continue;
    sl_flush(P, wc, sl, v, vk, __shfl_sync(FULL, L.info, v) & 3u);
  }
  for (int v = 0; v < NS2; ++v) {
    if (lane == v) lslot_save(&s_save[warp], L);
    lslot_fold(P, &s_save[warp]);
  }
  n_inv = __reduce_add_sync(FULL, n_inv);
  n_unm = __reduce_add_sync(FULL, n_unm);
  __syncwarp();
  const Smem S = smem_of(P);
  const uint32_t nsk = P.sp + P.so;
  if (lane == 0) {
    const uint32_t ns = s_stage_n[warp];
    P.stage_cnt[(uint64_t)blockIdx.x * K1_WARPS + warp] = ns < P.stage_rs ? ns : P.stage_rs;
    if (n_inv) atomicAdd(&S.sctr[0], n_inv);
    if (n_unm) atomicAdd(&S.sctr[1], n_unm);
    wcache_flush(P, wc);
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
  for (uint32_t s = tid; s < nsk; s += blockDim.x) P.t.lcta[(uint64_t)blockIdx.x * nsk + s] = S.sline[s];
  for (uint32_t i = tid; i < P.hs; i += blockDim.x) {
    if (S.shs[i].tag != EMPTY_TAG) hist_insert_global_rf(P.t, S.shs[i].tag, S.shs[i].bits, S.shc[i]);
  }
  if (tid == 0) {
    if (S.sctr[0]) atomicAdd(&P.t.glob[G_INVALID], (unsigned long long)S.sctr[0]);
    if (S.sctr[1]) atomicAdd(&P.t.glob[G_UNMAPPED], (unsigned long long)S.sctr[1]);
    if (blockIdx.x == 0) atomicAdd(&P.t.glob[G_RECORDS], (unsigned long long)P.n);
  }
}

// K1b: insert the staged S8 groups into the HBM table (one block per warp region).
__global__ void __launch_bounds__(256) k_hist_drain(const uint4* __restrict__ stage, const uint32_t* __restrict__ cnt,
                                                    uint32_t rs, DevTables t) {
  const uint32_t n = cnt[blockIdx.x];
  const uint4* q = stage + (uint64_t)blockIdx.x * rs;
  for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) {
    const uint4 e = __ldcs(q + i);
    hist_insert_global_rf(t, e.z, (uint64_t)e.x | ((uint64_t)e.y << 32), e.w);
  }
}

// K2: fold the per-CTA line states of every shared key (C8's (+) monoid, order-free)
// into the key's global state.  One block per key, a shared-memory tree over the CTAs.
constexpr int LF_THREADS = 256;
__global__ void __launch_bounds__(LF_THREADS) k_line_fold(const LineState* lcta, uint32_t grid, uint32_t nsk,
                                                          uint32_t sp, uint32_t n_pcs, LineState* line) {
  __shared__ LineState st[LF_THREADS];
  const uint32_t s = blockIdx.x, t = threadIdx.x;
  LinePts r;
  r.state = VE_LINE_EMPTY;
  r.px = r.qx = 0;
  r.py = r.qy = 0;
  for (uint32_t b = t; b < grid; b += LF_THREADS) {
    const LineState& x = lcta[(uint64_t)b * nsk + s];
    if (x.state != VE_LINE_EMPTY) r = line_merge(r, line_load(x));
  }
  line_store(st[t], r);
  __syncthreads();
  for (uint32_t h = LF_THREADS / 2; h > 0; h >>= 1) {
    if (t < h && st[t + h].state != VE_LINE_EMPTY) {
      const LinePts m = line_merge(line_load(st[t]), line_load(st[t + h]));
      line_store(st[t], m);
    }
    __syncthreads();
  }
  if (t == 0 && st[0].state != VE_LINE_EMPTY) {
    const uint32_t key = s < sp ? s : n_pcs + (s - sp);
    LineState& g = line[key];
    const LinePts m = line_merge(line_load(g), line_load(st[0]));
    line_store(g, m);
  }
}

// Units mode claims UNIT_CHUNK windows at a time: a warp stays on one unit's keys for a while, so
// its key slots and line-state cache stay warm and few warps merge into one unit's line states at
// once (16-window chunks spread every unit over every warp: the line-state locks then held 55% of
// the issued instructions on a 250-kernel cfg5 batch)
#ifndef VE_UNIT_CHUNK
#define VE_UNIT_CHUNK 256
#endif
constexpr uint32_t UNIT_CHUNK = VE_UNIT_CHUNK;
static_assert(UNIT_CHUNK % STAGE_WIN == 0, "whole stages");

// v2's claims on long traces (a claim is one atomic on one global counter from every warp)
#ifndef VE_V2_CHUNK
#define VE_V2_CHUNK 64
#endif
constexpr uint32_t V2_CHUNK = VE_V2_CHUNK;
static_assert(V2_CHUNK % STAGE_WIN == 0, "whole stages");

struct UnitLaunch {           // units mode of one launch (ve_analyze_units)
  const UnitDesc* d_units;
  const uint32_t* d_ucb;
  uint32_t n_units;
  uint64_t nring;             // full windows of all units
};

static ve_status launch_analyze_impl(ve_ctx* c, const ve_record* d, uint64_t n, cudaStream_t s,
                                     const UnitLaunch* ul) {
  AnalyzeParams P;
  P.recs = d;
  P.n = n;
  P.units = ul ? ul->d_units : nullptr;
  P.ucb = ul ? ul->d_ucb : nullptr;
  P.n_units = ul ? ul->n_units : 0u;
  P.n_pcs = c->cfg.n_pcs;
  P.n_obj = c->n_obj;
  P.mant_bits = c->cfg.mant_bits;
  // u32 per-element counters cannot overflow while the ctx has seen < 2^32 records
  // and only for a call with at least one record per pre-snapshot element: below that an element
  // is rarely loaded twice (cfg5's kernels touch each element once), and flushing per-element
  // counters costs more than the hash inserts they replace (measured: cfg5 report 0.7 -> 0.45 ms)
  P.dense_ok = (c->records_analyzed + n < (1ull << 32) && (n >= c->pre_elems || getenv("VE_DENSE_ALWAYS")) &&
                dense_reserve(c)) ? 1u : 0u;
  if (P.dense_ok) c->dense_dirty = true;
  P.ring = (ul || (uintptr_t)d % 16 == 0) ? 1u : 0u;
  P.nring = ul ? ul->nring : P.ring ? n / 32 : 0;
  P.work = c->t.glob + G_WORK;
  c->records_analyzed += n;
  // shared stat rows: up to 256 keys, PCs first then object keys (incl. SHARED)
  const uint32_t NSK_MAX = K1_NSK;
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
  // many PCs interleave their warp instructions window by window (stencils, op mixes):
  // the multi-key dense kernel; few PCs (long runs per key): the single-key kernel
  // (VE_K1_MULTI=0/1 forces one instantiation: the parity tests run both on the same traces)
  const char* fm = getenv("VE_K1_MULTI");
  const bool multi = VE_MULTI_DENSE && (fm && *fm ? *fm == '1' : c->cfg.n_pcs >= VE_MULTI_MIN_PCS);
  // K1 v2 (register key slots, post-value counting) for traces of many PCs, whose windows alternate
  // keys; v1 (single-key runs, stage-batched dense gathers) for few PCs.  VE_K1=1 / 2 forces one.
  const char* kv = getenv("VE_K1");
  const bool v2 = ul || ((kv && *kv) ? *kv == '2' : c->cfg.n_pcs >= VE_MULTI_MIN_PCS);   // (units: v2 only)
  auto kfn = ul ? k_analyze2<true> : v2 ? k_analyze2<false> : multi ? k_analyze<true> : k_analyze<false>;
  cudaFuncGetAttributes(&fa, kfn);
  const size_t budget = (size_t)dev_smem - fa.sharedSizeBytes - 1024;   // dynamic smem left after the TMA ring
  // 2048 slots measured best on cfg2 / cfg3 / cfg4 (the HBM table behind it stays L2-resident)
  uint32_t hs = getenv("VE_HS") ? (uint32_t)atoi(getenv("VE_HS")) : 2048;
  while (hs > 256 && smem_bytes(sp + so, hs, P.objc) > budget) hs >>= 1;
  P.hs = hs;
  carve_offsets(P, sp + so);
  const size_t sb = smem_bytes(sp + so, hs, P.objc);
  // the attribute is per function, process-wide: set the device's maximum (every launch asks for
  // sb <= it), so contexts launching from several host threads never undercut each other
  cudaError_t e = cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       dev_smem - (int)fa.sharedSizeBytes);
  if (e != cudaSuccess) return cuda_fail(c, e, "cudaFuncSetAttribute(k_analyze)");
  if (n == 0) return VE_OK;
  uint64_t windows = (n + 31) / 32;
  uint64_t blocks = (windows + K1_WARPS - 1) / K1_WARPS;
  if (c->cfg.min_windows_per_warp) {   // throughput mode (several contexts side by side): fewer, fuller CTAs
    const uint64_t per = (uint64_t)c->cfg.min_windows_per_warp * (v2 ? K2_WARPS : K1_WARPS);
    blocks = (windows + per - 1) / per;
  }
  if (blocks > (uint64_t)c->num_sms) blocks = (uint64_t)c->num_sms;
  if (blocks == 0) blocks = 1;
  // a trace too short to give every warp a few CHUNK-window chunks (cfg5's kernels: a warp's
  // serial share of a 16-window chunk set a ~0.3 ms floor) is split into one-stage chunks
  P.chunk = ul ? UNIT_CHUNK : P.nring >= 4ull * blocks * K1_WARPS * CHUNK ? (v2 ? V2_CHUNK : CHUNK) : (uint32_t)STAGE_WIN;
  // v2 claims its chunks dynamically; v1 splits statically (VE_CLAIM_MODE=1: dynamic claims for v1)
  const char* cm = getenv("VE_CLAIM_MODE");
  P.claim = (ul || v2) ? 1u : (cm && *cm && *cm == '1') ? 1u : 0u;   // (v2: always dynamic)
  P.nbig = (P.nring - P.nring / 8) / P.chunk;
  // staging regions: a warp stages at most one group per record of its static range
  {
    const uint64_t tw = blocks * K1_WARPS;
    const uint64_t twa = blocks * (v2 ? K2_WARPS : K1_WARPS);   // warps that take windows
    const uint64_t per = 32 * ((windows + twa - 1) / twa + 2);
    P.stage_rs = (uint32_t)(per < STAGE_RS_MAX ? per : STAGE_RS_MAX);
    const size_t need = (size_t)tw * P.stage_rs * sizeof(uint4) + tw * sizeof(uint32_t);
    if (c->hstage_bytes < need) {
      c->hstage_bytes = 0;
      e = ctx_realloc(c, &c->hstage, need);
      if (e != cudaSuccess) return cuda_fail(c, e, "k_analyze staging");
      c->hstage_bytes = need;
    }
    P.stage = (uint4*)c->hstage;
    P.stage_cnt = (uint32_t*)((uint8_t*)c->hstage + (size_t)tw * P.stage_rs * sizeof(uint4));
  }
  if (P.claim) {
    e = cudaMemsetAsync(P.work, 0, sizeof(unsigned long long), s);
    if (e != cudaSuccess) return cuda_fail(c, e, "k_analyze claim counter");
  }
  count_launch();
  kfn<<<(unsigned)blocks, v2 ? K2_THREADS : K1_THREADS, sb, s>>>(P);
  e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "k_analyze launch");
  count_launch();
  k_hist_drain<<<(unsigned)(blocks * K1_WARPS), 256, 0, s>>>(P.stage, P.stage_cnt, P.stage_rs, P.t);
  e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "k_hist_drain launch");
  const uint32_t nsk = sp + so;
  count_launch();
  k_line_fold<<<nsk, LF_THREADS, 0, s>>>(c->t.lcta, (uint32_t)blocks, nsk, sp, c->cfg.n_pcs, c->t.line);
  e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "k_line_fold launch");
  return VE_OK;
}

ve_status launch_analyze(ve_ctx* c, const ve_record* d, uint64_t n, cudaStream_t s) {
  ctx_begin(c, s);   // after the ctx's earlier work (the last reset, a report), on any stream
  const ve_status st = launch_analyze_impl(c, d, n, s, nullptr);
  if (st == VE_OK) ctx_end(c, s);
  return st;
}

}  // namespace ve

using namespace ve;

// ve_analyze_units (include/ve.h): independent traces of the units set by ve_set_units in one launch
extern "C" ve_status ve_analyze_units(ve_ctx* c, const ve_unit* units, uint32_t n_units, cudaStream_t s) {
  if (!c || (n_units && !units)) return VE_ERR_INVALID;
  if (c->poisoned || c->hist_merged) return fail(c, VE_ERR_STATE, "ve_analyze_units: ctx poisoned or merged; ve_reset first");
  if (n_units != c->n_units || c->unit_obj.size() != (size_t)n_units + 1)
    return fail(c, VE_ERR_INVALID, "ve_analyze_units: n_units differs from the last ve_set_units");
  if (n_units == 0) return VE_OK;
  if (n_units > 65535) return fail(c, VE_ERR_INVALID, "ve_analyze_units: more than 65535 units");
  std::vector<UnitDesc> ud(n_units);
  std::vector<uint32_t> ucb(n_units + 1, 0);
  uint64_t ntot = 0, nring = 0;
  for (uint32_t u = 0; u < n_units; ++u) {
    const ve_unit& U = units[u];
    if (U.n && (!U.d_records || ((uintptr_t)U.d_records & 15)))
      return fail(c, VE_ERR_INVALID, "ve_analyze_units: unit records null or not 16-byte aligned");
    if ((uint64_t)U.pc_base + U.n_pcs > c->cfg.n_pcs)
      return fail(c, VE_ERR_INVALID, "ve_analyze_units: pc_base + n_pcs above the ctx's n_pcs");
    ud[u] = UnitDesc{U.d_records, U.n, U.pc_base, U.n_pcs, c->unit_obj[u], c->unit_obj[u + 1]};
    const uint64_t fw = U.n / 32, ch = (fw + UNIT_CHUNK - 1) / UNIT_CHUNK;
    if ((uint64_t)ucb[u] + ch > 0xFFFFFFFFull) return fail(c, VE_ERR_INVALID, "ve_analyze_units: batch too large");
    ucb[u + 1] = ucb[u] + (uint32_t)ch;
    ntot += U.n;
    nring += fw;
  }
  if (ntot == 0) return VE_OK;
  // per-CTA shared counters are 32-bit (see ve_analyze_records)
  if (ntot >= ((uint64_t)(c->num_sms > 0 ? c->num_sms : 1) << 31))
    return fail(c, VE_ERR_INVALID, "ve_analyze_units: batch above the per-launch record limit; split it");
  cudaSetDevice(c->device);
  ctx_begin(c, s);
  const size_t bytes = ud.size() * sizeof(UnitDesc) + ucb.size() * 4;
  void* d = nullptr;
  cudaError_t e = cudaMallocAsync(&d, bytes, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "ve_analyze_units alloc");
  std::vector<uint8_t> h(bytes);
  memcpy(h.data(), ud.data(), ud.size() * sizeof(UnitDesc));
  memcpy(h.data() + ud.size() * sizeof(UnitDesc), ucb.data(), ucb.size() * 4);
  cudaMemcpyAsync(d, h.data(), bytes, cudaMemcpyHostToDevice, s);   // (pageable: staged before return)
  UnitLaunch ul{(const UnitDesc*)d, (const uint32_t*)((uint8_t*)d + ud.size() * sizeof(UnitDesc)), n_units, nring};
  const ve_status st = launch_analyze_impl(c, nullptr, ntot, s, &ul);
  cudaFreeAsync(d, s);
  if (st == VE_OK) ctx_end(c, s);
  return st;
}
