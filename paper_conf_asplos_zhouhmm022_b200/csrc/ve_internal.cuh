// ve_internal.cuh -- shared internals of libve.so (device layout, record
// decoding, bit-level value tests).  Product code: includes nothing from
// oracle/ or gen/.
//
// Citations: P:L<n> = PAPER.md line n; C<k>/Q<k> = DESIGN.md section 3.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <cstdio>

#include <string>
#include <vector>

#include "ve.h"

namespace ve {

// ---- per-key statistic layout (SoA blocks, one NCCL call each) ------------
constexpr int NSUM = 24;  // 23 SUM fields + pad (C1, C2, C5)
enum : int {
  F_LD = 0, F_ST, F_ZERO, F_LDEQ, F_STEQ, F_NOSNAP,
  F_TYPE0 = 6,  // .. 17: n_type[12]
  F_NAN = 18, F_NONINT, F_NF16, F_NBF16, F_NF32, F_PAD
};
constexpr int NMM = 3;  // raw, ord, trunc  (min block and max block)
enum : int { M_RAW = 0, M_ORD = 1, M_TRUNC = 2 };

constexpr uint32_t EMPTY_TAG = 0xFFFFFFFFu;  // histogram slot free
constexpr uint32_t KO_NONE = 0xFFFFu;        // record maps to no object key
constexpr int WARP = 32;
constexpr uint32_t K1_NSK = 256;              // K1 keys with shared-memory rows (PCs first, then objects)

// line state of C8 / the (+) monoid of DESIGN.md 3.3; y is signed 128-bit
struct __align__(16) LineState {
  uint32_t state;  // VE_LINE_*
  uint32_t lock;   // spin lock for concurrent (+)
  uint64_t px, qx;
  uint64_t pylo;
  int64_t pyhi;
  uint64_t qylo;
  int64_t qyhi;
  uint64_t pad;
};
static_assert(sizeof(LineState) == 64, "LineState layout");

struct __align__(16) HSlot {  // exact histogram key: (pc, object key) tag + value bits
  uint64_t bits;
  uint32_t tag;
  uint32_t pad;
};

// ---- device views -----------------------------------------------------------
struct DevTables {
  unsigned long long* sum;  // [n_keys][NSUM]
  unsigned long long* mn;   // [n_keys][NMM]
  unsigned long long* mx;   // [n_keys][NMM]
  LineState* line;          // [n_keys]
  LineState* lcta;          // [grid][K1_NSK]: per-CTA line states of K1's shared keys, folded by K2
  unsigned long long* glob; // [8]: n_records, n_invalid, n_unmapped, overflow
  uint32_t* W;              // written-element bitmaps (all objects)
  uint32_t* L;              // eq_pre-load start-element bitmaps
  HSlot* hslot;             // [hcap]
  unsigned long long* hcount;  // [hcap]
  uint64_t hmask;           // hcap - 1
  uint32_t* occ_bm;         // [hcap / 32] occupancy bitmap: bit h set by the claim of slot h (a fire-and-
                            // forget RED.OR, nothing on the claim's critical path); null for temporary tables.
                            // The report and the reset walk it (hcap / 8 bytes) instead of the slots: O(entries
                            // + hcap / 32).  (Round 2's occupancy list took one returning atomic per claim on a
                            // shared counter: 0.42 ms of cfg2's 2.07 ms gemm epoch.)
};
__device__ __forceinline__ void occ_append(const DevTables& t, uint64_t h) {
  if (t.occ_bm) atomicOr(&t.occ_bm[h >> 5], 1u << (h & 31u));   // (result unused: compiled to RED)
}
enum : int { G_RECORDS = 0, G_INVALID = 1, G_UNMAPPED = 2, G_OVERFLOW = 3, G_WORK = 7 };  // 7: K1 chunk counter

struct DevObjects {          // sorted by base
  const uint64_t* base;
  const uint64_t* end;
  const uint32_t* id;
  const uint32_t* ew;
  const uint64_t* pre;       // device pointers as integers (0 = none)
  const uint64_t* post;      // post snapshot (0 = none)
  const uint64_t* bmoff;     // first bitmap word of the object
  // dense per-element access counters for loads that read the pre value: up to
  // DENSE_PER_OBJ arrays per object, each claimed by one (pc, access type):
  // dense_pc[D*i+j] = claim key, DENSE_FREE or DENSE_OFF; the claimer allocates the
  // array from the pool (bump cursor *dense_next) and publishes its first counter in
  // dense_off[D*i+j] (DENSE_NOT_READY until then, DENSE_NONE if the pool is full)
  uint32_t* dense_pc;
  unsigned long long* dense_off;
  uint32_t* dense_pool;
  unsigned long long* dense_next;
  uint64_t dense_cap;        // counters in the pool
  uint32_t n;
};
constexpr uint32_t DENSE_FREE = 0xFFFFFFFFu;
constexpr uint32_t DENSE_OFF = 0xFFFFFFFEu;
constexpr unsigned long long DENSE_NOT_READY = ~0ull;
constexpr unsigned long long DENSE_NONE = ~1ull;
constexpr int DENSE_PER_OBJ = 8;
// A claim key is meta << 16 | pc; DENSE_POST marks an array that counts records whose value equals the
// POST snapshot's element (records that read a value written earlier by the same API call, and stores
// of an element's final value): their histogram entry is that post value (K1 v2 claims these)
constexpr uint32_t DENSE_POST = 1u << 31;
constexpr int G_DENSE_NEXT = 4;   // glob slot of the dense pool cursor

// ---- host-side context ------------------------------------------------------
struct HostObject {
  uint64_t base, size;
  uint64_t pre, post;
  uint32_t id, ew;
  uint64_t n_elems, bmoff, bmwords;
};

}  // namespace ve

struct ve_ctx {
  ve_config cfg;
  int device;
  int num_sms;
  std::string err;
  bool poisoned = false;
  bool hist_merged = false;  // set by an NCCL merge: top-k/n_distinct precomputed
  bool table_clean = false;  // the value table holds only the slots marked in t.occ_bm (else: full clear)
  // Stream order of the ctx's work (no device-wide synchronisation anywhere): every call that
  // touches the ctx's device state waits for ord_ev on its stream first and records ord_ev there
  // after its last launch (ctx_begin / ctx_end), so the ctx's calls run in call order whatever
  // streams they use; ctx-internal work (resets, the report) runs on the ctx's own stream cs.
  cudaEvent_t ord_ev = nullptr;
  cudaStream_t cs = nullptr;
  uint32_t n_obj = 0;
  uint32_t n_keys = 0;
  std::vector<ve::HostObject> objs;          // sorted by base
  std::vector<uint32_t> sorted_of_id;        // id -> index in objs
  uint32_t n_units = 1;                      // ve_set_units: independent units (ve_set_objects: one)
  std::vector<uint32_t> unit_obj;            // [n_units + 1]: unit u's objects are objs[unit_obj[u] .. unit_obj[u+1])
  // device memory
  ve::DevTables t{};
  ve::DevObjects o{};
  void* obj_block = nullptr;                 // backing store of DevObjects arrays
  size_t obj_block_bytes = 0;
  uint64_t bm_words = 0;
  uint64_t bm_cap = 0;                       // words allocated for W and L
  uint64_t hcap = 0;
  // dense counters (see DevObjects); disabled once 2^32 records could overflow a u32 counter
  void* dense_pool = nullptr;
  uint64_t dense_cap = 0;                    // counters allocated
  uint64_t dense_want = 0;                   // counters the current object set may claim (0: none)
  bool dense_dirty = false;                  // pool may hold counts not yet flushed
  std::vector<uint32_t> dense_pc_init;       // [DENSE_PER_OBJ*n_obj]: DENSE_FREE or DENSE_OFF
  uint64_t records_analyzed = 0;
  uint64_t pre_elems = 0;                    // elements of the objects with a pre snapshot
  // finalize scratch
  void* scratch = nullptr;
  void* pin = nullptr;                       // pinned host staging of small report-time copies
  void* rpin = nullptr;                      // pinned staging of the report's table copies
  size_t rpin_bytes = 0;
  size_t scratch_bytes = 0;
  void* occ_flat = nullptr;                  // the report's list of occupied slots (+ its length)
  size_t occ_flat_bytes = 0;
  uint64_t last_nocc = 0;                    // occupied value-table slots at the last report
  // merged histogram results (NCCL path)
  std::vector<uint64_t> merged_ndistinct;
  std::vector<ve_topk_entry> merged_topk;
  // host staging for ve_analyze_records_host
  void* stage[2] = {nullptr, nullptr};
  cudaEvent_t stage_ev[2] = {nullptr, nullptr};
  cudaEvent_t copied_ev[2] = {nullptr, nullptr};
  cudaStream_t copy_stream = nullptr;        // H2D of the staging buffers, overlapped with analysis
  size_t stage_bytes = 0;
  // K1's S8 insert staging (k_hist_drain)
  void* hstage = nullptr;
  size_t hstage_bytes = 0;
};

struct ve_rep {
  uint32_t n_keys, n_obj, topk;
  std::vector<ve_key_stats> keys;
  std::vector<ve_topk_entry> top;
  std::vector<ve_obj_stats> objs;
  ve_globals glob;
};

// ---- internal entry points (one .cu each) ----------------------------------
namespace ve {
ve_status fail(ve_ctx* c, ve_status s, const std::string& msg);
ve_status cuda_fail(ve_ctx* c, cudaError_t e, const char* where);
ve_status launch_analyze(ve_ctx* c, const ve_record* d, uint64_t n, cudaStream_t s);
ve_status launch_reset(ve_ctx* c, cudaStream_t s);
void ctx_begin(ve_ctx* c, cudaStream_t s);      // order s after the ctx's earlier work
void ctx_end(ve_ctx* c, cudaStream_t s);        // the ctx's work so far ends with s's queued work
cudaError_t ctx_quiesce(ve_ctx* c);             // host wait for the ctx's queued work (not the device's)
bool dense_reserve(ve_ctx* c);                  // the dense counter pool for the current object set
cudaError_t ctx_realloc(ve_ctx* c, void** p, size_t bytes);   // grow a ctx buffer without a device sync
ve_status finalize_hist(ve_ctx* c, cudaStream_t s, std::vector<uint64_t>& ndistinct,
                        std::vector<ve_topk_entry>& top);
ve_status bitmap_counts(ve_ctx* c, cudaStream_t s, std::vector<ve_obj_stats>& out);
ve_status run_diff(ve_ctx* c, uint32_t obj_index, uint32_t mode, const uint32_t* d_mask, ve_diff* out,
                   cudaStream_t s);
ve_status run_dedup(ve_ctx* c, const ve_object* objs, uint32_t n, uint32_t* group_of, cudaStream_t s);
ve_status merge_local(ve_ctx* dst, const ve_ctx* src, cudaStream_t s);
// ---- rank transports (nccl_merge.cu: NCCL, and same-device simulated ranks) ----
enum { OP_SUM = 0, OP_MIN = 1, OP_MAX = 2 };
struct Comm {
  int G = 1;                      // number of ranks
  std::vector<int> local;         // global rank of each local context
  std::string err;
  virtual ~Comm() {}
  // u64 in-place allreduce of count elements in bufs[i] (one per local rank)
  virtual bool allreduce(const std::vector<void*>& bufs, size_t count, int op, cudaStream_t s) = 0;
  // recv[i] receives G blocks of bytes, block g from global rank g
  virtual bool allgather(const std::vector<const void*>& send, const std::vector<void*>& recv, size_t bytes,
                         cudaStream_t s) = 0;
  // send[i] + soff[i][g] (sbytes[i][g]) goes to rank g; recv[i] + roff[i][g] gets rbytes[i][g] from rank g
  virtual bool alltoallv(const std::vector<const uint8_t*>& send, const std::vector<std::vector<size_t>>& soff,
                         const std::vector<std::vector<size_t>>& sbytes, const std::vector<uint8_t*>& recv,
                         const std::vector<std::vector<size_t>>& roff, const std::vector<std::vector<size_t>>& rbytes,
                         cudaStream_t s) = 0;
};
struct LocalComm : Comm {        // one rank: every exchange is the identity
  LocalComm() { G = 1; local = {0}; }
  bool allreduce(const std::vector<void*>&, size_t, int, cudaStream_t) override { return true; }
  bool allgather(const std::vector<const void*>& send, const std::vector<void*>& recv, size_t bytes,
                 cudaStream_t s) override {
    return !bytes || cudaMemcpyAsync(recv[0], send[0], bytes, cudaMemcpyDeviceToDevice, s) == cudaSuccess;
  }
  bool alltoallv(const std::vector<const uint8_t*>&, const std::vector<std::vector<size_t>>&,
                 const std::vector<std::vector<size_t>>&, const std::vector<uint8_t*>&,
                 const std::vector<std::vector<size_t>>&, const std::vector<std::vector<size_t>>&,
                 cudaStream_t) override { return false; }
};
// S11 / S10 sharded by object over the ranks of comm (cs: one context per local rank): the owner
// rank of object k (position k of the eligible list, k mod G) hashes / diffs it, candidate pairs
// are verified by rank (pair index mod G), and the partial results are allreduced -- every rank
// ends with the same full result.  One rank (LocalComm) is the plain call.
ve_status dedup_ranks(const std::vector<ve_ctx*>& cs, Comm& comm, const ve_object* objs, uint32_t n,
                      uint32_t* group_of, cudaStream_t s);
ve_status diff_ranks(const std::vector<ve_ctx*>& cs, Comm& comm, uint32_t mode, ve_diff* out_by_id, cudaStream_t s);
ve_status merge_nccl(ve_ctx* c, void* comm, cudaStream_t s);
ve_status dense_flush(ve_ctx* c, cudaStream_t s);  // move dense counts into the exact histogram
ve_status approx_topk(ve_ctx* c, cudaStream_t s, const std::vector<uint8_t>& akind, std::vector<uint64_t>& ndistinct,
                      std::vector<ve_topk_entry>& top);
struct ViewTable {                                 // per-key (PC view, object view) value counts
  HSlot* vs = nullptr;
  unsigned long long* vc = nullptr;
  uint64_t vcap = 0;
};
ve_status build_views(ve_ctx* c, cudaStream_t s, ViewTable& V);
ve_status alloc_views(ve_ctx* c, cudaStream_t s, uint64_t n, ViewTable& V);
void free_views(ViewTable& V, cudaStream_t s);
ve_status view_topk(ve_ctx* c, const ViewTable& V, cudaStream_t s, std::vector<uint64_t>& ndistinct,
                    std::vector<ve_topk_entry>& top);
void count_launch();  // process-wide kernel launch counter (ve_kernel_launches)
size_t sort_scratch_bytes(uint64_t m);              // k_interval.cu: stable LSD radix sort of u64 pairs
ve_status sort_pairs(ve_ctx* c, uint64_t*& S, uint64_t*& E, uint64_t*& S2, uint64_t*& E2, uint64_t m, uint8_t* scr,
                     cudaStream_t s);
}  // namespace ve

// ============================================================================
// Device helpers: record decoding and bit-level value tests.  Everything is
// integer arithmetic on bit patterns (no FP arithmetic result is
// ever compared), written from the definitions, independent of the oracle.
// ============================================================================
namespace ve {

__device__ __forceinline__ uint32_t meta_lg(uint32_t m) { return m & 3u; }
__device__ __forceinline__ uint32_t meta_kind(uint32_t m) { return (m >> 2) & 3u; }
__device__ __forceinline__ bool meta_store(uint32_t m) { return (m >> 4) & 1u; }
__device__ __forceinline__ bool meta_shared(uint32_t m) { return (m >> 5) & 1u; }

// record validity (DESIGN.md 3.1 / include/ve.h)
__device__ __forceinline__ bool rec_valid(uint64_t addr, uint64_t value, uint32_t pc, uint32_t meta,
                                          uint32_t n_pcs) {
  uint32_t lg = meta & 3u, kind = (meta >> 2) & 3u;
  bool ok = (meta >> 6) == 0u;
  ok &= !(kind == 2u && lg == 0u);
  ok &= !(kind == 3u && lg != 1u);
  ok &= pc < n_pcs;
  ok &= (lg == 3u) || (value >> (8u << lg)) == 0ull;
  ok &= addr < (1ull << 48);
  return ok;
}

// type code u8 u16 u32 u64 i8 i16 i32 i64 f16 f32 f64 bf16 (C1)
__device__ __forceinline__ uint32_t type_code(uint32_t kind, uint32_t lg) {
  return kind == 0u ? lg : kind == 1u ? 4u + lg : kind == 3u ? 11u : 7u + lg;
}

// IEEE layout of a float record: exponent bits, mantissa bits
__device__ __forceinline__ void float_layout(uint32_t kind, uint32_t lg, int& eb, int& mb) {
  if (kind == 3u) { eb = 8; mb = 7; }
  else if (lg == 1u) { eb = 5; mb = 10; }
  else if (lg == 2u) { eb = 8; mb = 23; }
  else { eb = 11; mb = 52; }
}

// C5 orderable key
__device__ __forceinline__ uint64_t ord_key(uint64_t b, uint32_t kind, uint32_t lg) {
  if (kind == 0u) return b;
  uint32_t nb = 8u << lg;
  if (kind == 1u) {
    uint32_t sh = 64u - nb;
    int64_t s = (int64_t)(b << sh) >> sh;
    return (uint64_t)s ^ (1ull << 63);
  }
  uint64_t mask = (nb == 64u) ? ~0ull : ((1ull << nb) - 1ull);
  uint64_t sign = 1ull << (nb - 1u);
  return (b & sign) ? (~b & mask) : (b | sign);
}

// Is the exact value sig * 2^ex (sig > 0) representable in a binary format
// with eb exponent / mb mantissa bits?  (round trip through it is the identity)
__device__ __forceinline__ bool representable(uint64_t sig, int ex, int eb, int mb) {
  int tz = __ffsll((long long)sig) - 1;
  sig >>= tz;
  ex += tz;
  int nbits = 64 - __clzll((long long)sig);
  int top = ex + nbits - 1;             // exponent of the leading bit
  int bias = (1 << (eb - 1)) - 1;
  int emin = 1 - bias;
  if (top > bias) return false;         // overflow
  int lowest = (top >= emin) ? (top - mb) : (emin - mb);
  return ex >= lowest && ex >= emin - mb;
}

// C5 float flags: bit0 NaN, bit1 nonint, bit2 not_f16, bit3 not_bf16, bit4 not_f32
// (f64 only).  Also returns the exact integer value when nonint is clear.
__device__ __forceinline__ uint32_t float_flags(uint64_t b, uint32_t kind, uint32_t lg, int64_t& ival) {
  int eb, mb;
  float_layout(kind, lg, eb, mb);
  uint32_t nb = 8u << lg;
  bool is_f64 = (kind == 2u && lg == 3u);
  uint64_t emax = (1ull << eb) - 1ull;
  bool sign = (b >> (nb - 1u)) & 1ull;
  uint64_t E = (b >> mb) & emax;
  uint64_t M = b & ((1ull << mb) - 1ull);
  ival = 0;
  if (E == emax) {
    if (M != 0ull) return 1u | 2u | 4u | 8u | (is_f64 ? 16u : 0u);  // NaN fails everything
    return 2u;                                                           // +-Inf: nonint only
  }
  uint64_t sig = (E == 0ull) ? M : (M | (1ull << mb));
  int ex = (E == 0ull ? 1 : (int)E) - ((1 << (eb - 1)) - 1) - mb;
  if (sig == 0ull) return sign ? 2u : 0u;                                // -0.0 is nonint
  // value = sig * 2^ex; its set bits span exponents [low, top]
  const int low = ex + __ffsll((long long)sig) - 1;
  const int top = ex + 63 - __clzll((long long)sig);
  uint32_t f = 0;
  if (top >= 63 || low < 0) {
    f |= 2u;                                                             // |v| >= 2^63 or a fraction
  } else {
    const uint64_t mag = (ex >= 0) ? (sig << ex) : (sig >> -ex);
    ival = sign ? -(int64_t)mag : (int64_t)mag;
  }
  // representable in a format with bias B and m mantissa bits <=> top <= B and
  // low >= max(top - m, 1 - B - m)  (round trip through it is then the identity)
  if (!(top <= 15 && low >= max(top - 10, -24))) f |= 4u;               // binary16
  if (!(top <= 127 && low >= max(top - 7, -133))) f |= 8u;              // bfloat16
  if (is_f64 && !(top <= 127 && low >= max(top - 23, -149))) f |= 16u;  // binary32
  return f;
}

// float_flags of an IEEE binary32 value in closed form (same results as
// float_flags(b, 2, 2, .) for every bit pattern; checked exhaustively by
// scripts/check_fflags.cu).  E = exponent field, tz = trailing zeros of the
// significand with its implicit bit: the value is sig * 2^(E-150), its lowest set
// bit has exponent E-150+tz and its leading bit E-127, so
//   integer           <=> E + tz >= 150 and E <= 189 (|v| < 2^63)
//   binary16 exact    <=> E <= 142, tz >= 13, E + tz >= 126 (normal or subnormal f16)
//   bfloat16 exact    <=> the low 16 bits are zero (same exponent range as binary32)
__device__ __forceinline__ uint32_t fflags_f32(uint32_t b) {
  const uint32_t E = (b >> 23) & 0xFFu, M = b & 0x7FFFFFu;
  const uint32_t tz = (uint32_t)__ffs((int)(M | 0x800000u)) - 1u;
  const uint32_t t = E + tz;
  const bool special = E == 0xFFu;                        // Inf or NaN
  uint32_t f = (b != 0u && !(t >= 150u && E <= 189u)) ? 2u : 0u;
  if (!((b << 1) == 0u || (special && M == 0u) || (E <= 142u && tz >= 13u && t >= 126u))) f |= 4u;
  if (b & 0xFFFFu) f |= 8u;
  return (special && M != 0u) ? 15u : f;                  // NaN fails everything
}

// C7 mantissa truncation
__device__ __forceinline__ uint64_t trunc_bits(uint64_t b, uint32_t kind, uint32_t lg, uint32_t K) {
  uint32_t m = kind == 3u ? 7u : lg == 1u ? 10u : lg == 2u ? 23u : 52u;
  if (K >= m) return b;
  return b & ~((1ull << (m - K)) - 1ull);
}

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z ^= z >> 33;
  z *= 0xff51afd7ed558ccdull;
  z ^= z >> 33;
  z *= 0xc4ceb9fe1a85ec53ull;
  z ^= z >> 33;
  return z;
}
__device__ __forceinline__ uint64_t hist_hash(uint32_t tag, uint64_t bits) {
  return mix64(bits ^ ((uint64_t)tag * 0x9E3779B97F4A7C15ull));
}

// 128-bit CAS (sm_90+): returns the old value
__device__ __forceinline__ void cas128_global(void* p, uint64_t elo, uint64_t ehi, uint64_t nlo, uint64_t nhi,
                                              uint64_t& olo, uint64_t& ohi) {
  asm volatile(
      "{\n\t.reg .b128 e, n, o;\n\t"
      "mov.b128 e, {%2, %3};\n\tmov.b128 n, {%4, %5};\n\t"
      "atom.relaxed.gpu.global.cas.b128 o, [%6], e, n;\n\t"
      "mov.b128 {%0, %1}, o;\n\t}"
      : "=l"(olo), "=l"(ohi)
      : "l"(elo), "l"(ehi), "l"(nlo), "l"(nhi), "l"(p)
      : "memory");
}
__device__ __forceinline__ void cas128_shared(void* p, uint64_t elo, uint64_t ehi, uint64_t nlo, uint64_t nhi,
                                              uint64_t& olo, uint64_t& ohi) {
  uint32_t a = (uint32_t)__cvta_generic_to_shared(p);
  asm volatile(
      "{\n\t.reg .b128 e, n, o;\n\t"
      "mov.b128 e, {%2, %3};\n\tmov.b128 n, {%4, %5};\n\t"
      "atom.relaxed.cta.shared.cas.b128 o, [%6], e, n;\n\t"
      "mov.b128 {%0, %1}, o;\n\t}"
      : "=l"(olo), "=l"(ohi)
      : "l"(elo), "l"(ehi), "l"(nlo), "l"(nhi), "r"(a)
      : "memory");
}
__device__ __forceinline__ void ld128_volatile(const void* p, uint64_t& lo, uint64_t& hi) {
  asm volatile("ld.volatile.global.v2.u64 {%0, %1}, [%2];" : "=l"(lo), "=l"(hi) : "l"(p));
}

// Insert (tag, bits) += cnt into the global exact histogram; false on overflow.
// CAS first (an empty slot is all-ones; an occupied one has pad 0): one L2 round
// trip claims a free slot or returns the occupant, so a probe never needs a
// separate read; the count update is a fire-and-forget reduction.
__device__ __forceinline__ bool hist_insert_global(const DevTables& t, uint32_t tag, uint64_t bits,
                                                   unsigned long long cnt) {
  uint64_t h = hist_hash(tag, bits) & t.hmask;
  for (uint64_t probe = 0; probe <= t.hmask; ++probe) {
    HSlot* s = &t.hslot[h];
    uint64_t olo, ohi;
    cas128_global(s, ~0ull, ~0ull, bits, (uint64_t)tag, olo, ohi);
    if (olo == ~0ull && ohi == ~0ull) {          // claimed: record the slot
      occ_append(t, h);
      atomicAdd(&t.hcount[h], cnt);
      return true;
    }
    if (olo == bits && ohi == (uint64_t)tag) {
      atomicAdd(&t.hcount[h], cnt);
      return true;
    }
    h = (h + 1) & t.hmask;
  }
  atomicExch(&t.glob[G_OVERFLOW], 1ull);
  return false;
}

// Read-first insert for hit-heavy callers (report-time flushes, the K1 drain): a plain
// 16-byte load finds an existing entry with one atomic (the count add) instead of two.
// Slots go from empty to their final (bits, tag) once, by CAS, so a load whose low word is
// neither empty nor `bits` proves another key (skip); any other observation (a possibly
// torn read of a slot being claimed) is settled by the CAS itself.
#ifndef VE_READ_FIRST
#define VE_READ_FIRST 1
#endif
__device__ __forceinline__ bool hist_insert_global_rf(const DevTables& t, uint32_t tag, uint64_t bits,
                                                      unsigned long long cnt) {
#if VE_READ_FIRST
  uint64_t h = hist_hash(tag, bits) & t.hmask;
  for (uint64_t probe = 0; probe <= t.hmask; ++probe) {
    HSlot* s = &t.hslot[h];
    uint64_t lo, hi;
    asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(lo), "=l"(hi) : "l"(s) : "memory");
    if (lo == bits && hi == (uint64_t)tag && bits != ~0ull) {   // (value ~0: confirmed by the CAS below)
      atomicAdd(&t.hcount[h], cnt);
      return true;
    }
    if (lo == ~0ull || lo == bits) {
      uint64_t olo, ohi;
      cas128_global(s, ~0ull, ~0ull, bits, (uint64_t)tag, olo, ohi);
      if (olo == ~0ull && ohi == ~0ull) {        // claimed: record the slot
        occ_append(t, h);
        atomicAdd(&t.hcount[h], cnt);
        return true;
      }
      if (olo == bits && ohi == (uint64_t)tag) {
        atomicAdd(&t.hcount[h], cnt);
        return true;
      }
    }
    h = (h + 1) & t.hmask;
  }
  atomicExch(&t.glob[G_OVERFLOW], 1ull);
  return false;
#else
  return hist_insert_global(t, tag, bits, cnt);
#endif
}

// ---- line-state monoid (+) --------------------------------
__device__ __forceinline__ __int128 mk128(uint64_t lo, int64_t hi) {
  return (__int128)(((unsigned __int128)(uint64_t)hi << 64) | lo);
}
__device__ __forceinline__ bool collinear(uint64_t px, __int128 py, uint64_t qx, __int128 qy, uint64_t x,
                                          __int128 y) {
  // (y - py)(qx - px) == (qy - py)(x - px); |dy| < 2^66, |dx| < 2^48
  __int128 dxq = (__int128)((int64_t)(qx - px));
  __int128 dx = (__int128)((int64_t)(x - px));
  return (y - py) * dxq == (qy - py) * dx;
}

struct LinePts {
  uint32_t state;
  uint64_t px, qx;
  __int128 py, qy;
};

__device__ __forceinline__ LinePts line_load(const LineState& s) {
  LinePts r;
  r.state = s.state;
  r.px = s.px; r.qx = s.qx;
  r.py = mk128(s.pylo, s.pyhi);
  r.qy = mk128(s.qylo, s.qyhi);
  return r;
}
__device__ __forceinline__ void line_store(LineState& s, const LinePts& r) {
  s.px = r.px; s.qx = r.qx;
  s.pylo = (uint64_t)r.py; s.pyhi = (int64_t)(r.py >> 64);
  s.qylo = (uint64_t)r.qy; s.qyhi = (int64_t)(r.qy >> 64);
  s.state = r.state;
}

// a (+) b ; EMPTY identity, FAIL absorbing; result depends only on the point set
__device__ __forceinline__ LinePts line_merge(LinePts a, const LinePts& b) {
  if (b.state == VE_LINE_EMPTY || a.state == VE_LINE_FAIL) return a;
  if (a.state == VE_LINE_EMPTY || b.state == VE_LINE_FAIL) return b;
  // both POINT or LINE: a has extreme points p (min x), q (max x); same for b
  LinePts r;
  if (a.state == VE_LINE_POINT && b.state == VE_LINE_POINT) {
    if (a.px == b.px) {
      r = a;
      if (a.py != b.py) r.state = VE_LINE_FAIL;
      return r;
    }
    r.state = VE_LINE_LINE;
    if (a.px < b.px) { r.px = a.px; r.py = a.py; r.qx = b.px; r.qy = b.py; }
    else { r.px = b.px; r.py = b.py; r.qx = a.px; r.qy = a.py; }
    return r;
  }
  // at least one LINE: use it as the reference line, test the other's points
  const LinePts& L = (a.state == VE_LINE_LINE) ? a : b;
  const LinePts& O = (a.state == VE_LINE_LINE) ? b : a;
  bool ok = collinear(L.px, L.py, L.qx, L.qy, O.px, O.py);
  if (O.state == VE_LINE_LINE) ok = ok && collinear(L.px, L.py, L.qx, L.qy, O.qx, O.qy);
  if (!ok) { r = a; r.state = VE_LINE_FAIL; return r; }
  r.state = VE_LINE_LINE;
  if (O.px < L.px) { r.px = O.px; r.py = O.py; } else { r.px = L.px; r.py = L.py; }
  uint64_t oqx = (O.state == VE_LINE_LINE) ? O.qx : O.px;
  __int128 oqy = (O.state == VE_LINE_LINE) ? O.qy : O.py;
  if (oqx > L.qx) { r.qx = oqx; r.qy = oqy; } else { r.qx = L.qx; r.qy = L.qy; }
  return r;
}

// merge b into *s under the state's spin lock (global or shared)
__device__ __forceinline__ void line_merge_locked(LineState* s, const LinePts& b) {
  if (b.state == VE_LINE_EMPTY) return;
  uint32_t spins = 0;
  while (atomicCAS(&s->lock, 0u, 1u) != 0u) {
    __nanosleep(20);
    if (++spins == (1u << 26)) {  // a lost lock is a bug: fail loudly instead of hanging
      printf("libve: line-state lock %p stuck (state %u lock %u) block %d thread %d\n", (void*)s, s->state, s->lock,
             blockIdx.x, threadIdx.x);
      __trap();
    }
  }
  __threadfence();
  volatile LineState* vs = s;
  LinePts a;
  a.state = vs->state;
  a.px = vs->px; a.qx = vs->qx;
  a.py = mk128(vs->pylo, vs->pyhi);
  a.qy = mk128(vs->qylo, vs->qyhi);
  LinePts r = line_merge(a, b);
  vs->px = r.px; vs->qx = r.qx;
  vs->pylo = (uint64_t)r.py; vs->pyhi = (int64_t)(r.py >> 64);
  vs->qylo = (uint64_t)r.qy; vs->qyhi = (int64_t)(r.qy >> 64);
  vs->state = r.state;
  __threadfence();
  atomicExch(&s->lock, 0u);
}

}  // namespace ve
