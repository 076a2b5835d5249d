/*
 * ve.h -- C ABI of libve.so: B200-native ValueExpert value-trace analysis.
 *
 * The boundary of the hot path of Zhou et al., "ValueExpert: Exploring Value
 * Patterns in GPU-Accelerated Applications", ASPLOS '22.  Citations
 * P:L<n> are PAPER.md line numbers; C<k>/Q<k> are the definitions / readings
 * restated in DESIGN.md section 3.
 *
 * Conventions for every call:
 *   - All integers little-endian.  No C++ types cross the ABI.
 *   - Pointers named d_* are DEVICE pointers (caller-owned, on the ctx's
 *     device, valid until the work queued on the stream completes; the library
 *     never writes or frees them).  Pointers named h_* or plain arrays are HOST
 *     memory, copied before the call returns unless stated otherwise.
 *   - Every call returns ve_status; nothing throws or aborts across the ABI.
 *     ve_last_error(ctx) describes the last failure (cudaGetErrorString for
 *     CUDA errors).  Asynchronous kernel faults surface at the next
 *     synchronising call (ve_snapshot_diff, ve_object_dedup, ve_report).
 *   - A ctx is bound to one CUDA device and is not thread-safe; different
 *     contexts may be driven from different host threads at once.
 *   - Stream order, no device-wide synchronisation: a ctx's calls run in call
 *     order whatever streams they are given (each waits for the ctx's previous
 *     work through a per-ctx event); calls that return host results wait only
 *     for that ctx's work (its event / its own internal stream), never for the
 *     device, so other contexts and application streams keep running.
 */
#ifndef VE_H
#define VE_H
#include <stdint.h>
#include <cuda_runtime_api.h>   /* cudaStream_t only */

#ifdef __cplusplus
extern "C" {
#endif

/* One value-trace record: the (PC, address, size, raw value) the paper's
 * collector emits per thread per memory instruction, plus the access
 * type its offline analyzer derives.  24 bytes, alignment 8,
 * arrays are AoS.  Vector accesses (STG.64 = 2 x f32) are split by the
 * producer into one record per value at consecutive addresses (Q16). */
typedef struct ve_record {
  uint64_t addr;   /* effective byte address; >= 2^48 => invalid record            */
  uint64_t value;  /* raw bits of ONE value, zero-extended from w bytes; bits >= 8w */
                   /* must be 0 (else invalid)                                      */
  uint32_t pc;     /* dense PC id; >= cfg.n_pcs => invalid                          */
  uint32_t meta;   /* [1:0] log2 w (w in 1,2,4,8)                                   */
                   /* [3:2] kind: 0 uint, 1 sint, 2 IEEE float (w 2/4/8), 3 bf16 (w 2) */
                   /* [4] store   [5] shared space   [31:6] must be 0               */
} ve_record;

/* A data object: address range + pre/post snapshots of one GPU API. */
typedef struct ve_object {
  uint64_t base, size;     /* [base, base+size), size > 0, base+size <= 2^48, no overlaps */
  const void* pre;         /* device ptr: snapshot before the API (size bytes) or NULL     */
  const void* post;        /* device ptr: snapshot after the API (size bytes) or NULL      */
  uint32_t id;             /* dense: the n objects of one call carry ids 0..n-1            */
  uint32_t elem_width;     /* 1,2,4,8: granularity of bitmaps and of the diff (Q4)         */
} ve_object;

typedef struct ve_config {
  uint32_t n_pcs;           /* 1..65535                                                   */
  uint32_t max_objects;     /* <= 65534; SHARED pseudo-object key = n_pcs + n_objects     */
  uint32_t topk;            /* 1..64, default 8 (Q18)                                     */
  uint32_t mant_bits;       /* K of Def 3.8, default 7 (Q6)                               */
  uint32_t t_redundant_pct; /* default 33 (footnote P:L267)                               */
  uint32_t t_frequent_pct;  /* default 33 (Q2)                                            */
  uint64_t hist_capacity;   /* exact value-histogram slots (rounded up to 2^k); overflow  */
                            /* => VE_ERR_CAPACITY, never silently wrong stats              */
  uint32_t min_windows_per_warp; /* 0 = every analysis launch spans all SMs; k > 0: a short */
                            /* trace gets only the CTAs that give each warp >= k 32-record  */
                            /* windows, so contexts analysing small traces on several        */
                            /* streams run side by side (throughput over latency)            */
  uint32_t reserved;        /* 0                                                         */
} ve_config;

typedef enum {
  VE_OK = 0, VE_ERR_INVALID = 1, VE_ERR_CUDA = 2, VE_ERR_NOMEM = 3,
  VE_ERR_CAPACITY = 4, VE_ERR_NCCL = 5, VE_ERR_STATE = 6
} ve_status;

enum { VE_DIFF_WRITTEN = 0, VE_DIFF_ALL = 1, VE_DIFF_MASK = 2 };
enum { VE_LINE_EMPTY = 0, VE_LINE_POINT = 1, VE_LINE_LINE = 2, VE_LINE_FAIL = 3 };

typedef struct ve_ctx ve_ctx;
typedef struct ve_rep ve_rep;         /* host report, library-owned */

/* C10 result of ve_snapshot_diff. */
typedef struct ve_diff {
  uint64_t n_elems, n_masked, n_unchanged, n_changed, n_untouched;
  uint32_t redundant;      /* n_masked > 0 && 100*n_unchanged > t_redundant_pct*n_masked */
  uint32_t pad;
} ve_diff;

/* Per-key statistics (key index: PCs [0,n_pcs), object id -> n_pcs+id, SHARED
 * n_pcs+n_objects).  Raw fields are the parity target; derived flags are
 * recomputed from them. */
typedef struct ve_key_stats {
  uint64_t n_ld, n_st, n_zero, n_ld_eq_pre, n_st_eq_pre, n_nosnap;     /* C1, C2 */
  uint64_t n_type[12];          /* u8 u16 u32 u64 i8 i16 i32 i64 f16 f32 f64 bf16  */
  uint64_t n_nan, n_nonint, n_not_f16, n_not_bf16, n_not_f32;          /* C5 */
  uint64_t raw_min, raw_max, ord_min, ord_max, trunc_min, trunc_max;   /* C4 C5 C7 */
  uint64_t line_state;          /* VE_LINE_*                                  C8 */
  uint64_t p_x, p_ylo; int64_t p_yhi;   /* min-x end point, y as signed 128 bit */
  uint64_t q_x, q_ylo; int64_t q_yhi;   /* max-x end point                      */
  uint64_t n_distinct, n_top;   /* C9 */
  uint32_t single_value, single_zero, frequent, structured, approx, dict8;
  uint32_t heavy;               /* type code of the narrowest type, 255 = none (C6) */
  uint32_t single_type;
} ve_key_stats;

typedef struct ve_topk_entry { uint64_t bits, count; } ve_topk_entry;

typedef struct ve_obj_stats {
  uint64_t n_elems, n_written, n_loaded_eq, n_ld_reload, n_touched;    /* C3, C10 */
} ve_obj_stats;

typedef struct ve_globals {
  uint64_t n_records, n_invalid, n_unmapped;
  uint64_t hist_entries;        /* occupied slots of the device value table after the report's
                                   dense flush (implementation statistic, not a parity field;
                                   0 after a rank merge) */
} ve_globals;

/* ---- lifecycle ----------------------------------------------------------- */
ve_status   ve_create(const ve_config* cfg, int cuda_device, ve_ctx** out);
ve_status   ve_destroy(ve_ctx* ctx);
const char* ve_last_error(const ve_ctx* ctx);   /* valid until the next call on ctx */
/* Host array of n objects (device snapshot pointers) is copied, sorted and
 * validated (VE_ERR_INVALID on overlap, bad id/size/width); resets all stats. */
ve_status   ve_set_objects(ve_ctx* ctx, const ve_object* objs, uint32_t n);
ve_status   ve_reset(ve_ctx* ctx);              /* zero all statistics, clear poison */

/* ---- the five hot-path calls --------------------------------------------- */

/* S1-S9: analyze n device records (C1-C9, C3 bitmaps), accumulating into the
 * ctx; may be called repeatedly on chunks of one trace (the paper's buffer
 * flushes).  d_records must be 8-byte aligned.  Asynchronous
 * on s.  VE_ERR_STATE if the ctx is poisoned (histogram overflow). */
ve_status ve_analyze_records(ve_ctx* ctx, const ve_record* d_records, uint64_t n, cudaStream_t s);

/* Several independent traces in one launch (units): cfg5's thousands of small
 * kernels (the paper's whole-application runs, P:L105,
 * Table 5) pay one launch and one report instead of one each.  ve_set_units
 * takes the objects of n_units units, unit u being the next unit_nobj[u]
 * entries of objs (ids 0..n-1 over the whole set, so each unit's objects have
 * their own keys n_pcs + id); objects may overlap across units, not within one
 * (the units' address spaces are separate).  Errors as ve_set_objects, plus
 * VE_ERR_INVALID when the counts do not sum to n or n_units is 0 or > 65535. */
ve_status ve_set_units(ve_ctx* ctx, const ve_object* objs, uint32_t n, const uint32_t* unit_nobj, uint32_t n_units);

/* Unit u's device records (16-byte aligned); its record pc p < n_pcs is key
 * pc_base + p of the ctx (pc_base + n_pcs <= cfg.n_pcs), p >= n_pcs is invalid;
 * its addresses map to its own objects only (an address outside them is
 * unmapped).  The result equals analysing each unit alone with its PCs shifted
 * to pc_base (C12); the SHARED key and the globals add over the units. */
typedef struct ve_unit {
  const ve_record* d_records;
  uint64_t n;
  uint32_t pc_base, n_pcs;
} ve_unit;
/* All units in one launch (K1 v2), accumulating into the ctx like
 * ve_analyze_records.  n_units must equal the last ve_set_units' (or 1 after
 * ve_set_objects).  VE_ERR_INVALID on misaligned records, a PC range outside
 * the ctx or a batch of >= 2^31 records per SM (split it).  Asynchronous on s. */
ve_status ve_analyze_units(ve_ctx* ctx, const ve_unit* units, uint32_t n_units, cudaStream_t s);

/* End-to-end variant: records in HOST memory (pinned or pageable), streamed to
 * the device in chunks through a double-buffered staging area and analyzed
 * (the paper's collector->analyzer buffer path).  Returns after the
 * last chunk is queued; h_records must stay valid until s completes. */
ve_status ve_analyze_records_host(ve_ctx* ctx, const ve_record* h_records, uint64_t n, cudaStream_t s);

/* S10 / C10 (Def 3.1): compare pre and post of object
 * obj_id element-wise over the mask: W (written elements, VE_DIFF_WRITTEN),
 * all elements (VE_DIFF_ALL) or the caller's device bitmap d_mask (bit e in
 * word e/32, LSB first, VE_DIFF_MASK).  Needs both snapshots.  Synchronizes s;
 * writes *h_out. */
ve_status ve_snapshot_diff(ve_ctx* ctx, uint32_t obj_id, uint32_t mode, const uint32_t* d_mask,
                           ve_diff* h_out, cudaStream_t s);

/* S11 / C11 (Def 3.2): duplicate objects among the n given
 * objects (their post snapshots; ids need not be dense here).  Content hash
 * as a filter, byte verification for every grouping.  h_group_of[i] = min id
 * of object i's class (its own id if size 0 or post NULL).  Synchronizes s. */
ve_status ve_object_dedup(ve_ctx* ctx, const ve_object* objs, uint32_t n, uint32_t* h_group_of,
                          cudaStream_t s);

/* S10 / S11 sharded by memory object (the paper claims
 * multi-GPU support without a mechanism).  Every rank holds the same
 * objects (after ve_merge_stats the W / L bitmaps are merged).
 *   ve_snapshot_diff_all: C10 of EVERY object with both snapshots, mode
 *     VE_DIFF_WRITTEN or VE_DIFF_ALL; the object at position k of the sorted
 *     object table is diffed by rank k mod G, the partial results are
 *     SUM-allreduced: h_out[id] (n_objects entries, indexed by object id;
 *     objects without both snapshots report n_elems only).  nccl_comm NULL: one
 *     rank (every object diffed locally).  Synchronizes s.
 *   ve_object_dedup_comm: C11 over NCCL: eligible object k is hashed by rank
 *     k mod G (hashes SUM-allreduced), candidate pair p is byte-verified by rank
 *     p mod G (flags SUM-allreduced); every rank gets the full h_group_of.
 *     Objects' post snapshots must be readable on every rank.  Synchronizes s.
 *   ..._group: the same algorithms with n contexts on one device playing ranks
 *     0..n-1 (device copies instead of NCCL; the tests' transport). */
ve_status ve_snapshot_diff_all(ve_ctx* ctx, uint32_t mode, void* nccl_comm_or_null, ve_diff* h_out, cudaStream_t s);
ve_status ve_object_dedup_comm(ve_ctx* ctx, const ve_object* objs, uint32_t n, void* nccl_comm, uint32_t* h_group_of,
                               cudaStream_t s);
ve_status ve_snapshot_diff_all_group(ve_ctx** ctxs, uint32_t n, uint32_t mode, ve_diff* h_out, cudaStream_t s);
ve_status ve_object_dedup_group(ve_ctx** ctxs, uint32_t n, const ve_object* objs, uint32_t n_objs,
                                uint32_t* h_group_of, cudaStream_t s);

/* S12 / C12: merge statistics.  src != NULL: dst <- dst (+) src on one device
 * (same config and object table).  nccl_comm != NULL (an ncclComm_t over all
 * ranks, each holding a ctx with the same config/objects): every rank ends
 * with the merged statistics of all ranks (sum/min/max allreduce, line-state
 * allgather + monoid merge, bitmap allgather + OR, exact histogram by hash
 * partition all-to-all + top-k re-rank).  Synchronizes s. */
ve_status ve_merge_stats(ve_ctx* dst, const ve_ctx* src_or_null, void* nccl_comm_or_null, cudaStream_t s);

/* S12 on one device: merge n contexts (same config, objects and device) with the
 * same rank-merge algorithm ve_merge_stats runs over NCCL (context i plays rank
 * i: allreduce, allgather and hash-partitioned all-to-all done with device
 * copies); afterwards every context holds the merged statistics.  Synchronizes s. */
ve_status ve_merge_group(ve_ctx** ctxs, uint32_t n, cudaStream_t s);

/* S13: finalize (top-k, distinct counts, bitmap popcounts, derived flags) and
 * copy to a library-owned host report.  Synchronizes the ctx's streams.
 * VE_ERR_STATE if poisoned. */
ve_status ve_report(ve_ctx* ctx, ve_rep** h_out);
void      ve_report_free(ve_rep* r);

/* report accessors (host memory, caller-allocated arrays) */
uint32_t  ve_report_n_keys(const ve_rep* r);
uint32_t  ve_report_n_objects(const ve_rep* r);
uint32_t  ve_report_topk(const ve_rep* r);
ve_status ve_report_keys(const ve_rep* r, ve_key_stats* out);          /* n_keys entries         */
ve_status ve_report_topk_entries(const ve_rep* r, ve_topk_entry* out); /* n_keys * topk entries  */
ve_status ve_report_objects(const ve_rep* r, ve_obj_stats* out);       /* n_objects entries      */
ve_status ve_report_globals(const ve_rep* r, ve_globals* out);
/* S13 report dump (SURVEY 8(a) S13, 8(c) "full report == oracle").  format 0:
 * binary, little-endian, no padding between parts:
 *   u32 magic 0x50524556 ("VERP"), u32 version 1, u32 n_keys, u32 n_objects,
 *   u32 topk, ve_globals (4 x u64), ve_key_stats[n_keys] (336 B each; p_* / q_*
 *   are 0 unless line_state is POINT or LINE), ve_topk_entry[n_keys][topk]
 *   (entries j >= n_top are {0, 0}), ve_obj_stats[n_objects] (indexed by id).
 * format 1: JSON: {"n_records", "n_invalid", "n_unmapped", "keys": [{every raw
 *   field, derived flag and n_type, "p"/"q": [x, y_hi, y_lo], "top": [[bits,
 *   count] x n_top]}], "objects": [{"id", "n_elems", "n_written",
 *   "n_loaded_eq", "n_ld_reload", "n_touched"}]}.
 * Returns VE_ERR_INVALID for a null report / path, an unknown format or a file
 * that cannot be opened. */
ve_status ve_report_dump(const ve_rep* r, const char* path, int format);

/* ---- LoadSpy temporal load redundancy in trace order --------
 * Q1 / R6 (Table 5; LoadSpy, ref [47]): for every valid
 * global-space load r of the n device records, in array order, let r' be the
 * most recent earlier valid global-space load of the same address.  r is
 * temporal if r' exists and temporally redundant if r' also has r's width and
 * value bits.  h_out[2*key] = temporal, h_out[2*key + 1] = redundant, for the
 * ctx's n_keys keys (PC key; object key of the object holding addr, from the
 * ctx's object table).  Order-dependent: one call covers one ordered trace.
 * n < 2^32.  Synchronizes s. */
ve_status ve_temporal_loads(ve_ctx* ctx, const ve_record* d_records, uint64_t n, uint64_t* h_out, cudaStream_t s);
/* The same, plus the per-(PC, object) table (Table 5's redundancy analysis P:L470 per
 * instruction AND data object): h_pairs[2 (pc (n_objects + 1) + id)] = temporal, + 1 =
 * redundant loads of PC pc whose first byte lies in object id (id = n_objects: in none).
 * h_pairs NULL: ve_temporal_loads.  VE_ERR_INVALID if n_pcs x (n_objects + 1) > 2^24. */
ve_status ve_temporal_loads_ex(ve_ctx* ctx, const ve_record* d_records, uint64_t n, uint64_t* h_out,
                               uint64_t* h_pairs, cudaStream_t s);

/* ---- approximate frequent values ---------------------------
 * Def 3.3 (frequent values) over the truncated values of Def 3.8
 * (P:L191-L193): for every key whose records all have one float type (Q15),
 * the exact histogram of its values with the low (m - K) mantissa bits cleared
 * (K = cfg.mant_bits; NaNs keep their bits, R5): h_ndistinct[n_keys] distinct
 * truncated values and h_top[n_keys * topk] by (count desc, bits asc), zero-
 * filled; integer and mixed-type keys report 0.  "Approximate frequent" holds
 * when 100 * h_top[k*topk].count > t_frequent_pct * (n_ld + n_st).  Works on
 * the ctx's statistics as accumulated so far (local merges included);
 * VE_ERR_STATE after an NCCL rank merge.  Synchronizes s. */
ve_status ve_approx_topk(ve_ctx* ctx, uint64_t* h_ndistinct, ve_topk_entry* h_top, cudaStream_t s);

/* ---- dyadic-scaled exact linear fit ------------------------
 * Def 3.7 (structured values) over the EXACT values of the
 * records (R10): a float encodes the dyadic rational (-1)^s M 2^E,
 * so structured floats with non-integral values (k/64 ramps, 3 + i 2^-40) are
 * recognised, which C8's integral-value fit cannot.  Per key of the ctx (PC key,
 * object key of the first byte from the ctx's object table, SHARED key):
 * NaN / inf -> FAIL; scale = T = the largest number of fractional bits, every
 * Y = value * 2^T must satisfy |Y| < 2^62 (else FAIL); P = (min addr, min Y at
 * that addr), Q = (max addr, min Y at that addr); every point collinear with P
 * and Q and equal to the anchor at P.x / Q.x -> LINE (POINT if one address),
 * else FAIL.  Invalid records are skipped.  "Dyadic structured" holds when
 * state == VE_LINE_LINE and py != qy; the line is y = (py + (x - px)(qy - py)
 * / (qx - px)) 2^-scale.  h_out[n_keys] (host memory; EMPTY / FAIL entries
 * zero apart from state).  d_records: device, 8-byte aligned.  Three passes
 * over the records; independent of the ctx's statistics.  Synchronizes s. */
typedef struct ve_dyadic { uint32_t state, scale; uint64_t px, qx; int64_t py, qy; } ve_dyadic;
ve_status ve_dyadic_fit(ve_ctx* ctx, const ve_record* d_records, uint64_t n, ve_dyadic* h_out, cudaStream_t s);

/* ---- approximate structured and structured with <= eps outliers ----
 * The paper's approximate patterns cover "some fine-grained patterns" (Def 3.8,
 * P:L191) without a definition, and Table 1 marks srad_v1 structured
 * although its clamped boundary breaks an exact fit (Def 3.7).
 *   ve_dyadic_fit_ex(flags = VE_FIT_TRUNC): C22 (R11) -- C21 over the
 *     values every float record carries after Def 3.8's truncation to
 *     cfg.mant_bits mantissa bits (toward zero); integers unchanged.  flags 0 is
 *     ve_dyadic_fit.
 *   ve_outlier_fit: C23 (R12) -- per key, points as in C21 (with
 *     VE_FIT_TRUNC: truncated first); the line through the INTERIOR anchors A =
 *     (second-smallest distinct address, smallest Y there) and B = (second-largest
 *     distinct address, smallest Y there); n_off = records off it (exact 128-bit
 *     check), n = records.  state FAIL (NaN / inf, |Y| >= 2^62), EMPTY, POINT
 *     (fewer than 4 distinct addresses), LINE.  "Structured with <= eps outliers"
 *     is LINE with ay != by and 100 n_off <= eps_pct n.
 * Both: device records (8-byte aligned), h_out[n_keys] host; four (C23) or three
 * streaming passes; synchronize s. */
enum { VE_FIT_TRUNC = 1 };
typedef struct ve_outlier { uint32_t state, scale; uint64_t ax, bx; int64_t ay, by; uint64_t n_off, n; } ve_outlier;
ve_status ve_dyadic_fit_ex(ve_ctx* ctx, const ve_record* d_records, uint64_t n, uint32_t flags, ve_dyadic* h_out,
                           cudaStream_t s);
ve_status ve_outlier_fit(ve_ctx* ctx, const ve_record* d_records, uint64_t n, uint32_t flags, ve_outlier* h_out,
                         cudaStream_t s);

/* ---- accessed intervals and the adaptive copy plan --------
 * PAPER.md section 6.1: "We define an interval [start, end] as
 * the memory range accessed by each GPU instruction" and merge intervals "if
 * they are adjacent or overlapped", on the GPU (Figure 4);
 * the merged intervals drive the choice between segment copy and min-max copy
 * of a data object's snapshot (Figure 5).  DESIGN.md 3 (R1-R4). */
typedef struct ve_interval { uint64_t start, end; } ve_interval;   /* inclusive bytes */

enum { VE_COPY_NONE = 0, VE_COPY_SEGMENT = 1, VE_COPY_MINMAX = 2 };
typedef struct ve_copy_plan {
  uint64_t n_segments;      /* merged intervals clipped to the object (segment copies)  */
  uint64_t accessed_bytes;  /* bytes they cover (segment copy volume, Fig. 5c)          */
  uint64_t lo, hi;          /* min / max accessed byte address, inclusive (0, 0: none)  */
  uint64_t direct_bytes;    /* object size (direct copy, Fig. 5a)                       */
  uint64_t minmax_bytes;    /* hi - lo + 1 (min-max copy, Fig. 5b); 0 when untouched     */
  uint32_t choice;          /* VE_COPY_*: SEGMENT iff n_segments <= seg_max and          */
                            /* 100*accessed_bytes < dense_pct*minmax_bytes (R4)          */
  uint32_t pad;
} ve_copy_plan;

/* Merge n device intervals d_in (start > end = empty, skipped) into the sorted
 * maximal runs of their union: out[k].end + 1 < out[k+1].start.  d_out (device,
 * room for n) receives *h_n_out intervals.  n < 2^32.  Synchronizes s. */
ve_status ve_interval_merge(ve_ctx* ctx, const ve_interval* d_in, uint64_t n, ve_interval* d_out,
                            uint64_t* h_n_out, cudaStream_t s);

/* The merged intervals accessed by n device records: [addr, addr + w - 1] of
 * every valid global-space record (shared-space and invalid records skipped;
 * validity uses the ctx's n_pcs).  d_out needs room for n.  n < 2^32.
 * Synchronizes s. */
ve_status ve_record_intervals(ve_ctx* ctx, const ve_record* d_records, uint64_t n, ve_interval* d_out,
                              uint64_t* h_n_out, cudaStream_t s);

/* Copy plan of every object of the ctx (h_plan[id], n_objects entries) from a
 * merged interval set (output of the two calls above; VE_ERR_INVALID if it is
 * not sorted, disjoint and non-adjacent).  Synchronizes s. */
ve_status ve_plan_copies(ve_ctx* ctx, const ve_interval* d_merged, uint64_t n, uint32_t seg_max,
                         uint32_t dense_pct, ve_copy_plan* h_plan, cudaStream_t s);

/* ---- value flow graph (Defs 5.1-5.3) ----------
 * Host-side bookkeeping over an API-event log (no device work, no ctx).  The
 * log is the program-order list of data-object accesses of GPU API
 * invocations; accesses of one invocation share a sequence number.  Readings
 * R7-R9 in DESIGN.md section 3. */
#define VE_HOST_VERTEX 0xFFFFFFFFu                 /* v_host */
enum { VE_ACC_READ = 1, VE_ACC_WRITE = 2 };         /* edge labels (bit set)                     */
enum { VE_EV_DEVICE = 0, VE_EV_ALLOC = 1, VE_EV_H2D = 2, VE_EV_D2H = 3 };

typedef struct ve_api_access {
  uint64_t seq;        /* invocation sequence number, non-decreasing over the log         */
  uint64_t bytes;      /* bytes accessed: the edge importance I(e)                */
  uint32_t vertex;     /* vertex id = the API's call path: equal ids merge        */
  uint32_t object;     /* data object id (dense, < 2^32 - 1)                              */
  uint32_t mode;       /* VE_ACC_READ | VE_ACC_WRITE (ALLOC / H2D imply WRITE, D2H READ)   */
  uint32_t kind;       /* VE_EV_*: ALLOC creates the object (its first writer);   */
                       /* H2D adds a source edge host -> vertex, D2H a sink edge vertex -> host */
} ve_api_access;

typedef struct ve_vfg_edge {
  uint32_t src, dst;   /* vertex ids; VE_HOST_VERTEX for source / sink edges              */
  uint32_t object;     /* D_{v_k}                                                         */
  uint32_t label;      /* VE_ACC_* of the accessing (dst) side, ORed over merged invocations */
  uint64_t bytes;      /* summed accessed bytes                                           */
  uint64_t count;      /* invocations merged into the edge                                */
} ve_vfg_edge;

typedef struct ve_vfg_vertex {
  uint32_t vertex, pad;
  uint64_t invocations;   /* I(v) */
} ve_vfg_vertex;

typedef struct ve_vfg ve_vfg;   /* opaque, host memory */

/* Def 5.1: build the graph.  VE_ERR_INVALID if seq decreases or an object is
 * accessed before its allocation.  Edges sorted by (src, dst, object),
 * vertices by id (v_host not listed). */
ve_status ve_vfg_build(const ve_api_access* log, uint64_t n, ve_vfg** out);
/* Def 5.2: the vertex slice graph of vertex v (VE_ERR_INVALID if v is absent). */
ve_status ve_vfg_slice(const ve_vfg* g, uint32_t v, ve_vfg** out);
/* Def 5.3: edges with bytes >= min_edge_bytes; vertices on a kept edge or with
 * invocations >= min_vertex_invocations. */
ve_status ve_vfg_important(const ve_vfg* g, uint64_t min_edge_bytes, uint64_t min_vertex_invocations,
                           ve_vfg** out);
ve_status ve_vfg_size(const ve_vfg* g, uint64_t* n_vertices, uint64_t* n_edges);
ve_status ve_vfg_vertices(const ve_vfg* g, ve_vfg_vertex* out);   /* n_vertices entries */
ve_status ve_vfg_edges(const ve_vfg* g, ve_vfg_edge* out);         /* n_edges entries    */
void      ve_vfg_free(ve_vfg* g);

/* Number of libve kernels launched by this process so far (all contexts). */
uint64_t  ve_kernel_launches(void);

/* NCCL helpers (NCCL is loaded at run time; only ve_merge_stats with a comm needs it) */
ve_status ve_nccl_get_unique_id(void* out128);                          /* 128-byte ncclUniqueId */
ve_status ve_nccl_comm_init(void** comm_out, int nranks, const void* id128, int rank);
ve_status ve_nccl_comm_destroy(void* comm);

#ifdef __cplusplus
}
#endif
#endif /* VE_H */
