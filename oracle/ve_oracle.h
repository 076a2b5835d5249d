/*
 * ve_oracle.h -- CPU ORACLE for the ValueExpert value-trace analysis.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load liboracle.so.
 * The product library (libve.so) never includes, links or calls this code,
 * and this code includes nothing from the product tree.
 *
 * A plain, slow, single-threaded implementation of the definitions of
 * SURVEY.md 8(c) C1-C12, which restate PAPER.md Defs 3.1-3.8
 * (section 3) and section 5.1.
 * Every statistic is an order-free function of the record multiset plus the
 * snapshots, so the oracle computes each definition directly (sort +
 * run-length for histograms, two passes over the points for the exact line
 * fit, bytewise memcmp for snapshots).  Readings of ambiguous passages are
 * listed in DESIGN.md section 3 (Q1-Q23).
 *
 * Parity pins: see tests/test_oracle_pins.py (paper worked examples
 * P1-P14, closed forms of cfg1, brute force B1-B5, invariants I1-I10).
 * Every function below is pinned; none is "parity unpinned".
 *
 * The record / object byte layouts are the only thing shared with the product
 * ABI (include/ve.h); they are re-declared here, not included.
 */
#ifndef VE_ORACLE_H
#define VE_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct vo_record {       /* 24 bytes: same byte layout as ve_record */
  uint64_t addr;
  uint64_t value;
  uint32_t pc;
  uint32_t meta;
} vo_record;

typedef struct vo_object {       /* host-memory snapshots */
  uint64_t base, size;
  const uint8_t* pre;            /* NULL = no pre snapshot  */
  const uint8_t* post;           /* NULL = no post snapshot */
  uint32_t id;                   /* dense 0..n-1 */
  uint32_t elem_width;           /* 1,2,4,8 */
} vo_object;

typedef struct vo_config {
  uint32_t n_pcs;
  uint32_t topk;                 /* <= 64 */
  uint32_t mant_bits;            /* K */
  uint32_t t_redundant_pct;
  uint32_t t_frequent_pct;
  uint32_t pad;
} vo_config;

#define VO_MAX_TOPK 64

/* line states (C8) */
enum { VO_LINE_EMPTY = 0, VO_LINE_POINT = 1, VO_LINE_LINE = 2, VO_LINE_FAIL = 3 };

/* per-key statistics; key index: PCs [0,n_pcs), objects n_pcs+id, SHARED n_pcs+n_obj */
typedef struct vo_key {
  /* C1, C2, C5 sums */
  uint64_t n_ld, n_st, n_zero, n_ld_eq_pre, n_st_eq_pre, n_nosnap;
  uint64_t n_type[12];
  uint64_t n_nan, n_nonint, n_not_f16, n_not_bf16, n_not_f32;
  /* C4, C5, C7 min/max (identity values when no contributor: min=~0, max=0) */
  uint64_t raw_min, raw_max, ord_min, ord_max, trunc_min, trunc_max;
  /* C8 line state; y is a signed 128-bit integer split in (lo, hi) */
  uint64_t line_state;
  uint64_t p_x, p_ylo; int64_t p_yhi;
  uint64_t q_x, q_ylo; int64_t q_yhi;
  /* C9 */
  uint64_t n_distinct;
  uint64_t n_top;
  uint64_t top_bits[VO_MAX_TOPK];
  uint64_t top_count[VO_MAX_TOPK];
  /* derived flags (report-time, from the fields above) */
  uint32_t single_value, single_zero, frequent, structured, approx, dict8;
  uint32_t heavy;                /* type code 0..11 of the narrowest type, 255 = none */
  uint32_t single_type;          /* 1 iff exactly one n_type bin is non-zero */
} vo_key;

typedef struct vo_globals {
  uint64_t n_records, n_invalid, n_unmapped;
  uint64_t u_touched;            /* U of SURVEY 8(d): distinct pre elements referenced with eq_pre defined */
} vo_globals;

typedef struct vo_objstat {
  uint64_t n_elems;
  uint64_t n_written;            /* |W| */
  uint64_t n_loaded_eq;          /* |L| */
  uint64_t n_ld_reload;          /* C3 */
  uint64_t n_touched;            /* |W u L| */
} vo_objstat;

typedef struct vo_diff {
  uint64_t n_elems, n_masked, n_unchanged, n_changed, n_untouched;
  uint32_t redundant, pad;
} vo_diff;

enum { VO_DIFF_WRITTEN = 0, VO_DIFF_ALL = 1, VO_DIFF_MASK = 2 };

/* Analyze records (C1-C9, C3); keys has n_pcs + n_obj + 1 entries, objstat n_obj.
 * Returns 0 on success, -1 on invalid arguments. */
int vo_analyze(const vo_config* cfg, const vo_object* objs, uint32_t n_obj,
               const vo_record* recs, uint64_t n,
               vo_key* keys, vo_globals* glob, vo_objstat* objstat);

/* C10: snapshot diff of object obj_id (mask bit e in word e/32, LSB first). */
int vo_snapshot_diff(const vo_config* cfg, const vo_object* objs, uint32_t n_obj,
                     const vo_record* recs, uint64_t n, uint32_t obj_id,
                     uint32_t mode, const uint32_t* mask, vo_diff* out);

/* C11: duplicate objects; group_of[i] = min id of i's class. */
int vo_object_dedup(const vo_object* objs, uint32_t n, uint32_t* group_of);

/* ---- accessed intervals and the adaptive copy plan -------
 * PAPER.md section 6.1 (Figures 4 and 5).  The paper defines an
 * interval [start, end] as the memory range accessed by a GPU instruction and
 * merges intervals that are "adjacent or overlapped"; the merged set
 * is the union's maximal runs of consecutive byte addresses.
 * readings R1-R4. */
typedef struct vo_interval { uint64_t start, end; } vo_interval;   /* inclusive */

typedef struct vo_copy_plan {
  uint64_t n_segments;      /* merged intervals clipped to the object        */
  uint64_t accessed_bytes;  /* bytes they cover (segment copy, Fig. 5c)      */
  uint64_t lo, hi;          /* min / max accessed byte address (inclusive)   */
  uint64_t direct_bytes;    /* object size (direct copy, Fig. 5a)            */
  uint64_t minmax_bytes;    /* hi - lo + 1 (min-max copy, Fig. 5b), 0 if none */
  uint32_t choice;          /* VO_COPY_*                                     */
  uint32_t pad;
} vo_copy_plan;

enum { VO_COPY_NONE = 0, VO_COPY_SEGMENT = 1, VO_COPY_MINMAX = 2 };

/* C13: merge n intervals (start > end = empty, ignored) into the sorted
 * maximal runs of their union; out needs room for n.  Returns the count. */
uint64_t vo_interval_merge(const vo_interval* in, uint64_t n, vo_interval* out);

/* C14: the merged intervals accessed by the valid global-space records
 * ([addr, addr + w - 1] per record). */
uint64_t vo_record_intervals(uint32_t n_pcs, const vo_record* recs, uint64_t n, vo_interval* out);

/* C15: adaptive copy plan per object; merged must be the output
 * of C13/C14.  plan[id] for every object id. */
int vo_plan_copies(const vo_object* objs, uint32_t n_obj, const vo_interval* merged, uint64_t n,
                 uint32_t seg_max, uint32_t dense_pct, vo_copy_plan* plan);

/* ---- value flow graph (Defs 5.1-5.3) -------------
 * Layouts equal ve.h's ve_api_access / ve_vfg_edge / ve_vfg_vertex (re-declared).
 * Build (C18): for every non-allocation access of D_k by v_j, the edge from the
 * vertex of the latest earlier invocation that writes D_k (allocation, host copy
 * or a write access), found by scanning the log backwards -- Def 5.1 read
 * literally -- plus source / sink edges of host copies.  Slice (C19): a fixpoint
 * of "reaches v" / "reached from v" over each object's edges.  Important (C20):
 * the two thresholds of Def 5.3.  Edges sorted by (src, dst, object). */
#define VO_HOST 0xFFFFFFFFu
typedef struct vo_access { uint64_t seq, bytes; uint32_t vertex, object, mode, kind; } vo_access;
typedef struct vo_vfg_edge { uint32_t src, dst, object, label; uint64_t bytes, count; } vo_vfg_edge;
typedef struct vo_vfg_vertex { uint32_t vertex, pad; uint64_t invocations; } vo_vfg_vertex;

/* edges: room for 2n, verts: room for n.  Returns -1 on an access before allocation. */
int vo_vfg_build(const vo_access* log, uint64_t n, vo_vfg_edge* edges, uint64_t* ne, vo_vfg_vertex* verts,
                 uint64_t* nv);
int vo_vfg_slice(const vo_vfg_edge* edges, uint64_t ne, const vo_vfg_vertex* verts, uint64_t nv, uint32_t v,
                 vo_vfg_edge* oe, uint64_t* one, vo_vfg_vertex* ov, uint64_t* onv);
int vo_vfg_important(const vo_vfg_edge* edges, uint64_t ne, const vo_vfg_vertex* verts, uint64_t nv,
                     uint64_t min_edge_bytes, uint64_t min_vertex_invocations,
                     vo_vfg_edge* oe, uint64_t* one, vo_vfg_vertex* ov, uint64_t* onv);

/* ---- LoadSpy temporal load redundancy in trace order --------
 * Q1 / R6 (Table 5 "redundancy analysis"; LoadSpy, ref [47]): for
 * every valid global-space load r, in record order, let r' be the most recent
 * earlier valid global-space load of the same address.  r is *temporal* if r'
 * exists, and *temporally redundant* if moreover r' has r's width and value
 * bits.  Counted per key (PC key; object key of r's first byte, unmapped loads
 * PC only): out[2 * key] = temporal, out[2 * key + 1] = redundant (C17). */
int vo_temporal_loads(const vo_config* cfg, const vo_object* objs, uint32_t n_obj, const vo_record* recs,
                      uint64_t n, uint64_t* out);
/* the same per (PC, object): out[2 (pc (n_obj + 1) + id)], id = n_obj for loads outside every object */
int vo_temporal_pairs(const vo_config* cfg, const vo_object* objs, uint32_t n_obj, const vo_record* recs,
                      uint64_t n, uint64_t* out);

/* ---- approximate frequent values -------------------------
 * Def 3.3 (frequent values) over the truncated values of Def 3.8
 * ("approximate values ... some fine-grained patterns"): for every
 * key whose records all have one float type (Q15), each value's low (m - K)
 * mantissa bits are cleared (C7; NaNs keep their bits, R5) and the exact
 * histogram of the truncated values gives n_distinct and the top-k by (count
 * desc, bits asc).  Keys of mixed or integer type report 0 / nothing (C16).
 * ndistinct[n_keys], top_bits / top_count[n_keys * topk] (0-filled). */
int vo_approx_topk(const vo_config* cfg, const vo_object* objs, uint32_t n_obj, const vo_record* recs,
                   uint64_t n, uint64_t* ndistinct, uint64_t* top_bits, uint64_t* top_count);

/* ---- dyadic-scaled exact linear fit (C21) ----------------
 * Def 3.7 (structured values) over the EXACT values of the
 * records (floats as the dyadic rationals they encode; R10): per key,
 * NaN / inf -> FAIL; T = max fractional bits; every Y = y 2^T must satisfy
 * |Y| < 2^62 (else FAIL); anchors P = (min x, min Y at that x), Q = (max x,
 * min Y at that x); all points collinear -> LINE (POINT if one x), else FAIL.
 * out[n_keys]; EMPTY / FAIL entries are zero apart from state. */
typedef struct vo_dyadic { uint32_t state, scale; uint64_t px, qx; int64_t py, qy; } vo_dyadic;
int vo_dyadic_fit(const vo_config* cfg, const vo_object* objs, uint32_t n_obj, const vo_record* recs, uint64_t n,
                  vo_dyadic* out);

/* ---- approximate structured (C22) and structured with <= eps outliers (C23) ----
 * C22: C21 over the float values truncated to K mantissa bits (Def 3.8 over Def 3.7; R11).
 * C23: anchors at the second-smallest and second-largest distinct address (min Y there), n_off =
 * records off that line, n = records (R12); flags & 1: the C22 truncation first.
 * State FAIL on NaN / inf or |Y| >= 2^62, EMPTY, POINT (< 4 distinct addresses), LINE. */
int vo_dyadic_fit_trunc(const vo_config* cfg, const vo_object* objs, uint32_t n_obj, const vo_record* recs,
                        uint64_t n, vo_dyadic* out);
typedef struct vo_outlier { uint32_t state, scale; uint64_t ax, bx; int64_t ay, by; uint64_t n_off, n; } vo_outlier;
int vo_outlier_fit(const vo_config* cfg, const vo_object* objs, uint32_t n_obj, const vo_record* recs, uint64_t n,
                   uint32_t flags, vo_outlier* out);

/* helpers exposed for pinning */
uint64_t vo_ord(uint64_t b, uint32_t kind, uint32_t w);
uint32_t vo_float_flags(uint64_t b, uint32_t kind, uint32_t w);   /* bit0 nan, 1 nonint, 2 not_f16, 3 not_bf16, 4 not_f32 */
uint64_t vo_trunc(uint64_t b, uint32_t kind, uint32_t w, uint32_t K);
uint64_t vo_sizeof(int which);

#ifdef __cplusplus
}
#endif
#endif
