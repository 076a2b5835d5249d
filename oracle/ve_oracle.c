/*
 * ve_oracle.c -- CPU ORACLE (test infrastructure only; see ve_oracle.h).
 *
 * Plain C11 + gcc extensions (__int128, _Float16, __bf16).  Single-threaded.
 * Each function cites the passage it follows.  P:L<n> = PAPER.md line n;
 * "C<k>" / "Q<k>" = the definition / reading in SURVEY.md 8(c), restated in
 * DESIGN.md section 3.
 *
 * Nothing here is blocked, fused or reordered: records are visited in array
 * order, histograms are "sort + run-length", the line fit visits every point
 * against the extreme-x pair, snapshots are compared with memcmp.
 */
#include "ve_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

typedef __int128 i128;

/* ---- record decoding (SURVEY 8(b) ve_record.meta) --------- */

static uint32_t rec_w(uint32_t meta) { return 1u << (meta & 3u); }
static uint32_t rec_kind(uint32_t meta) { return (meta >> 2) & 3u; }
static int rec_store(uint32_t meta) { return (meta >> 4) & 1u; }
static int rec_shared(uint32_t meta) { return (meta >> 5) & 1u; }

/* Validity rules of SURVEY 8(b) "Invalid records are data, not errors". */
static int rec_valid(const vo_record* r, uint32_t n_pcs) {
  uint32_t w = rec_w(r->meta), kind = rec_kind(r->meta);
  if (r->meta >> 6) return 0;
  if (kind == 2 && w == 1) return 0;
  if (kind == 3 && w != 2) return 0;
  if (r->pc >= n_pcs) return 0;
  if (w < 8 && (r->value >> (8 * w)) != 0) return 0;
  if (r->addr >= (1ull << 48)) return 0;
  return 1;
}

/* Type code order u8 u16 u32 u64 i8 i16 i32 i64 f16 f32 f64 bf16 (C1). */
static uint32_t type_code(uint32_t kind, uint32_t w) {
  uint32_t lg = (w == 1) ? 0 : (w == 2) ? 1 : (w == 4) ? 2 : 3;
  if (kind == 0) return lg;
  if (kind == 1) return 4 + lg;
  if (kind == 3) return 11;
  return (w == 2) ? 8 : (w == 4) ? 9 : 10;
}

static uint32_t tc_width(uint32_t tc) {
  static const uint32_t wid[12] = {1, 2, 4, 8, 1, 2, 4, 8, 2, 4, 8, 2};
  return wid[tc];
}

/* Exact value of a float record, through the compiler's own conversions
 * (an independent path from the GPU's bit manipulation). */
static double float_value(uint64_t b, uint32_t kind, uint32_t w) {
  if (kind == 3) {                     /* bfloat16 = top half of a binary32 */
    uint32_t u = (uint32_t)b << 16;
    float f;
    memcpy(&f, &u, 4);
    return (double)f;
  }
  if (w == 2) {
    uint16_t u = (uint16_t)b;
    _Float16 h;
    memcpy(&h, &u, 2);
    return (double)h;
  }
  if (w == 4) {
    uint32_t u = (uint32_t)b;
    float f;
    memcpy(&f, &u, 4);
    return (double)f;
  }
  double d;
  memcpy(&d, &b, 8);
  return d;
}

static int64_t sext(uint64_t b, uint32_t w) {
  if (w == 8) return (int64_t)b;
  uint32_t sh = 64 - 8 * w;
  return (int64_t)(b << sh) >> sh;
}

/* C5: orderable key.  uint -> b; sint -> sext(b) XOR 2^63;
 * float -> sign set ? ~b & mask_w : b | signbit_w. */
uint64_t vo_ord(uint64_t b, uint32_t kind, uint32_t w) {
  if (kind == 0) return b;
  if (kind == 1) return (uint64_t)sext(b, w) ^ (1ull << 63);
  uint64_t mask = (w == 8) ? ~0ull : ((1ull << (8 * w)) - 1);
  uint64_t sign = 1ull << (8 * w - 1);
  return (b & sign) ? (~b & mask) : (b | sign);
}

/* C5 float flags: bit0 NaN, bit1 nonint, bit2 not_f16, bit3 not_bf16,
 * bit4 not_f32 (f64 sources only).  "not_X" = the round trip through X
 * (round-to-nearest-even) is not the identity; NaNs fail all of them. */
uint32_t vo_float_flags(uint64_t b, uint32_t kind, uint32_t w) {
  if (kind < 2) return 0;
  double v = float_value(b, kind, w);
  int is_f64 = (kind == 2 && w == 8);
  if (isnan(v)) return 1u | 2u | 4u | 8u | (is_f64 ? 16u : 0u);
  uint32_t f = 0;
  /* nonint: +-Inf, non-integral, -0.0, or |v| >= 2^63 (C5; Q11) */
  if (isinf(v) || v != trunc(v) || (v == 0.0 && signbit(v)) || fabs(v) >= 9223372036854775808.0)
    f |= 2u;
  if ((double)(_Float16)v != v) f |= 4u;
  if ((double)(__bf16)v != v) f |= 8u;
  if (is_f64 && (double)(float)v != v) f |= 16u;
  return f;
}

/* C7: clear the low (m-K) mantissa bits; m = 10/7/23/52 (Def 3.8; Q6). */
uint64_t vo_trunc(uint64_t b, uint32_t kind, uint32_t w, uint32_t K) {
  uint32_t m = (kind == 3) ? 7 : (w == 2) ? 10 : (w == 4) ? 23 : 52;
  if (K >= m) return b;
  return b & ~((1ull << (m - K)) - 1);
}

/* ---- object table (start address + size per object) ------------ */

typedef struct {
  const vo_object** by_base;
  uint32_t n;
} objtab;

static int cmp_obj_base(const void* a, const void* b) {
  const vo_object* x = *(const vo_object* const*)a;
  const vo_object* y = *(const vo_object* const*)b;
  return (x->base > y->base) - (x->base < y->base);
}

static int objtab_build(objtab* t, const vo_object* objs, uint32_t n) {
  t->n = n;
  t->by_base = (const vo_object**)malloc(sizeof(*t->by_base) * (n ? n : 1));
  char* seen = (char*)calloc(n ? n : 1, 1);
  for (uint32_t i = 0; i < n; ++i) {
    const vo_object* o = &objs[i];
    uint32_t ew = o->elem_width;
    if (o->size == 0 || o->id >= n || seen[o->id] || !(ew == 1 || ew == 2 || ew == 4 || ew == 8) ||
        o->base >= (1ull << 48) || o->size > (1ull << 48) - o->base) {
      free(seen);
      free(t->by_base);
      return -1;
    }
    seen[o->id] = 1;
    t->by_base[i] = o;
  }
  free(seen);
  qsort(t->by_base, n, sizeof(*t->by_base), cmp_obj_base);
  for (uint32_t i = 1; i < n; ++i)
    if (t->by_base[i - 1]->base + t->by_base[i - 1]->size > t->by_base[i]->base) {
      free(t->by_base);
      return -1;
    }
  return 0;
}

/* The object containing addr (first byte), or NULL. */
static const vo_object* objtab_find(const objtab* t, uint64_t addr) {
  uint32_t lo = 0, hi = t->n;          /* first object with base > addr */
  while (lo < hi) {
    uint32_t mid = lo + (hi - lo) / 2;
    if (t->by_base[mid]->base <= addr) lo = mid + 1; else hi = mid;
  }
  if (lo == 0) return NULL;
  const vo_object* o = t->by_base[lo - 1];
  return (addr - o->base < o->size) ? o : NULL;
}

static uint64_t n_elems_of(const vo_object* o) {
  return (o->size + o->elem_width - 1) / o->elem_width;
}

/* ---- one decoded record ------------------------------------------------- */

typedef struct {
  int valid, store, shared;
  uint32_t w, kind, tc, fflags;
  const vo_object* obj;     /* mapped object (global space) */
  int inside;               /* [addr, addr+w) inside obj */
  int eq_defined, eq_pre;   /* C2 */
} dec_t;

static void decode(const vo_config* cfg, const objtab* t, const vo_record* r, dec_t* d) {
  memset(d, 0, sizeof(*d));
  d->valid = rec_valid(r, cfg->n_pcs);
  if (!d->valid) return;
  d->w = rec_w(r->meta);
  d->kind = rec_kind(r->meta);
  d->store = rec_store(r->meta);
  d->shared = rec_shared(r->meta);
  d->tc = type_code(d->kind, d->w);
  d->fflags = vo_float_flags(r->value, d->kind, d->w);
  if (d->shared) return;                                  /* Q20: no snapshot */
  d->obj = objtab_find(t, r->addr);
  if (!d->obj) return;
  uint64_t off = r->addr - d->obj->base;
  d->inside = (off + d->w <= d->obj->size);               /* Q21 */
  if (d->inside && d->obj->pre) {
    d->eq_defined = 1;
    int eq = 1;                                           /* C2: little-endian bytes */
    for (uint32_t i = 0; i < d->w; ++i)
      if (d->obj->pre[off + i] != (uint8_t)(r->value >> (8 * i))) eq = 0;
    d->eq_pre = eq;
  }
}

/* ---- histogram entries for C9 ------------------------------------------ */

typedef struct { uint64_t key, bits, count; } hent;

static int cmp_key_bits(const void* a, const void* b) {
  const hent* x = (const hent*)a;
  const hent* y = (const hent*)b;
  if (x->key != y->key) return x->key < y->key ? -1 : 1;
  if (x->bits != y->bits) return x->bits < y->bits ? -1 : 1;
  return 0;
}

/* (key asc, count desc, bits asc): the top-k order of C9 / Q18 */
static int cmp_key_count_bits(const void* a, const void* b) {
  const hent* x = (const hent*)a;
  const hent* y = (const hent*)b;
  if (x->key != y->key) return x->key < y->key ? -1 : 1;
  if (x->count != y->count) return x->count > y->count ? -1 : 1;
  if (x->bits != y->bits) return x->bits < y->bits ? -1 : 1;
  return 0;
}

/* ---- line fit (C8, Def 3.7) ---------------------------------- */

typedef struct {
  int have, fail;
  uint64_t px, qx;
  i128 py, qy;
} line_acc;

/* y of a record for the structured check; returns 0 if the record FAILs it */
static int point_y(uint64_t b, uint32_t kind, uint32_t w, uint32_t fflags, i128* y) {
  if (kind == 0) { *y = (i128)b; return 1; }
  if (kind == 1) { *y = (i128)sext(b, w); return 1; }
  if (fflags & 2u) return 0;                               /* nonint float => FAIL */
  *y = (i128)(int64_t)float_value(b, kind, w);
  return 1;
}

static int collinear(i128 px, i128 py, i128 qx, i128 qy, i128 x, i128 y) {
  return (y - py) * (qx - px) == (qy - py) * (x - px);
}

/* ---- C6 heavy type (report-time) --------------------------------------- */

static double ord_to_double(uint64_t ord, uint32_t kind, uint32_t w) {
  uint64_t mask = (w == 8) ? ~0ull : ((1ull << (8 * w)) - 1);
  uint64_t sign = 1ull << (8 * w - 1);
  uint64_t b = (ord & sign) ? (ord & ~sign) : (~ord & mask);
  return float_value(b, kind, w);
}

static uint32_t heavy_type(const vo_key* k, uint32_t tc) {
  uint32_t w = tc_width(tc);
  static const uint32_t cand_w[3] = {1, 2, 4};
  if (tc <= 3) {                                           /* uint source */
    for (int i = 0; i < 3; ++i) {
      uint32_t v = cand_w[i];
      if (v >= w) break;
      if (k->ord_max <= ((1ull << (8 * v)) - 1)) return (v == 1) ? 0 : (v == 2) ? 1 : 2;
    }
    return 255;
  }
  if (tc <= 7) {                                           /* sint source */
    int64_t mn = (int64_t)(k->ord_min ^ (1ull << 63));
    int64_t mx = (int64_t)(k->ord_max ^ (1ull << 63));
    for (int i = 0; i < 3; ++i) {
      uint32_t v = cand_w[i];
      if (v >= w) break;
      int64_t lo = -(1ll << (8 * v - 1)), hi = (1ll << (8 * v - 1)) - 1;
      if (mn >= lo && mx <= hi) return (v == 1) ? 4 : (v == 2) ? 5 : 6;
    }
    return 255;
  }
  /* float source: integer candidates by exact range when every value is
   * integral, then the float formats by exact round trip (C6, Q10) */
  uint32_t kind = (tc == 11) ? 3 : 2;
  double mn = ord_to_double(k->ord_min, kind, w), mx = ord_to_double(k->ord_max, kind, w);
  for (int i = 0; i < 3; ++i) {
    uint32_t v = cand_w[i];
    if (v >= w) break;
    if (k->n_nonint == 0) {
      if (mn >= 0) {
        if (mx <= (double)((1ull << (8 * v)) - 1)) return (v == 1) ? 0 : (v == 2) ? 1 : 2;
      } else {
        double lo = -(double)(1ull << (8 * v - 1)), hi = (double)(1ull << (8 * v - 1)) - 1;
        if (mn >= lo && mx <= hi) return (v == 1) ? 4 : (v == 2) ? 5 : 6;
      }
    }
    if (v == 2 && k->n_not_f16 == 0) return 8;
    if (v == 2 && k->n_not_bf16 == 0) return 11;
    if (v == 4 && k->n_not_f32 == 0) return 9;
  }
  return 255;
}

static void derive_flags(const vo_config* cfg, vo_key* k) {
  uint64_t n = k->n_ld + k->n_st;
  uint32_t nt = 0, tc = 0;
  for (uint32_t t = 0; t < 12; ++t)
    if (k->n_type[t]) { ++nt; tc = t; }
  k->single_type = (nt == 1);
  k->single_value = (n > 0 && k->raw_min == k->raw_max);                  /* Def 3.4 */
  k->single_zero = (n > 0 && k->n_zero == n);                             /* Def 3.5 */
  k->frequent = (k->n_top > 0 &&                                          /* Def 3.3 */
                 (unsigned __int128)100 * k->top_count[0] > (unsigned __int128)cfg->t_frequent_pct * n);
  k->structured = 0; k->approx = 0; k->dict8 = 0; k->heavy = 255;
  if (!k->single_type) return;                                            /* Q15 */
  int is_float = (tc >= 8);
  i128 py = (i128)(((unsigned __int128)(uint64_t)k->p_yhi << 64) | k->p_ylo);
  i128 qy = (i128)(((unsigned __int128)(uint64_t)k->q_yhi << 64) | k->q_ylo);
  k->structured = (k->line_state == VO_LINE_LINE && py != qy);            /* Def 3.7 */
  k->approx = (is_float && k->n_nan == 0 && n > 0 && k->trunc_min == k->trunc_max &&
               !k->single_value);                                          /* Def 3.8 */
  k->dict8 = (k->n_distinct <= 256 && tc_width(tc) > 1);
  k->heavy = heavy_type(k, tc);                                            /* Def 3.6 */
}

/* ---- vo_analyze: C1-C9 per key, C3 per object --------------------------- */

int vo_analyze(const vo_config* cfg, const vo_object* objs, uint32_t n_obj,
               const vo_record* recs, uint64_t n,
               vo_key* keys, vo_globals* glob, vo_objstat* objstat) {
  if (!cfg || cfg->topk > VO_MAX_TOPK || cfg->n_pcs == 0) return -1;
  objtab t;
  if (objtab_build(&t, objs, n_obj) != 0) return -1;
  const uint64_t n_keys = (uint64_t)cfg->n_pcs + n_obj + 1;
  const uint64_t key_shared = (uint64_t)cfg->n_pcs + n_obj;

  memset(keys, 0, sizeof(vo_key) * n_keys);
  for (uint64_t k = 0; k < n_keys; ++k) {
    keys[k].raw_min = keys[k].ord_min = keys[k].trunc_min = ~0ull;
  }
  memset(glob, 0, sizeof(*glob));

  /* per-object element marks: W (written), L (eq_pre loads), U (eq-defined refs) */
  unsigned char** Wm = (unsigned char**)calloc(n_obj ? n_obj : 1, sizeof(*Wm));
  unsigned char** Lm = (unsigned char**)calloc(n_obj ? n_obj : 1, sizeof(*Lm));
  unsigned char** Um = (unsigned char**)calloc(n_obj ? n_obj : 1, sizeof(*Um));
  for (uint32_t i = 0; i < n_obj; ++i) {
    uint64_t ne = n_elems_of(&objs[i]);
    Wm[objs[i].id] = (unsigned char*)calloc(ne, 1);
    Lm[objs[i].id] = (unsigned char*)calloc(ne, 1);
    Um[objs[i].id] = (unsigned char*)calloc(ne, 1);
  }

  hent* pairs = (hent*)malloc(sizeof(hent) * (2 * n + 1));
  uint64_t n_pairs = 0;
  line_acc* la = (line_acc*)calloc(n_keys, sizeof(line_acc));

  glob->n_records = n;
  /* pass 1: sums, min/max, histogram pairs, extreme-x points */
  for (uint64_t i = 0; i < n; ++i) {
    const vo_record* r = &recs[i];
    dec_t d;
    decode(cfg, &t, r, &d);
    if (!d.valid) { glob->n_invalid++; continue; }
    if (!d.shared && !d.obj) glob->n_unmapped++;

    uint64_t kset[2];
    int nk = 0;
    kset[nk++] = r->pc;                                    /* PC key */
    if (d.shared) kset[nk++] = key_shared;                 /* Q20 */
    else if (d.obj) kset[nk++] = (uint64_t)cfg->n_pcs + d.obj->id;

    uint64_t ord = vo_ord(r->value, d.kind, d.w);
    int is_nan = (d.fflags & 1u) != 0;
    for (int j = 0; j < nk; ++j) {
      vo_key* k = &keys[kset[j]];
      if (d.store) k->n_st++; else k->n_ld++;
      if (r->value == 0) k->n_zero++;                      /* Q8: bitwise zero */
      if (d.eq_defined) {
        if (d.eq_pre) { if (d.store) k->n_st_eq_pre++; else k->n_ld_eq_pre++; }
      } else {
        k->n_nosnap++;
      }
      k->n_type[d.tc]++;
      if (d.kind >= 2) {
        if (d.fflags & 1u) k->n_nan++;
        if (d.fflags & 2u) k->n_nonint++;
        if (d.fflags & 4u) k->n_not_f16++;
        if (d.fflags & 8u) k->n_not_bf16++;
        if (d.fflags & 16u) k->n_not_f32++;
      }
      if (r->value < k->raw_min) k->raw_min = r->value;
      if (r->value > k->raw_max) k->raw_max = r->value;
      if (!is_nan) {
        if (ord < k->ord_min) k->ord_min = ord;
        if (ord > k->ord_max) k->ord_max = ord;
      }
      if (d.kind >= 2 && !is_nan) {
        uint64_t tb = vo_trunc(r->value, d.kind, d.w, cfg->mant_bits);
        if (tb < k->trunc_min) k->trunc_min = tb;
        if (tb > k->trunc_max) k->trunc_max = tb;
      }
      pairs[n_pairs].key = kset[j];
      pairs[n_pairs].bits = r->value;
      pairs[n_pairs].count = 1;
      n_pairs++;

      line_acc* L = &la[kset[j]];
      i128 y;
      if (!point_y(r->value, d.kind, d.w, d.fflags, &y)) { L->fail = 1; continue; }
      if (!L->have) {
        L->have = 1; L->px = L->qx = r->addr; L->py = L->qy = y;
      } else {
        if (r->addr < L->px) { L->px = r->addr; L->py = y; }
        if (r->addr > L->qx) { L->qx = r->addr; L->qy = y; }
      }
    }

    /* per-object marks (C3, C10) */
    if (d.obj && d.inside) {
      const vo_object* o = d.obj;
      uint64_t off = r->addr - o->base;
      uint64_t e0 = off / o->elem_width, e1 = (off + d.w - 1) / o->elem_width;
      if (d.store)
        for (uint64_t e = e0; e <= e1; ++e) Wm[o->id][e] = 1;
      if (!d.store && d.eq_pre) Lm[o->id][e0] = 1;
      if (d.eq_defined)
        for (uint64_t e = e0; e <= e1; ++e) Um[o->id][e] = 1;
    }
  }

  /* pass 2: every point against the extreme-x pair (C8) */
  for (uint64_t i = 0; i < n; ++i) {
    const vo_record* r = &recs[i];
    dec_t d;
    decode(cfg, &t, r, &d);
    if (!d.valid) continue;
    uint64_t kset[2];
    int nk = 0;
    kset[nk++] = r->pc;
    if (d.shared) kset[nk++] = key_shared;
    else if (d.obj) kset[nk++] = (uint64_t)cfg->n_pcs + d.obj->id;
    for (int j = 0; j < nk; ++j) {
      line_acc* L = &la[kset[j]];
      if (L->fail) continue;
      i128 y;
      if (!point_y(r->value, d.kind, d.w, d.fflags, &y)) { L->fail = 1; continue; }
      if (L->px == L->qx) {
        if (y != L->py) L->fail = 1;               /* same x, different y */
      } else if (!collinear((i128)L->px, L->py, (i128)L->qx, L->qy, (i128)r->addr, y)) {
        L->fail = 1;
      }
    }
  }
  for (uint64_t k = 0; k < n_keys; ++k) {
    line_acc* L = &la[k];
    vo_key* K = &keys[k];
    if (L->fail) K->line_state = VO_LINE_FAIL;
    else if (!L->have) K->line_state = VO_LINE_EMPTY;
    else {
      K->line_state = (L->px == L->qx) ? VO_LINE_POINT : VO_LINE_LINE;
      K->p_x = L->px; K->q_x = L->qx;
      K->p_ylo = (uint64_t)L->py; K->p_yhi = (int64_t)(L->py >> 64);
      K->q_ylo = (uint64_t)L->qy; K->q_yhi = (int64_t)(L->qy >> 64);
    }
  }
  free(la);

  /* C9: exact histogram = sort (key, bits) + run-length, then top-k by
   * (count desc, bits asc) */
  qsort(pairs, n_pairs, sizeof(hent), cmp_key_bits);
  uint64_t n_runs = 0;
  for (uint64_t i = 0; i < n_pairs;) {
    uint64_t j = i;
    while (j < n_pairs && pairs[j].key == pairs[i].key && pairs[j].bits == pairs[i].bits) ++j;
    pairs[n_runs].key = pairs[i].key;
    pairs[n_runs].bits = pairs[i].bits;
    pairs[n_runs].count = j - i;
    ++n_runs;
    i = j;
  }
  qsort(pairs, n_runs, sizeof(hent), cmp_key_count_bits);
  for (uint64_t i = 0; i < n_runs; ++i) {
    vo_key* K = &keys[pairs[i].key];
    if (K->n_distinct < cfg->topk) {
      K->top_bits[K->n_distinct] = pairs[i].bits;
      K->top_count[K->n_distinct] = pairs[i].count;
      K->n_top = K->n_distinct + 1;
    }
    K->n_distinct++;
  }
  free(pairs);

  for (uint64_t k = 0; k < n_keys; ++k) derive_flags(cfg, &keys[k]);

  /* C3 per object, and U */
  for (uint32_t i = 0; i < n_obj; ++i) {
    uint32_t id = objs[i].id;
    uint64_t ne = n_elems_of(&objs[i]);
    vo_objstat* s = &objstat[id];
    memset(s, 0, sizeof(*s));
    s->n_elems = ne;
    for (uint64_t e = 0; e < ne; ++e) {
      s->n_written += Wm[id][e];
      s->n_loaded_eq += Lm[id][e];
      s->n_touched += (Wm[id][e] | Lm[id][e]);
      glob->u_touched += Um[id][e];
    }
    s->n_ld_reload = keys[(uint64_t)cfg->n_pcs + id].n_ld_eq_pre - s->n_loaded_eq;
    free(Wm[id]); free(Lm[id]); free(Um[id]);
  }
  free(Wm); free(Lm); free(Um);
  free(t.by_base);
  return 0;
}

/* ---- C10: snapshot diff (Def 3.1; footnote P:L267) */

int vo_snapshot_diff(const vo_config* cfg, const vo_object* objs, uint32_t n_obj,
                     const vo_record* recs, uint64_t n, uint32_t obj_id,
                     uint32_t mode, const uint32_t* mask, vo_diff* out) {
  objtab t;
  if (objtab_build(&t, objs, n_obj) != 0) return -1;
  const vo_object* o = NULL;
  for (uint32_t i = 0; i < n_obj; ++i) if (objs[i].id == obj_id) o = &objs[i];
  if (!o || !o->pre || !o->post || mode > VO_DIFF_MASK || (mode == VO_DIFF_MASK && !mask)) {
    free(t.by_base);
    return -1;
  }
  uint64_t ne = n_elems_of(o);
  unsigned char* W = (unsigned char*)calloc(ne, 1);
  unsigned char* L = (unsigned char*)calloc(ne, 1);
  for (uint64_t i = 0; i < n; ++i) {
    dec_t d;
    decode(cfg, &t, &recs[i], &d);
    if (!d.valid || d.obj != o || !d.inside) continue;
    uint64_t off = recs[i].addr - o->base;
    uint64_t e0 = off / o->elem_width, e1 = (off + d.w - 1) / o->elem_width;
    if (d.store) for (uint64_t e = e0; e <= e1; ++e) W[e] = 1;
    if (!d.store && d.eq_pre) L[e0] = 1;
  }
  memset(out, 0, sizeof(*out));
  out->n_elems = ne;
  uint64_t touched = 0;
  for (uint64_t e = 0; e < ne; ++e) {
    int m = (mode == VO_DIFF_ALL) ? 1 : (mode == VO_DIFF_WRITTEN) ? W[e] : (int)((mask[e / 32] >> (e % 32)) & 1u);
    touched += (W[e] | L[e]);
    if (!m) continue;
    out->n_masked++;
    uint64_t b0 = e * o->elem_width;
    uint64_t len = (b0 + o->elem_width <= o->size) ? o->elem_width : o->size - b0;
    if (memcmp(o->pre + b0, o->post + b0, len) == 0) out->n_unchanged++;
  }
  out->n_changed = out->n_masked - out->n_unchanged;
  out->n_untouched = ne - touched;
  out->redundant = (out->n_masked > 0 &&
                    (unsigned __int128)100 * out->n_unchanged >
                        (unsigned __int128)cfg->t_redundant_pct * out->n_masked);
  free(W); free(L); free(t.by_base);
  return 0;
}

/* ---- C11: duplicate objects (Def 3.2; Q17) --------------- */

int vo_object_dedup(const vo_object* objs, uint32_t n, uint32_t* group_of) {
  for (uint32_t i = 0; i < n; ++i) {
    group_of[i] = objs[i].id;
    if (objs[i].size == 0 || !objs[i].post) continue;
    for (uint32_t j = 0; j < n; ++j) {
      if (objs[j].size != objs[i].size || !objs[j].post) continue;
      if (objs[j].id < group_of[i] && memcmp(objs[i].post, objs[j].post, objs[i].size) == 0)
        group_of[i] = objs[j].id;
    }
  }
  return 0;
}

/* ---- C18-C20: value flow graph (f4; Defs 5.1-5.3) ------------- */

enum { VO_ACC_R = 1, VO_ACC_W = 2, VO_EV_DEV = 0, VO_EV_ALLOC = 1, VO_EV_H2D = 2, VO_EV_D2H = 3 };

static int vo_writes(const vo_access* a, uint32_t k) {
  return a->object == k && (a->kind == VO_EV_ALLOC || a->kind == VO_EV_H2D || (a->kind == VO_EV_DEV && (a->mode & VO_ACC_W)));
}

static void vo_edge_add(vo_vfg_edge* E, uint64_t* ne, uint64_t* last, uint32_t src, uint32_t dst, uint32_t k,
                        uint32_t label, uint64_t bytes, uint64_t seq) {
  for (uint64_t i = 0; i < *ne; ++i)
    if (E[i].src == src && E[i].dst == dst && E[i].object == k) {
      E[i].label |= label;
      E[i].bytes += bytes;
      if (last[i] != seq) { E[i].count++; last[i] = seq; }
      return;
    }
  E[*ne].src = src; E[*ne].dst = dst; E[*ne].object = k; E[*ne].label = label;
  E[*ne].bytes = bytes; E[*ne].count = 1;
  last[*ne] = seq;
  (*ne)++;
}

static int cmp_edge(const void* a, const void* b) {
  const vo_vfg_edge* x = (const vo_vfg_edge*)a;
  const vo_vfg_edge* y = (const vo_vfg_edge*)b;
  if (x->src != y->src) return (x->src > y->src) - (x->src < y->src);
  if (x->dst != y->dst) return (x->dst > y->dst) - (x->dst < y->dst);
  return (x->object > y->object) - (x->object < y->object);
}
static int cmp_vertex(const void* a, const void* b) {
  const vo_vfg_vertex* x = (const vo_vfg_vertex*)a;
  const vo_vfg_vertex* y = (const vo_vfg_vertex*)b;
  return (x->vertex > y->vertex) - (x->vertex < y->vertex);
}

int vo_vfg_build(const vo_access* log, uint64_t n, vo_vfg_edge* edges, uint64_t* ne, vo_vfg_vertex* verts,
                 uint64_t* nv) {
  uint64_t* last = (uint64_t*)malloc(sizeof(uint64_t) * (2 * n + 1));
  *ne = 0;
  *nv = 0;
  for (uint64_t j = 0; j < n; ++j) {
    const vo_access* a = &log[j];
    /* I(v): the number of distinct invocations (sequence numbers) of the vertex */
    int first = 1;
    for (uint64_t i = 0; i < j; ++i)
      if (log[i].vertex == a->vertex && log[i].seq == a->seq) first = 0;
    if (first) {
      uint64_t q = 0;
      while (q < *nv && verts[q].vertex != a->vertex) ++q;
      if (q == *nv) { verts[q].vertex = a->vertex; verts[q].pad = 0; verts[q].invocations = 0; (*nv)++; }
      verts[q].invocations++;
    }
    if (a->kind == VO_EV_ALLOC) continue;
    /* Def 5.1: v_i writes D_k and no v_u writes D_k after it and before v_j */
    int64_t w = -1;
    for (int64_t i = (int64_t)j - 1; i >= 0; --i)
      if (log[i].seq < a->seq && vo_writes(&log[i], a->object)) { w = i; break; }
    if (w < 0) { free(last); return -1; }
    uint32_t mode = a->mode & (VO_ACC_R | VO_ACC_W);
    if (a->kind == VO_EV_H2D) mode = VO_ACC_W;
    if (a->kind == VO_EV_D2H) mode = VO_ACC_R;
    vo_edge_add(edges, ne, last, log[w].vertex, a->vertex, a->object, mode, a->bytes, a->seq);
    if (a->kind == VO_EV_H2D) vo_edge_add(edges, ne, last, VO_HOST, a->vertex, a->object, VO_ACC_W, a->bytes, a->seq);
    if (a->kind == VO_EV_D2H) vo_edge_add(edges, ne, last, a->vertex, VO_HOST, a->object, VO_ACC_R, a->bytes, a->seq);
  }
  free(last);
  qsort(edges, *ne, sizeof(vo_vfg_edge), cmp_edge);
  qsort(verts, *nv, sizeof(vo_vfg_vertex), cmp_vertex);
  return 0;
}

static int in_set(const uint32_t* s, uint64_t n, uint32_t x) {
  for (uint64_t i = 0; i < n; ++i) if (s[i] == x) return 1;
  return 0;
}

static void vo_keep_vertices(const vo_vfg_edge* oe, uint64_t one, const vo_vfg_vertex* verts, uint64_t nv,
                             vo_vfg_vertex* ov, uint64_t* onv, uint64_t min_inv) {
  *onv = 0;
  for (uint64_t q = 0; q < nv; ++q) {
    int on = verts[q].invocations >= min_inv;
    for (uint64_t i = 0; i < one && !on; ++i) on = oe[i].src == verts[q].vertex || oe[i].dst == verts[q].vertex;
    if (on) ov[(*onv)++] = verts[q];
  }
}

int vo_vfg_slice(const vo_vfg_edge* edges, uint64_t ne, const vo_vfg_vertex* verts, uint64_t nv, uint32_t v,
                 vo_vfg_edge* oe, uint64_t* one, vo_vfg_vertex* ov, uint64_t* onv) {
  *one = 0;
  uint32_t* rin = (uint32_t*)malloc(sizeof(uint32_t) * (2 * ne + 2));
  uint32_t* rout = (uint32_t*)malloc(sizeof(uint32_t) * (2 * ne + 2));
  for (uint64_t e0 = 0; e0 < ne; ++e0) {                 /* every object v reads or writes */
    if (edges[e0].src != v && edges[e0].dst != v) continue;
    const uint32_t k = edges[e0].object;
    int dup = 0;
    for (uint64_t e1 = 0; e1 < e0; ++e1)
      if ((edges[e1].src == v || edges[e1].dst == v) && edges[e1].object == k) dup = 1;
    if (dup) continue;
    uint64_t nin = 1, nout = 1;
    rin[0] = v; rout[0] = v;
    for (int changed = 1; changed;) {                    /* fixpoint: vertices with a D_k path to v */
      changed = 0;
      for (uint64_t i = 0; i < ne; ++i)
        if (edges[i].object == k && in_set(rin, nin, edges[i].dst) && !in_set(rin, nin, edges[i].src)) {
          rin[nin++] = edges[i].src;
          changed = 1;
        }
    }
    for (int changed = 1; changed;) {                    /* ... and with a D_k path from v */
      changed = 0;
      for (uint64_t i = 0; i < ne; ++i)
        if (edges[i].object == k && in_set(rout, nout, edges[i].src) && !in_set(rout, nout, edges[i].dst)) {
          rout[nout++] = edges[i].dst;
          changed = 1;
        }
    }
    for (uint64_t i = 0; i < ne; ++i)
      if (edges[i].object == k && (in_set(rin, nin, edges[i].dst) || in_set(rout, nout, edges[i].src)))
        oe[(*one)++] = edges[i];
  }
  free(rin);
  free(rout);
  qsort(oe, *one, sizeof(vo_vfg_edge), cmp_edge);
  vo_keep_vertices(oe, *one, verts, nv, ov, onv, ~0ull);
  return 0;
}

int vo_vfg_important(const vo_vfg_edge* edges, uint64_t ne, const vo_vfg_vertex* verts, uint64_t nv,
                     uint64_t min_edge_bytes, uint64_t min_vertex_invocations,
                     vo_vfg_edge* oe, uint64_t* one, vo_vfg_vertex* ov, uint64_t* onv) {
  *one = 0;
  for (uint64_t i = 0; i < ne; ++i)
    if (edges[i].bytes >= min_edge_bytes) oe[(*one)++] = edges[i];
  vo_keep_vertices(oe, *one, verts, nv, ov, onv, min_vertex_invocations);
  return 0;
}

/* ---- C17: LoadSpy temporal load redundancy in record order (f3; Q1, R6) ----
 * The definition, walked in record order with a table of the last load seen at
 * every address (open addressing on the address; a plain map). */
typedef struct { uint64_t addr; uint64_t value; uint32_t w; uint32_t used; } lastload;

int vo_temporal_loads(const vo_config* cfg, const vo_object* objs, uint32_t n_obj, const vo_record* recs,
                      uint64_t n, uint64_t* out) {
  if (!cfg || cfg->n_pcs == 0) return -1;
  objtab t;
  if (objtab_build(&t, objs, n_obj) != 0) return -1;
  const uint64_t n_keys = (uint64_t)cfg->n_pcs + n_obj + 1;
  memset(out, 0, sizeof(uint64_t) * 2 * n_keys);
  uint64_t cap = 16;
  while (cap < 2 * n + 2) cap <<= 1;
  lastload* tab = (lastload*)calloc(cap, sizeof(lastload));
  for (uint64_t i = 0; i < n; ++i) {
    const vo_record* r = &recs[i];
    dec_t d;
    decode(cfg, &t, r, &d);
    if (!d.valid || d.shared || d.store) continue;
    uint64_t h = (r->addr * 0x9E3779B97F4A7C15ull) >> 17 & (cap - 1);
    while (tab[h].used && tab[h].addr != r->addr) h = (h + 1) & (cap - 1);
    if (tab[h].used) {                                     /* r' = the last load of this address */
      const int red = tab[h].w == d.w && tab[h].value == r->value;
      out[2 * r->pc]++;
      out[2 * r->pc + 1] += red;
      if (d.obj) {
        const uint64_t ko = (uint64_t)cfg->n_pcs + d.obj->id;
        out[2 * ko]++;
        out[2 * ko + 1] += red;
      }
    }
    tab[h].used = 1;
    tab[h].addr = r->addr;
    tab[h].value = r->value;
    tab[h].w = d.w;
  }
  free(tab);
  free(t.by_base);
  return 0;
}

/* ---- C16: approximate frequent values (f2; Def 3.3 over Def 3.8) ---------- */

int vo_approx_topk(const vo_config* cfg, const vo_object* objs, uint32_t n_obj, const vo_record* recs,
                   uint64_t n, uint64_t* ndistinct, uint64_t* top_bits, uint64_t* top_count) {
  if (!cfg || cfg->topk > VO_MAX_TOPK || cfg->n_pcs == 0) return -1;
  objtab t;
  if (objtab_build(&t, objs, n_obj) != 0) return -1;
  const uint64_t n_keys = (uint64_t)cfg->n_pcs + n_obj + 1;
  const uint64_t key_shared = (uint64_t)cfg->n_pcs + n_obj;
  const uint32_t K = cfg->topk;
  memset(ndistinct, 0, sizeof(uint64_t) * n_keys);
  memset(top_bits, 0, sizeof(uint64_t) * n_keys * K);
  memset(top_count, 0, sizeof(uint64_t) * n_keys * K);
  /* pass 1: the type codes of every key (Q15: one type only) */
  uint32_t* types = (uint32_t*)calloc(n_keys, sizeof(uint32_t));   /* bit tc set if seen */
  for (uint64_t i = 0; i < n; ++i) {
    dec_t d;
    decode(cfg, &t, &recs[i], &d);
    if (!d.valid) continue;
    types[recs[i].pc] |= 1u << d.tc;
    if (d.shared) types[key_shared] |= 1u << d.tc;
    else if (d.obj) types[(uint64_t)cfg->n_pcs + d.obj->id] |= 1u << d.tc;
  }
  /* pass 2: (key, truncated bits) of every record of a single-float-type key */
  hent* pairs = (hent*)malloc(sizeof(hent) * (2 * n + 1));
  uint64_t np = 0;
  for (uint64_t i = 0; i < n; ++i) {
    const vo_record* r = &recs[i];
    dec_t d;
    decode(cfg, &t, r, &d);
    if (!d.valid || d.kind < 2) continue;
    uint64_t kset[2];
    int nk = 0;
    kset[nk++] = r->pc;
    if (d.shared) kset[nk++] = key_shared;
    else if (d.obj) kset[nk++] = (uint64_t)cfg->n_pcs + d.obj->id;
    /* R5: NaNs keep their bits (clearing mantissa bits could turn a NaN into an infinity) */
    uint64_t tb = (d.fflags & 1u) ? r->value : vo_trunc(r->value, d.kind, d.w, cfg->mant_bits);
    for (int j = 0; j < nk; ++j) {
      if (types[kset[j]] != (1u << d.tc)) continue;          /* mixed types: no approximate histogram */
      pairs[np].key = kset[j];
      pairs[np].bits = tb;
      pairs[np].count = 1;
      ++np;
    }
  }
  qsort(pairs, np, sizeof(hent), cmp_key_bits);
  uint64_t nr = 0;
  for (uint64_t i = 0; i < np;) {
    uint64_t j = i;
    while (j < np && pairs[j].key == pairs[i].key && pairs[j].bits == pairs[i].bits) ++j;
    pairs[nr].key = pairs[i].key;
    pairs[nr].bits = pairs[i].bits;
    pairs[nr].count = j - i;
    ++nr;
    i = j;
  }
  qsort(pairs, nr, sizeof(hent), cmp_key_count_bits);
  for (uint64_t i = 0; i < nr; ++i) {
    const uint64_t k = pairs[i].key;
    if (ndistinct[k] < K) {
      top_bits[k * K + ndistinct[k]] = pairs[i].bits;
      top_count[k * K + ndistinct[k]] = pairs[i].count;
    }
    ndistinct[k]++;
  }
  free(pairs);
  free(types);
  free(t.by_base);
  return 0;
}

/* ---- C13-C15: accessed intervals and the adaptive copy plan ---------------
 * PAPER.md 6.1.  The merged set is the definition itself: sort
 * the intervals by start and sweep, extending the current run while the next
 * interval starts at or before (run end + 1) -- "adjacent or overlapped"
 * (P:L305).  This is the textbook sequential merge the paper names as the CPU
 * alternative (O(N log N)); tests pin it against brute-force byte
 * coverage and against a literal transcription of Figure 4's steps 1-9. */

static int cmp_interval(const void* a, const void* b) {
  const vo_interval* x = (const vo_interval*)a;
  const vo_interval* y = (const vo_interval*)b;
  if (x->start != y->start) return (x->start > y->start) - (x->start < y->start);
  return (x->end > y->end) - (x->end < y->end);
}

uint64_t vo_interval_merge(const vo_interval* in, uint64_t n, vo_interval* out) {
  vo_interval* v = (vo_interval*)malloc(sizeof(*v) * (n ? n : 1));
  uint64_t m = 0;
  for (uint64_t i = 0; i < n; ++i)
    if (in[i].start <= in[i].end) v[m++] = in[i];      /* R1: start > end is the empty set */
  qsort(v, m, sizeof(*v), cmp_interval);
  uint64_t k = 0;
  for (uint64_t i = 0; i < m; ++i) {
    if (k > 0 && (out[k - 1].end == UINT64_MAX || v[i].start <= out[k - 1].end + 1)) {
      if (v[i].end > out[k - 1].end) out[k - 1].end = v[i].end;   /* overlapped or adjacent */
    } else {
      out[k++] = v[i];
    }
  }
  free(v);
  return k;
}

uint64_t vo_record_intervals(uint32_t n_pcs, const vo_record* recs, uint64_t n, vo_interval* out) {
  vo_interval* v = (vo_interval*)malloc(sizeof(*v) * (n ? n : 1));
  uint64_t m = 0;
  for (uint64_t i = 0; i < n; ++i) {
    if (!rec_valid(&recs[i], n_pcs) || rec_shared(recs[i].meta)) continue;   /* R2 */
    v[m].start = recs[i].addr;
    v[m].end = recs[i].addr + rec_w(recs[i].meta) - 1;
    ++m;
  }
  uint64_t k = vo_interval_merge(v, m, out);
  free(v);
  return k;
}

int vo_plan_copies(const vo_object* objs, uint32_t n_obj, const vo_interval* merged, uint64_t n,
                 uint32_t seg_max, uint32_t dense_pct, vo_copy_plan* plan) {
  for (uint32_t j = 0; j < n_obj; ++j) {
    const vo_object* o = &objs[j];
    if (o->id >= n_obj || o->size == 0) return -1;
    vo_copy_plan* p = &plan[o->id];
    memset(p, 0, sizeof(*p));
    p->lo = UINT64_MAX;
    p->direct_bytes = o->size;
    const uint64_t ob = o->base, oe = o->base + o->size - 1;
    for (uint64_t i = 0; i < n; ++i) {                  /* R3: clip every merged interval */
      if (merged[i].end < ob || merged[i].start > oe) continue;
      uint64_t s = merged[i].start > ob ? merged[i].start : ob;
      uint64_t e = merged[i].end < oe ? merged[i].end : oe;
      p->n_segments++;
      p->accessed_bytes += e - s + 1;
      if (s < p->lo) p->lo = s;
      if (e > p->hi) p->hi = e;
    }
    if (p->n_segments == 0) {
      p->lo = 0;
      p->choice = VO_COPY_NONE;
      continue;
    }
    p->minmax_bytes = p->hi - p->lo + 1;
    /* R4: segment copy when sparse AND few intervals, else min-max */
    int sparse = (unsigned __int128)100 * p->accessed_bytes < (unsigned __int128)dense_pct * p->minmax_bytes;
    p->choice = (sparse && p->n_segments <= seg_max) ? VO_COPY_SEGMENT : VO_COPY_MINMAX;
  }
  return 0;
}

/* struct sizes, for the ctypes harness to check its mirrors */
uint64_t vo_sizeof(int which) {
  switch (which) {
    case 0: return sizeof(vo_key);
    case 1: return sizeof(vo_globals);
    case 2: return sizeof(vo_objstat);
    case 3: return sizeof(vo_diff);
    case 4: return sizeof(vo_object);
    case 6: return sizeof(vo_copy_plan);
    default: return sizeof(vo_record);
  }
}

/* ---- C21: dyadic-scaled exact linear fit (f2; Def 3.7 P:L187-L189 over exact float values) ----
 * DESIGN.md reading R10.  Every valid record of a key is a point (x = addr, y = the exact real
 * value of its bits: integers as such, floats as the dyadic rational (-1)^s M 2^E they encode).
 * The key is a *dyadic line* when all points lie on one straight line.  Steps, in order:
 *  1. NaN or infinity among the key's records -> FAIL;
 *  2. T = the largest number of fractional bits of any y (0 for integers), so that every
 *     Y = y 2^T is an integer; some |Y| >= 2^62 -> FAIL (the bound of the exact check);
 *  3. P = (min x, smallest Y at that x), Q = (max x, smallest Y at that x);
 *  4. every point collinear with P and Q (exact 128-bit cross product), and a point at P.x or
 *     Q.x equal to that anchor (one value per address) -> LINE (POINT when P.x == Q.x), else FAIL.  No valid record -> EMPTY. */

/* exact value of a record as M * 2^E with M odd (or M = 0, E = 0); returns 0 for NaN / inf */
static int exact_value(uint64_t b, uint32_t kind, uint32_t w, int64_t* M, int* E) {
  if (kind == 0 || kind == 1) {
    if (kind == 0 && b >= (1ull << 63)) { *M = INT64_MAX; *E = 0; return 1; }   /* overflows step 2 */
    *M = (kind == 0) ? (int64_t)b : sext(b, w);
    *E = 0;
  } else {
    int eb, mb;
    if (kind == 3) { eb = 8; mb = 7; }
    else if (w == 2) { eb = 5; mb = 10; }
    else if (w == 4) { eb = 8; mb = 23; }
    else { eb = 11; mb = 52; }
    const uint64_t sign = (b >> (eb + mb)) & 1u;
    const uint64_t ex = (b >> mb) & ((1ull << eb) - 1);
    const uint64_t man = b & ((1ull << mb) - 1);
    const int bias = (1 << (eb - 1)) - 1;
    if (ex == (1ull << eb) - 1) return 0;                  /* inf / NaN */
    uint64_t sig;
    int e2;
    if (ex == 0) { sig = man; e2 = 1 - bias - mb; }         /* zero / subnormal */
    else { sig = man | (1ull << mb); e2 = (int)ex - bias - mb; }
    *M = sign ? -(int64_t)sig : (int64_t)sig;
    *E = e2;
  }
  if (*M == 0) { *E = 0; return 1; }
  while ((*M & 1) == 0) { *M /= 2; *E += 1; }
  return 1;
}

/* Y = M 2^s (s >= 0); returns 0 if |Y| >= 2^62 */
static int scaled_y(int64_t M, int s, i128* Y) {
  if (M == 0) { *Y = 0; return 1; }
  const uint64_t a = M < 0 ? (uint64_t)(-(M + 1)) + 1u : (uint64_t)M;
  int bits = 64 - __builtin_clzll(a);
  if (bits + s > 62) return 0;
  *Y = (i128)M * ((i128)1 << s);
  return 1;
}

int vo_dyadic_fit(const vo_config* cfg, const vo_object* objs, uint32_t n_obj, const vo_record* recs, uint64_t n,
                  vo_dyadic* out) {
  if (!cfg || cfg->n_pcs == 0) return -1;
  objtab t;
  if (objtab_build(&t, objs, n_obj) != 0) return -1;
  const uint64_t n_keys = (uint64_t)cfg->n_pcs + n_obj + 1;
  int* have = (int*)calloc(n_keys, sizeof(int));
  int* fail = (int*)calloc(n_keys, sizeof(int));
  int* T = (int*)calloc(n_keys, sizeof(int));
  int* hp = (int*)calloc(n_keys, sizeof(int));
  int* hq = (int*)calloc(n_keys, sizeof(int));
  i128* py = (i128*)calloc(n_keys, sizeof(i128));
  i128* qy = (i128*)calloc(n_keys, sizeof(i128));
  memset(out, 0, sizeof(vo_dyadic) * n_keys);
  for (int pass = 1; pass <= 3; ++pass) {
    for (uint64_t i = 0; i < n; ++i) {
      const vo_record* r = &recs[i];
      dec_t d;
      decode(cfg, &t, r, &d);
      if (!d.valid) continue;
      uint64_t kset[2];
      int nk = 0;
      kset[nk++] = r->pc;                                  /* PC key, object key as in C1 */
      if (d.shared) kset[nk++] = (uint64_t)cfg->n_pcs + n_obj;
      else if (d.obj) kset[nk++] = (uint64_t)cfg->n_pcs + d.obj->id;
      int64_t M = 0;
      int E = 0;
      const int finite = exact_value(r->value, d.kind, d.w, &M, &E);
      for (int j = 0; j < nk; ++j) {
        const uint64_t k = kset[j];
        vo_dyadic* o = &out[k];
        if (pass == 1) {                                   /* step 1, T of step 2, extreme x */
          if (!finite) { fail[k] = 1; continue; }
          if (-E > T[k]) T[k] = -E;
          if (!have[k] || r->addr < o->px) o->px = r->addr;
          if (!have[k] || r->addr > o->qx) o->qx = r->addr;
          have[k] = 1;
          continue;
        }
        if (fail[k]) continue;
        i128 Y;
        if (!scaled_y(M, E + T[k], &Y)) { fail[k] = 1; continue; }   /* step 2 bound */
        if (pass == 2) {                                   /* step 3: anchors */
          if (r->addr == o->px && (!hp[k] || Y < py[k])) { py[k] = Y; hp[k] = 1; }
          if (r->addr == o->qx && (!hq[k] || Y < qy[k])) { qy[k] = Y; hq[k] = 1; }
        } else if (!collinear((i128)o->px, py[k], (i128)o->qx, qy[k], (i128)r->addr, Y) ||
                   (r->addr == o->px && Y != py[k]) || (r->addr == o->qx && Y != qy[k])) {
          fail[k] = 1;                                     /* step 4 (one value per x) */
        }
      }
    }
  }
  for (uint64_t k = 0; k < n_keys; ++k) {
    vo_dyadic* o = &out[k];
    if (fail[k] || !have[k]) {
      memset(o, 0, sizeof(*o));
      o->state = fail[k] ? VO_LINE_FAIL : VO_LINE_EMPTY;
      continue;
    }
    o->state = (o->px == o->qx) ? VO_LINE_POINT : VO_LINE_LINE;
    o->scale = (uint32_t)T[k];
    o->py = (int64_t)py[k];
    o->qy = (int64_t)qy[k];
  }
  free(hp); free(hq);
  free(have); free(fail); free(T); free(py); free(qy);
  free(t.by_base);
  return 0;
}

/* ---- C22: approximate structured (f2; Def 3.7 over Def 3.8's truncated values) ----------------
 * DESIGN.md reading R11 (SURVEY 8(f) f2 "approximate structured").  Exactly C21 (vo_dyadic_fit),
 * step for step, over the values every float record carries after Def 3.8's truncation to K
 * mantissa bits (C7: clear the low m-K mantissa bits, toward zero); integer records unchanged.
 * A NaN or infinity in the record fails the key (truncation keeps a finite value finite). */
static int trunc_exact_value(uint64_t b, uint32_t kind, uint32_t w, uint32_t K, int trunc, int64_t* M, int* E) {
  if (trunc && kind >= 2) {
    int64_t m0;
    int e0;
    if (!exact_value(b, kind, w, &m0, &e0)) return 0;      /* NaN / inf in the record itself */
    b = vo_trunc(b, kind, w, K);
  }
  return exact_value(b, kind, w, M, E);
}

int vo_dyadic_fit_trunc(const vo_config* cfg, const vo_object* objs, uint32_t n_obj, const vo_record* recs,
                        uint64_t n, vo_dyadic* out) {
  if (!cfg || cfg->n_pcs == 0) return -1;
  objtab t;
  if (objtab_build(&t, objs, n_obj) != 0) return -1;
  const uint64_t n_keys = (uint64_t)cfg->n_pcs + n_obj + 1;
  int* have = (int*)calloc(n_keys, sizeof(int));
  int* fail = (int*)calloc(n_keys, sizeof(int));
  int* T = (int*)calloc(n_keys, sizeof(int));
  int* hp = (int*)calloc(n_keys, sizeof(int));
  int* hq = (int*)calloc(n_keys, sizeof(int));
  i128* py = (i128*)calloc(n_keys, sizeof(i128));
  i128* qy = (i128*)calloc(n_keys, sizeof(i128));
  memset(out, 0, sizeof(vo_dyadic) * n_keys);
  for (int pass = 1; pass <= 3; ++pass) {
    for (uint64_t i = 0; i < n; ++i) {
      const vo_record* r = &recs[i];
      dec_t d;
      decode(cfg, &t, r, &d);
      if (!d.valid) continue;
      uint64_t kset[2];
      int nk = 0;
      kset[nk++] = r->pc;
      if (d.shared) kset[nk++] = (uint64_t)cfg->n_pcs + n_obj;
      else if (d.obj) kset[nk++] = (uint64_t)cfg->n_pcs + d.obj->id;
      int64_t M = 0;
      int E = 0;
      const int finite = trunc_exact_value(r->value, d.kind, d.w, cfg->mant_bits, 1, &M, &E);
      for (int j = 0; j < nk; ++j) {
        const uint64_t k = kset[j];
        vo_dyadic* o = &out[k];
        if (pass == 1) {
          if (!finite) { fail[k] = 1; continue; }
          if (-E > T[k]) T[k] = -E;
          if (!have[k] || r->addr < o->px) o->px = r->addr;
          if (!have[k] || r->addr > o->qx) o->qx = r->addr;
          have[k] = 1;
          continue;
        }
        if (fail[k]) continue;
        i128 Y;
        if (!scaled_y(M, E + T[k], &Y)) { fail[k] = 1; continue; }
        if (pass == 2) {
          if (r->addr == o->px && (!hp[k] || Y < py[k])) { py[k] = Y; hp[k] = 1; }
          if (r->addr == o->qx && (!hq[k] || Y < qy[k])) { qy[k] = Y; hq[k] = 1; }
        } else if (!collinear((i128)o->px, py[k], (i128)o->qx, qy[k], (i128)r->addr, Y) ||
                   (r->addr == o->px && Y != py[k]) || (r->addr == o->qx && Y != qy[k])) {
          fail[k] = 1;
        }
      }
    }
  }
  for (uint64_t k = 0; k < n_keys; ++k) {
    vo_dyadic* o = &out[k];
    if (fail[k] || !have[k]) {
      memset(o, 0, sizeof(*o));
      o->state = fail[k] ? VO_LINE_FAIL : VO_LINE_EMPTY;
      continue;
    }
    o->state = (o->px == o->qx) ? VO_LINE_POINT : VO_LINE_LINE;
    o->scale = (uint32_t)T[k];
    o->py = (int64_t)py[k];
    o->qy = (int64_t)qy[k];
  }
  free(hp); free(hq);
  free(have); free(fail); free(T); free(py); free(qy);
  free(t.by_base);
  return 0;
}

/* ---- C23: structured with <= eps outliers (f2; Def 3.7, srad_v1's clamped boundary) -----------
 * DESIGN.md reading R12.  Points as in C21 (x = addr, exact value y, Y = y 2^T; with flags & 1 the
 * float values truncated as in C22).  Steps, in order:
 *  1. NaN or infinity -> FAIL; T = max fractional bits; x1 = min x, xm = max x;
 *  2. x2 = the smallest x above x1, x_(m-1) = the largest x below xm (distinct addresses);
 *     |Y| >= 2^62 -> FAIL;
 *  3. interior anchors A = (x2, smallest Y at x2), B = (x_(m-1), smallest Y at x_(m-1));
 *  4. n_off = the records NOT collinear with A and B (exact 128-bit cross product), n = records.
 * State: FAIL (steps 1-2), EMPTY (no record), POINT (fewer than 4 distinct x: no interior line),
 * else LINE.  The flag "structured with <= eps outliers" is LINE with A.Y != B.Y and
 * 100 n_off <= eps_pct n (the report's integer test; eps_pct a caller parameter). */
/* (vo_outlier: ve_oracle.h) */

int vo_outlier_fit(const vo_config* cfg, const vo_object* objs, uint32_t n_obj, const vo_record* recs, uint64_t n,
                   uint32_t flags, vo_outlier* out) {
  if (!cfg || cfg->n_pcs == 0) return -1;
  objtab t;
  if (objtab_build(&t, objs, n_obj) != 0) return -1;
  const uint64_t n_keys = (uint64_t)cfg->n_pcs + n_obj + 1;
  int* have = (int*)calloc(n_keys, sizeof(int));
  int* fail = (int*)calloc(n_keys, sizeof(int));
  int* T = (int*)calloc(n_keys, sizeof(int));
  uint64_t* x1 = (uint64_t*)calloc(n_keys, sizeof(uint64_t));
  uint64_t* xm = (uint64_t*)calloc(n_keys, sizeof(uint64_t));
  uint64_t* x2 = (uint64_t*)calloc(n_keys, sizeof(uint64_t));
  uint64_t* xl = (uint64_t*)calloc(n_keys, sizeof(uint64_t));
  int* h2 = (int*)calloc(n_keys, sizeof(int));
  int* hl = (int*)calloc(n_keys, sizeof(int));
  int* ha = (int*)calloc(n_keys, sizeof(int));
  int* hb = (int*)calloc(n_keys, sizeof(int));
  i128* ay = (i128*)calloc(n_keys, sizeof(i128));
  i128* by = (i128*)calloc(n_keys, sizeof(i128));
  memset(out, 0, sizeof(vo_outlier) * n_keys);
  for (int pass = 1; pass <= 4; ++pass) {
    for (uint64_t i = 0; i < n; ++i) {
      const vo_record* r = &recs[i];
      dec_t d;
      decode(cfg, &t, r, &d);
      if (!d.valid) continue;
      uint64_t kset[2];
      int nk = 0;
      kset[nk++] = r->pc;
      if (d.shared) kset[nk++] = (uint64_t)cfg->n_pcs + n_obj;
      else if (d.obj) kset[nk++] = (uint64_t)cfg->n_pcs + d.obj->id;
      int64_t M = 0;
      int E = 0;
      const int finite = trunc_exact_value(r->value, d.kind, d.w, cfg->mant_bits, (int)(flags & 1u), &M, &E);
      for (int j = 0; j < nk; ++j) {
        const uint64_t k = kset[j];
        if (pass == 1) {                                   /* step 1 */
          if (!finite) { fail[k] = 1; continue; }
          if (-E > T[k]) T[k] = -E;
          if (!have[k] || r->addr < x1[k]) x1[k] = r->addr;
          if (!have[k] || r->addr > xm[k]) xm[k] = r->addr;
          have[k] = 1;
          out[k].n++;
          continue;
        }
        if (fail[k]) continue;
        i128 Y;
        if (!scaled_y(M, E + T[k], &Y)) { fail[k] = 1; continue; }
        if (pass == 2) {                                   /* step 2 */
          if (r->addr > x1[k] && (!h2[k] || r->addr < x2[k])) { x2[k] = r->addr; h2[k] = 1; }
          if (r->addr < xm[k] && (!hl[k] || r->addr > xl[k])) { xl[k] = r->addr; hl[k] = 1; }
        } else if (pass == 3) {                            /* step 3 */
          if (h2[k] && r->addr == x2[k] && (!ha[k] || Y < ay[k])) { ay[k] = Y; ha[k] = 1; }
          if (hl[k] && r->addr == xl[k] && (!hb[k] || Y < by[k])) { by[k] = Y; hb[k] = 1; }
        } else if (h2[k] && hl[k] && x2[k] < xl[k]) {      /* step 4 */
          if (!collinear((i128)x2[k], ay[k], (i128)xl[k], by[k], (i128)r->addr, Y)) out[k].n_off++;
        }
      }
    }
  }
  for (uint64_t k = 0; k < n_keys; ++k) {
    vo_outlier* o = &out[k];
    if (fail[k] || !have[k]) {
      memset(o, 0, sizeof(*o));
      o->state = fail[k] ? VO_LINE_FAIL : VO_LINE_EMPTY;
      continue;
    }
    o->scale = (uint32_t)T[k];
    if (!(h2[k] && hl[k] && x2[k] < xl[k])) {
      const uint64_t nn = o->n;
      memset(o, 0, sizeof(*o));
      o->state = VO_LINE_POINT;
      o->n = nn;
      continue;
    }
    o->state = VO_LINE_LINE;
    o->ax = x2[k];
    o->bx = xl[k];
    o->ay = (int64_t)ay[k];
    o->by = (int64_t)by[k];
  }
  free(have); free(fail); free(T); free(x1); free(xm); free(x2); free(xl); free(h2); free(hl); free(ha); free(hb);
  free(ay); free(by);
  free(t.by_base);
  return 0;
}

/* ---- C17 per (PC, object) (f3; Table 5's redundancy analysis P:L470, LoadSpy ref [47] P:L658) ----
 * DESIGN.md R6 split by the pair (pc, object of the load's first byte): out[(pc (n_obj + 1) + id) 2]
 * = temporal loads of that pair, + 1 = temporally redundant ones; column id = n_obj collects the
 * loads outside every object.  The same trace-order definition as vo_temporal_loads. */
int vo_temporal_pairs(const vo_config* cfg, const vo_object* objs, uint32_t n_obj, const vo_record* recs,
                      uint64_t n, uint64_t* out) {
  if (!cfg || cfg->n_pcs == 0) return -1;
  objtab t;
  if (objtab_build(&t, objs, n_obj) != 0) return -1;
  const uint64_t cols = (uint64_t)n_obj + 1;
  memset(out, 0, sizeof(uint64_t) * 2 * cfg->n_pcs * cols);
  uint64_t cap = 16;
  while (cap < 2 * n + 2) cap <<= 1;
  lastload* tab = (lastload*)calloc(cap, sizeof(lastload));
  for (uint64_t i = 0; i < n; ++i) {
    const vo_record* r = &recs[i];
    dec_t d;
    decode(cfg, &t, r, &d);
    if (!d.valid || d.shared || d.store) continue;
    uint64_t h = (r->addr * 0x9E3779B97F4A7C15ull) >> 17 & (cap - 1);
    while (tab[h].used && tab[h].addr != r->addr) h = (h + 1) & (cap - 1);
    if (tab[h].used) {
      const int red = tab[h].w == d.w && tab[h].value == r->value;
      const uint64_t p = (uint64_t)r->pc * cols + (d.obj ? d.obj->id : n_obj);
      out[2 * p]++;
      out[2 * p + 1] += red;
    }
    tab[h].used = 1;
    tab[h].addr = r->addr;
    tab[h].value = r->value;
    tab[h].w = d.w;
  }
  free(tab);
  free(t.by_base);
  return 0;
}
