/*
 * ve_gen_core.h -- seeded, counter-based SYNTHETIC INPUT GENERATOR.
 *
 * This is the one module both sides may use (oracle-side tests and the CUDA
 * path's tests/bench): it produces value-trace records and object snapshots
 * as pure functions of (config, epoch, seed, index), identically on the host
 * (gcc) and on the device (nvcc).  It holds none of the analysis arithmetic:
 * no statistic, no pattern test, no hashing of the method -- only the recipe
 * of DESIGN.md section 4 (shapes of SURVEY.md 8(d)).
 *
 * Values are built from integer hashes and exact bit constructions only (no
 * floating-point operation whose rounding could differ between host and
 * device).
 */
#ifndef VE_GEN_CORE_H
#define VE_GEN_CORE_H
#include <math.h>
#include <stdint.h>
#include <string.h>

#if defined(__CUDACC__)
#define VEG_FN static inline __host__ __device__
#else
#define VEG_FN static inline
#endif

typedef struct veg_record {      /* = ve_record byte layout (24 B) */
  uint64_t addr, value;
  uint32_t pc, meta;
} veg_record;

typedef struct veg_object {
  uint64_t base, size;
  uint32_t id, elem_width;
  uint32_t has_pre, has_post;
} veg_object;

typedef struct veg_info {
  uint64_t n_records;            /* records of this epoch (0 = unbounded stream, fuzz) */
  uint32_t n_pcs, n_obj;
  uint32_t n_epochs, pad;
} veg_info;

enum { VEG_CFG1 = 1, VEG_CFG2 = 2, VEG_CFG3 = 3, VEG_CFG4 = 4, VEG_CFG5 = 5, VEG_FUZZ = 100, VEG_DEDUP = 101 };
/* cfg codes of the scalable configs carry a size shift s in bits 8..11:
 * VEG_CFG3 | (s << 8) is cfg3 with every tensor 2^s times smaller (s = 0: full size) */
#define VEG_BASE(cfg) ((cfg) & 0xFF)
#define VEG_SHIFT(cfg) (((cfg) >> 8) & 15)

/* meta encoding (include/ve.h): [1:0] log2 w, [3:2] kind, [4] store, [5] shared */
#define VEG_META(lg, kind, st) ((uint32_t)(lg) | ((uint32_t)(kind) << 2) | ((uint32_t)(st) << 4))
#define VEG_SHARED_BIT 0x20u

/* ---- counter-based hashing (splitmix64 finalizer) ------------------------ */
VEG_FN uint64_t veg_mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
VEG_FN uint64_t veg_h(uint64_t seed, uint64_t stream, uint64_t i) {
  return veg_mix64(veg_mix64(seed ^ (stream * 0xD1B54A32D192ED03ull)) + i);
}

/* exact int -> float bit patterns (|x| < 2^24 for f32, < 2^53 for f64) */
VEG_FN uint32_t veg_f32_of_int(int64_t x) {
  float f = (float)x;
  uint32_t u;
  memcpy(&u, &f, 4);
  return u;
}
VEG_FN uint64_t veg_f64_of_int(int64_t x) {
  double d = (double)x;
  uint64_t u;
  memcpy(&u, &d, 8);
  return u;
}
/* f32 bits of (x * 2^-k), x exact in f32, result normal: adjust the exponent */
VEG_FN uint32_t veg_f32_scaled(int64_t x, int k) {
  uint32_t u = veg_f32_of_int(x);
  if ((u & 0x7FFFFFFFu) == 0) return u;
  return u - ((uint32_t)k << 23);
}
/* random finite non-zero f32 with |v| < 1 */
VEG_FN uint32_t veg_f32_small(uint64_t h) {
  uint32_t sign = (uint32_t)(h & 1) << 31;
  uint32_t ex = 0x60u + (uint32_t)((h >> 1) % 31u);        /* 2^-31 .. 2^-1 */
  uint32_t man = (uint32_t)(h >> 8) & 0x7FFFFFu;
  return sign | (ex << 23) | man;
}

/* nearest binary32 / binary64 to k/10, k = 1..10 */
VEG_FN uint32_t veg_tenth_f32(uint32_t k) {
  const uint32_t t[10] = {0x3dcccccdu, 0x3e4ccccdu, 0x3e99999au, 0x3ecccccdu, 0x3f000000u,
                          0x3f19999au, 0x3f333333u, 0x3f4ccccdu, 0x3f666666u, 0x3f800000u};
  return t[k - 1];
}
VEG_FN uint64_t veg_tenth_f64(uint32_t k) {
  const uint64_t t[10] = {0x3fb999999999999aull, 0x3fc999999999999aull, 0x3fd3333333333333ull,
                          0x3fd999999999999aull, 0x3fe0000000000000ull, 0x3fe3333333333333ull,
                          0x3fe6666666666666ull, 0x3fe999999999999aull, 0x3feccccccccccccdull,
                          0x3ff0000000000000ull};
  return t[k - 1];
}

/* =========================================================================
 * cfg1: single kernel trace, 2^20 4-byte records, 16 PCs, one 4 MiB object
 * (BASELINE.json configs[0]).
 * ========================================================================= */
#define VEG_CFG1_BASE 0x7f0000000000ull
#define VEG_CFG1_N (1ull << 20)
#define VEG_CFG1_SLICE 65536ull

VEG_FN uint32_t veg_cfg1_meta(uint32_t pc) {
  /* PC: 0 ld u32, 1 ld u32, 2 ld i32, 3 ld i32, 4 ld f32, 5 ld f32, 6 ld u32,
   * 7 ld f32, 8 st f32, 9 st u32, 10 st i32, 11 st f32, 12 st u32, 13 st f32,
   * 14 st f32, 15 st f32 */
  const uint8_t kind[16] = {0, 0, 1, 1, 2, 2, 0, 2, 2, 0, 1, 2, 0, 2, 2, 2};
  return VEG_META(2, kind[pc], pc >= 8 ? 1 : 0);
}

/* the value the record of PC p at element e carries (SURVEY cfg1 PC roles) */
VEG_FN uint32_t veg_cfg1_value(uint64_t seed, uint32_t pc, uint64_t e) {
  switch (pc) {
    case 0: return 0;
    case 1: return 0x2Au;
    case 2: return (uint32_t)(int32_t)(3 * (int64_t)e - 7);
    case 3: return (uint32_t)(int32_t)((int64_t)(e % 102) - 1);
    case 4: return (e % 10 == 9) ? veg_f32_small(veg_h(seed, 4, e)) : 0x3F800000u;
    case 5: return 0x3F800000u + (uint32_t)((e % 4096) << 2);            /* 1 + k 2^-21 */
    case 6: return (uint32_t)veg_mix64(e);
    case 7: return veg_tenth_f32((uint32_t)(e % 10) + 1);
    case 8: return 0;
    case 9: return (uint32_t)veg_h(seed, 9, e);
    case 10: return (uint32_t)(int32_t)e;
    case 11: return (e % 250 == 0) ? veg_f32_small(veg_h(seed, 11, e)) : 0;
    case 12: return (uint32_t)veg_h(seed, 12, e);
    case 13: return (e % 2 == 0) ? 0u : 0x80000000u;                      /* +0.0 / -0.0 */
    case 14: return veg_f32_of_int((int64_t)(e % 256));
    default: return veg_f32_scaled((int64_t)(e % 2049) - 1024, 6);        /* k / 64 */
  }
}

/* pre snapshot element: loads read the pre value; store slices hold value^1
 * unless the PC role says otherwise */
VEG_FN uint32_t veg_cfg1_pre(uint64_t seed, uint64_t e) {
  uint32_t pc = (uint32_t)(e / VEG_CFG1_SLICE);
  uint32_t v = veg_cfg1_value(seed, pc, e);
  if (pc < 8) return v;
  if (pc == 8 || pc == 11 || pc == 13) return 0;
  if (pc == 9) return (e % 2 == 0) ? v : (v ^ 1u);
  return v ^ 1u;
}
VEG_FN uint32_t veg_cfg1_post(uint64_t seed, uint64_t e) {
  uint32_t pc = (uint32_t)(e / VEG_CFG1_SLICE);
  return pc < 8 ? veg_cfg1_pre(seed, e) : veg_cfg1_value(seed, pc, e);
}

VEG_FN void veg_cfg1_record(uint64_t seed, uint64_t r, veg_record* out) {
  uint64_t g = r / 32;
  uint32_t pc = (uint32_t)(g % 16);
  uint64_t e = (uint64_t)pc * VEG_CFG1_SLICE + (g / 16) * 32 + (r % 32);
  out->addr = VEG_CFG1_BASE + 4 * e;
  out->value = veg_cfg1_value(seed, pc, e);
  out->pc = pc;
  out->meta = veg_cfg1_meta(pc);
}

/* =========================================================================
 * cfg2: Darknet YOLOv4 conv layer (BASELINE.json configs[1]):
 * epoch 0 = fill_ongpu zero-fill of l.output_gpu, epoch 1 = gemm beta=1.
 * M = 256 (c_out), K = 3*3*128 = 1152, N = 76*76 = 5776, batch 4, tile 64x64.
 * ========================================================================= */
#define VEG_C2_M 256ull
#define VEG_C2_K 1152ull
#define VEG_C2_N 5776ull
#define VEG_C2_B 4ull
#define VEG_C2_NT 91ull                              /* ceil(N / 64) */
#define VEG_C2_FULL_TILE (73728ull + 1280ull * 64)  /* 155648 */
#define VEG_C2_EDGE_TW (VEG_C2_N - 64 * 90)          /* 16 */
#define VEG_C2_EDGE_TILE (73728ull + 1280ull * VEG_C2_EDGE_TW)
#define VEG_C2_PER_BM (90 * VEG_C2_FULL_TILE + VEG_C2_EDGE_TILE)
#define VEG_C2_FILL_N (VEG_C2_B * VEG_C2_M * VEG_C2_N)  /* 5,914,624 */
#define VEG_C2_GEMM_N (VEG_C2_B * 4 * VEG_C2_PER_BM)    /* 225,640,448 */

VEG_FN veg_object veg_cfg2_object(uint32_t i) {
  veg_object o;
  o.id = i;
  o.elem_width = 4;
  o.has_pre = 1;
  o.has_post = 1;
  o.base = 0x7f1000000000ull + (uint64_t)i * 0x1000000000ull;
  o.size = (i == 0) ? VEG_C2_M * VEG_C2_K * 4 : (i == 1) ? VEG_C2_K * VEG_C2_N * 4 : VEG_C2_FILL_N * 4;
  return o;
}

/* weights: N(0, ~0.04)-shaped values from a 2^16-entry table (exact sums of
 * hashed integers, scaled by a power of two) */
VEG_FN uint32_t veg_cfg2_weight(uint64_t seed, uint64_t idx) {
  uint64_t t = veg_h(seed, 1, idx) & 0xFFFFu;
  int64_t s = 0;
  for (int j = 0; j < 4; ++j) s += (int64_t)(veg_h(seed, 100 + j, t) & 0xFFFFu);
  return veg_f32_scaled(s - 131070, 20);
}
/* workspace: leaky-ReLU activations, 30% exact 0.0, 2^20-entry table */
VEG_FN uint32_t veg_cfg2_work(uint64_t seed, uint64_t idx) {
  uint64_t h = veg_h(seed, 2, idx);
  if (h % 10 < 3) return 0;
  uint64_t t = (h >> 32) & 0xFFFFFu;
  int64_t s = 0;
  for (int j = 0; j < 4; ++j) s += (int64_t)(veg_h(seed, 200 + j, t) & 0xFFFFu);
  s -= 131070;
  return veg_f32_scaled(s, s < 0 ? 23 : 20);                 /* negative slope 1/8 */
}
/* gemm output C (non-zero) */
VEG_FN uint32_t veg_cfg2_out(uint64_t seed, uint64_t idx) {
  uint64_t h = veg_h(seed, 3, idx);
  int64_t s = (int64_t)(h & 0xFFFFFu) - 524288;
  if (s == 0) s = 1;
  return veg_f32_scaled(s, 16);
}

VEG_FN uint32_t veg_cfg2_elem(uint64_t seed, uint32_t epoch, uint32_t obj, int post, uint64_t e) {
  if (obj == 0) return veg_cfg2_weight(seed, e);
  if (obj == 1) return veg_cfg2_work(seed, e);
  if (obj == 2) return (epoch == 1 && post) ? veg_cfg2_out(seed, e) : 0;
  return 0;                                                   /* x_gpu: zeros */
}

VEG_FN void veg_cfg2_record(uint64_t seed, uint32_t epoch, uint64_t r, veg_record* out) {
  const uint32_t ld = VEG_META(2, 2, 0), st = VEG_META(2, 2, 1);
  if (epoch == 0) {                                           /* fill_ongpu(.., 0, output_gpu) */
    out->addr = veg_cfg2_object(2).base + 4 * r;
    out->value = 0;
    out->pc = 0;
    out->meta = st;
    return;
  }
  uint64_t bm = r / VEG_C2_PER_BM, rr = r % VEG_C2_PER_BM;
  uint64_t b = bm / 4, mt = bm % 4;
  uint64_t nt = rr / VEG_C2_FULL_TILE;
  if (nt > 90) nt = 90;
  uint64_t t = rr - nt * VEG_C2_FULL_TILE;
  uint64_t tw = (nt < 90) ? 64 : VEG_C2_EDGE_TW;
  uint64_t kblock = 2048 + 32 * tw;
  if (t < 36 * kblock) {
    uint64_t ks = t / kblock, u = t % kblock;
    if (u < 2048) {                                           /* A[m][k] */
      uint64_t m = 64 * mt + u / 32, k = 32 * ks + u % 32;
      uint64_t e = m * VEG_C2_K + k;
      out->addr = veg_cfg2_object(0).base + 4 * e;
      out->value = veg_cfg2_weight(seed, e);
      out->pc = 1;
      out->meta = ld;
    } else {                                                  /* B[k][n] */
      u -= 2048;
      uint64_t k = 32 * ks + u / tw, n = 64 * nt + u % tw;
      uint64_t e = k * VEG_C2_N + n;
      out->addr = veg_cfg2_object(1).base + 4 * e;
      out->value = veg_cfg2_work(seed, e);
      out->pc = 2;
      out->meta = ld;
    }
    return;
  }
  uint64_t v = t - 36 * kblock;                               /* C rows: load then store */
  uint64_t m = 64 * mt + v / (2 * tw), c2 = v % (2 * tw);
  int is_st = c2 >= tw;
  uint64_t n = 64 * nt + (is_st ? c2 - tw : c2);
  uint64_t e = (b * VEG_C2_M + m) * VEG_C2_N + n;
  out->addr = veg_cfg2_object(2).base + 4 * e;
  out->value = is_st ? veg_cfg2_out(seed, e) : 0;
  out->pc = is_st ? 4 : 3;
  out->meta = is_st ? st : ld;
}

/* f64 bits of (x * 2^-k), x exact in f64, result normal */
VEG_FN uint64_t veg_f64_scaled(int64_t x, int k) {
  uint64_t u = veg_f64_of_int(x);
  if ((u & 0x7FFFFFFFFFFFFFFFull) == 0) return u;
  return u - ((uint64_t)k << 52);
}

/* =========================================================================
 * cfg3: PyTorch op mix (BASELINE.json configs[2]), one epoch
 * per training iteration (seed 3 + iteration), 16 objects, 20 PCs:
 *   S0 embedding      ld ids (i64), then per token 24 x (ld weight row chunk, st out)
 *   S1 masked_fill_   st weight row 0 (padding) = +0.0 over a zero row (redundant)
 *   S2 add            ld a, ld b, st c = a + b        (c: the high-cardinality PC)
 *   S3 relu           ld c (new values), st r = max(c, +0)
 *   S4 mul by ones    ld r, ld ones (1.0), st m = r
 *   S5 sum-reduce     per row: 1024 x ld x, then ONE st (partial group: later
 *                     windows are not 32-aligned)
 *   S6 index_select   ld idx (i64 arange, structured), ld src, st dst = src
 *   S7 zeros_like, zero_, ones fill: st grad 0, st grad 0, st ones_t 1.0 (all
 *                     over equal pre values: redundant)
 * Sizes at shift s: T = 32768>>s tokens, D = 768, V = 30522, M = 16 Mi>>s,
 * R = 16384>>s rows of 1024, NI = 4 Mi>>s; 264,291,072 records at s = 0.
 * Values are exact binary fractions k * 2^-10 (sums stay exact).
 * ========================================================================= */
#define VEG_C3_V 30522ull
#define VEG_C3_D 768ull
#define VEG_C3_BASE 0x7c0000000000ull
#define VEG_C3_NOBJ 16u
#define VEG_C3_NPCS 20u

typedef struct veg_c3dims { uint64_t T, M, R, NI; } veg_c3dims;
VEG_FN veg_c3dims veg_c3_dims(uint32_t sh) {
  veg_c3dims d;
  d.T = 32768ull >> sh; d.M = (16ull << 20) >> sh; d.R = 16384ull >> sh; d.NI = (4ull << 20) >> sh;
  return d;
}
/* records per segment */
VEG_FN void veg_c3_seglen(uint32_t sh, uint64_t* L) {
  veg_c3dims d = veg_c3_dims(sh);
  L[0] = d.T + 2 * d.T * VEG_C3_D;
  L[1] = VEG_C3_D;
  L[2] = 3 * d.M;
  L[3] = 2 * d.M;
  L[4] = 3 * d.M;
  L[5] = 1025 * d.R;
  L[6] = 3 * d.NI;
  L[7] = 3 * d.M;
}
VEG_FN uint64_t veg_c3_n(uint32_t sh) {
  uint64_t L[8], n = 0;
  veg_c3_seglen(sh, L);
  for (int i = 0; i < 8; ++i) n += L[i];
  return n;
}
VEG_FN veg_object veg_c3_object(uint32_t sh, uint32_t i) {
  veg_c3dims d = veg_c3_dims(sh);
  const uint64_t elems[16] = {VEG_C3_V * VEG_C3_D, d.T, d.T * VEG_C3_D, d.M, d.M, d.M, d.M, d.M, d.M,
                              d.R * 1024, d.R, d.NI, d.NI, d.NI, d.M, d.M};
  veg_object o;
  o.id = i;
  o.base = VEG_C3_BASE + (uint64_t)i * (1ull << 36);
  o.elem_width = (i == 1 || i == 11) ? 8 : 4;
  o.size = elems[i] * o.elem_width;
  o.has_pre = 1;
  o.has_post = 1;
  return o;
}
/* embedding weights: N(0, ~0.02)-shaped, 2^16-entry table; the padding row 0 is zero */
VEG_FN uint32_t veg_c3_w(uint64_t seed, uint64_t e) {
  if (e < VEG_C3_D) return 0;
  uint64_t t = veg_h(seed, 30, e) & 0xFFFFu;
  int64_t s = 0;
  for (int j = 0; j < 4; ++j) s += (int64_t)(veg_h(seed, 300 + j, t) & 0xFFFFu);
  return veg_f32_scaled(s - 131070, 21);
}
/* token ids: 10% padding id 0, else a skewed (Zipf-like) id in [1, V) */
VEG_FN uint64_t veg_c3_id(uint64_t seed, uint64_t t) {
  uint64_t h = veg_h(seed, 31, t);
  if (h % 10 == 0) return 0;
  uint64_t span = 1 + (h >> 32) % (VEG_C3_V - 1);
  return 1 + ((h >> 8) & 0xFFFFFFu) % span;
}
VEG_FN int64_t veg_c3_k20(uint64_t seed, uint64_t st, uint64_t e) {   /* k in [-2^19, 2^19) */
  return (int64_t)(veg_h(seed, st, e) & 0xFFFFFu) - 524288;
}
VEG_FN int64_t veg_c3_kc(uint64_t seed, uint64_t e) { return veg_c3_k20(seed, 33, e) + veg_c3_k20(seed, 34, e); }
VEG_FN uint32_t veg_c3_r(uint64_t seed, uint64_t e) {
  int64_t k = veg_c3_kc(seed, e);
  return k > 0 ? veg_f32_scaled(k, 10) : 0u;
}
VEG_FN int64_t veg_c3_kx(uint64_t seed, uint64_t e) {                 /* reduce input, k in [-2^12, 2^12) */
  return (int64_t)(veg_h(seed, 35, e) & 0x1FFFu) - 4096;
}
VEG_FN uint32_t veg_c3_rowsum(uint64_t seed, uint64_t i) {
  int64_t s = 0;
  for (uint64_t j = 0; j < 1024; ++j) s += veg_c3_kx(seed, i * 1024 + j);
  return veg_f32_scaled(s, 10);
}
/* element e of object i: pre (post = 0) or post (post = 1) snapshot */
VEG_FN uint64_t veg_c3_elem(uint64_t seed, uint32_t sh, uint32_t i, int post, uint64_t e) {
  switch (i) {
    case 0: return veg_c3_w(seed, e);
    case 1: return veg_c3_id(seed, e);
    case 2: return post ? veg_c3_w(seed, veg_c3_id(seed, e / VEG_C3_D) * VEG_C3_D + e % VEG_C3_D) : 0;
    case 3: return veg_f32_scaled(veg_c3_k20(seed, 33, e), 10);
    case 4: return veg_f32_scaled(veg_c3_k20(seed, 34, e), 10);
    case 5: return post ? veg_f32_scaled(veg_c3_kc(seed, e), 10) : 0;
    case 6: return post ? veg_c3_r(seed, e) : 0;
    case 7: return 0x3F800000u;
    case 8: return post ? veg_c3_r(seed, e) : 0;
    case 9: return veg_f32_scaled(veg_c3_kx(seed, e), 10);
    case 10: return post ? veg_c3_rowsum(seed, e) : 0;
    case 11: return e;
    case 12: return veg_f32_scaled(veg_c3_k20(seed, 36, e), 10);
    case 13: return post ? veg_f32_scaled(veg_c3_k20(seed, 36, e), 10) : 0;
    case 14: return 0;
    default: return 0x3F800000u;
  }
  (void)sh;
}
VEG_FN void veg_c3_put(veg_record* out, uint32_t sh, uint32_t obj, uint64_t e, uint64_t v, uint32_t pc, int st) {
  veg_object o = veg_c3_object(sh, obj);
  out->addr = o.base + e * o.elem_width;
  out->value = v;
  out->pc = pc;
  out->meta = VEG_META(o.elem_width == 8 ? 3 : 2, o.elem_width == 8 ? 1 : 2, st);
}
VEG_FN void veg_cfg3_record(uint64_t seed, uint32_t sh, uint64_t r, veg_record* out) {
  uint64_t L[8];
  veg_c3_seglen(sh, L);
  int sg = 0;
  while (sg < 7 && r >= L[sg]) r -= L[sg++];
  const uint64_t D = VEG_C3_D;
  if (sg == 0) {                                   /* embedding: per 32-token block */
    const uint64_t blk = 32 + 32 * 24 * 64;
    uint64_t b = r / blk, u = r % blk;
    if (u < 32) { uint64_t t = b * 32 + u; veg_c3_put(out, sh, 1, t, veg_c3_id(seed, t), 0, 0); return; }
    u -= 32;
    uint64_t t = b * 32 + u / (24 * 64), v = u % (24 * 64);
    uint64_t d = (v / 64) * 32 + v % 32;
    uint64_t we = veg_c3_id(seed, t) * D + d;
    if (v % 64 < 32) veg_c3_put(out, sh, 0, we, veg_c3_w(seed, we), 1, 0);
    else veg_c3_put(out, sh, 2, t * D + d, veg_c3_w(seed, we), 2, 1);
    return;
  }
  if (sg == 1) { veg_c3_put(out, sh, 0, r, 0, 3, 1); return; }
  if (sg == 2 || sg == 4 || sg == 6) {             /* 3 groups per 32-element block */
    uint64_t e = (r / 96) * 32 + r % 32, g = (r % 96) / 32;
    if (sg == 2) {
      if (g == 0) veg_c3_put(out, sh, 3, e, veg_f32_scaled(veg_c3_k20(seed, 33, e), 10), 4, 0);
      else if (g == 1) veg_c3_put(out, sh, 4, e, veg_f32_scaled(veg_c3_k20(seed, 34, e), 10), 5, 0);
      else veg_c3_put(out, sh, 5, e, veg_f32_scaled(veg_c3_kc(seed, e), 10), 6, 1);
    } else if (sg == 4) {
      if (g == 0) veg_c3_put(out, sh, 6, e, veg_c3_r(seed, e), 9, 0);
      else if (g == 1) veg_c3_put(out, sh, 7, e, 0x3F800000u, 10, 0);
      else veg_c3_put(out, sh, 8, e, veg_c3_r(seed, e), 11, 1);
    } else {
      if (g == 0) veg_c3_put(out, sh, 11, e, e, 14, 0);
      else if (g == 1) veg_c3_put(out, sh, 12, e, veg_f32_scaled(veg_c3_k20(seed, 36, e), 10), 15, 0);
      else veg_c3_put(out, sh, 13, e, veg_f32_scaled(veg_c3_k20(seed, 36, e), 10), 16, 1);
    }
    return;
  }
  if (sg == 3) {                                   /* relu */
    uint64_t e = (r / 64) * 32 + r % 32;
    if ((r % 64) < 32) veg_c3_put(out, sh, 5, e, veg_f32_scaled(veg_c3_kc(seed, e), 10), 7, 0);
    else veg_c3_put(out, sh, 6, e, veg_c3_r(seed, e), 8, 1);
    return;
  }
  if (sg == 5) {                                   /* sum-reduce rows */
    uint64_t i = r / 1025, u = r % 1025;
    if (u < 1024) veg_c3_put(out, sh, 9, i * 1024 + u, veg_f32_scaled(veg_c3_kx(seed, i * 1024 + u), 10), 12, 0);
    else veg_c3_put(out, sh, 10, i, veg_c3_rowsum(seed, i), 13, 1);
    return;
  }
  {                                                /* zeros_like, zero_, ones fill */
    veg_c3dims d = veg_c3_dims(sh);
    uint64_t pass = r / d.M, e = r % d.M;
    if (pass < 2) veg_c3_put(out, sh, 14, e, 0, 17 + (uint32_t)pass, 1);
    else veg_c3_put(out, sh, 15, e, 0x3F800000u, 19, 1);
  }
}

/* =========================================================================
 * cfg4: LAMMPS / Castro-style f64 stencils (BASELINE.json configs[3]; SURVEY
 * 8(d) cfg4) on a G^3 grid, G = 512 >> s, point p = (z G + y) G + x.  Warps
 * take 32 consecutive points; each memory instruction is one 32-record group.
 *   epoch 0 (hotspot3D-like): 7 loads of T_in (centre, x-1, x+1, y-1, y+1, z-1,
 *     z+1; faces clamped), st T_out = T_in(centre).  T_in = 300 + 3q/8192,
 *     q = hash mod 4096: one K=7 truncation bucket (approximate), n_ld_reload
 *     = 6/7 of the T_in loads.
 *   epoch 1 (cellconslin_slopes-like): ld a (1.0 except every 20th point: 2.0),
 *     ld xc[x] (= x + 64: structured), ld vol (1.0), ld s[x-1], s, s[x+1]
 *     (clamped), st s (= s_pre where a == 1: redundant, else s_pre + 1).
 * Objects (f64, ew 8): 0 T_in, 1 T_out, 2 a, 3 s, 4 vol (G^3 each), 5 xc (G).
 * ========================================================================= */
#define VEG_C4_BASE 0x7b0000000000ull
#define VEG_C4_NPCS 15u

VEG_FN uint64_t veg_c4_g(uint32_t sh) { return 512ull >> sh; }
VEG_FN veg_object veg_c4_object(uint32_t sh, uint32_t i) {
  uint64_t G = veg_c4_g(sh);
  veg_object o;
  o.id = i;
  o.base = VEG_C4_BASE + (uint64_t)i * (1ull << 36);
  o.elem_width = 8;
  o.size = 8 * (i == 5 ? G : G * G * G);
  o.has_pre = 1;
  o.has_post = 1;
  return o;
}
VEG_FN uint64_t veg_c4_tin(uint64_t seed, uint64_t p) {
  return veg_f64_scaled(300 * 8192 + 3 * (int64_t)(veg_h(seed, 41, p) % 4096), 13);
}
VEG_FN int64_t veg_c4_spre(uint64_t seed, uint64_t p) { return (int64_t)(veg_h(seed, 42, p) % 1000); }
VEG_FN uint64_t veg_c4_elem(uint64_t seed, uint32_t sh, uint32_t epoch, uint32_t i, int post, uint64_t e) {
  uint64_t G = veg_c4_g(sh);
  switch (i) {
    case 0: return veg_c4_tin(seed, e);
    case 1: return (post && epoch == 0) ? veg_c4_tin(seed, e) : 0;
    case 2: return (e % 20 != 0) ? 0x3FF0000000000000ull : 0x4000000000000000ull;
    case 3: return veg_f64_of_int(veg_c4_spre(seed, e) + ((post && epoch == 1 && e % 20 == 0) ? 1 : 0));
    case 4: return 0x3FF0000000000000ull;
    default: return veg_f64_of_int((int64_t)(e % G) + 64);
  }
}
VEG_FN uint64_t veg_c4_n(uint32_t sh, uint32_t epoch) {
  uint64_t G = veg_c4_g(sh);
  return (epoch == 0 ? 8 : 7) * G * G * G;
}
VEG_FN void veg_cfg4_record(uint64_t seed, uint32_t sh, uint32_t epoch, uint64_t r, veg_record* out) {
  const uint64_t G = veg_c4_g(sh);
  const uint32_t ng = epoch == 0 ? 8 : 7;
  const uint64_t b = r / (32 * ng), g = (r % (32 * ng)) / 32, p = b * 32 + r % 32;
  const uint64_t x = p % G, y = (p / G) % G, z = p / (G * G);
  uint32_t obj;
  uint64_t e = p;
  int st = 0;
  if (epoch == 0) {
    obj = 0;
    if (g == 1) e = p - (x > 0);
    else if (g == 2) e = p + (x + 1 < G);
    else if (g == 3) e = p - (y > 0) * G;
    else if (g == 4) e = p + (y + 1 < G) * G;
    else if (g == 5) e = p - (z > 0) * G * G;
    else if (g == 6) e = p + (z + 1 < G) * G * G;
    else if (g == 7) { obj = 1; st = 1; }
    out->value = veg_c4_tin(seed, e);
    out->pc = (uint32_t)g;
  } else {
    const uint32_t objs[7] = {2, 5, 4, 3, 3, 3, 3};
    obj = objs[g];
    if (g == 1) e = x;
    else if (g == 3) e = p - (x > 0);
    else if (g == 5) e = p + (x + 1 < G);
    st = g == 6;
    out->value = veg_c4_elem(seed, sh, 1, obj, st, e);
    out->pc = 8 + (uint32_t)g;
  }
  const veg_object o = veg_c4_object(sh, obj);
  out->addr = o.base + 8 * e;
  out->meta = VEG_META(3, 2, st);
}

/* =========================================================================
 * FUZZ: adversarial mixed trace for unit parity (SURVEY section 4 "unit
 * parity"): 64 PCs (+ invalid 64..69), 6 objects with gaps, odd sizes,
 * every element width, a NULL pre and a NULL post, shared-space groups,
 * misaligned / straddling / unmapped / invalid records, NaN / -0.0 / Inf,
 * split and partial warp groups.
 * ========================================================================= */
#define VEG_FZ_REGION 0x7e0000000000ull
#define VEG_FZ_NPCS 64u
#define VEG_FZ_NOBJ 6u

VEG_FN veg_object veg_fuzz_object(uint32_t i) {
  const uint64_t off[6] = {0x0, 0x20000, 0x40000, 0x50000, 0x70000, 0x80000};
  const uint64_t size[6] = {65536, 40000, 4096, 65534, 32768, 131072};
  const uint32_t ew[6] = {4, 8, 1, 2, 4, 8};
  veg_object o;
  o.id = i;
  o.base = VEG_FZ_REGION + off[i];
  o.size = size[i];
  o.elem_width = ew[i];
  o.has_pre = (i != 2);
  o.has_post = (i != 4);
  return o;
}

VEG_FN uint64_t veg_pool64(uint32_t k) {
  const uint64_t p[16] = {0ull, 1ull, 0x2Aull, ~0ull, 0x3F800000ull, 0x3FF0000000000000ull,
                          0x8000000000000000ull, 0x80000000ull, 0x7FC00000ull, 0x7FF8000000000001ull,
                          0x3C00ull, 0x3F80ull, 0xFFFFFFFF00000000ull, 0x0000000100000000ull,
                          0x4049000000000000ull, 0x7F800000ull};
  return p[k & 15];
}
VEG_FN uint32_t veg_pool_bf16(uint32_t k) {
  const uint16_t p[16] = {0x3F80, 0x0000, 0x8000, 0x7FC0, 0x7F80, 0x4049, 0x4300, 0xC2F6,
                          0x3DCD, 0x0001, 0x4780, 0x477F, 0x3F81, 0x4120, 0xBF80, 0x42FE};
  return p[k & 15];
}
VEG_FN uint32_t veg_pool_f16(uint32_t k) {
  const uint16_t p[16] = {0x3C00, 0x0000, 0x8000, 0x7E00, 0x7C00, 0x4248, 0x5800, 0xD7B0,
                          0x2E66, 0x0001, 0x7BFF, 0x4900, 0xBC00, 0x57F0, 0x3C01, 0x5BF8};
  return p[k & 15];
}

/* 8-byte word j of fuzz object o (pre or post) */
VEG_FN uint64_t veg_fuzz_word(uint64_t seed, uint32_t o, int post, uint64_t j) {
  uint64_t h = veg_h(seed, 2000 + o, j);
  uint64_t pre = veg_pool64((uint32_t)(h % 16));
  if (h % 3 == 0) pre = (pre << 8) | (h >> 56);               /* some non-pool words */
  if (!post) return pre;
  uint64_t h2 = veg_h(seed, 3000 + o, j);
  return (h2 % 4 == 0) ? veg_pool64((uint32_t)(h2 >> 8)) : pre;
}
/* w little-endian bytes of fuzz object content at byte offset off (clipped) */
VEG_FN uint64_t veg_fuzz_bytes(uint64_t seed, uint32_t o, int post, uint64_t off, uint32_t w, uint64_t size) {
  uint64_t v = 0;
  for (uint32_t i = 0; i < w; ++i) {
    uint64_t p = off + i;
    if (p >= size) break;
    uint64_t b = (veg_fuzz_word(seed, o, post, p / 8) >> (8 * (p % 8))) & 0xFFu;
    v |= b << (8 * i);
  }
  return v;
}

/* PC roles (pc % 16): log2 width, kind, store */
VEG_FN uint32_t veg_fuzz_role_meta(uint32_t role) {
  const uint8_t lg[16] = {2, 2, 2, 2, 2, 2, 2, 3, 2, 3, 3, 3, 1, 1, 2, 0};
  const uint8_t kind[16] = {0, 0, 1, 1, 2, 2, 0, 2, 2, 0, 1, 2, 3, 2, 2, 0};
  const uint8_t st[16] = {0, 1, 0, 0, 0, 0, 0, 0, 1, 1, 1, 0, 0, 1, 1, 0};
  return VEG_META(lg[role], kind[role], st[role]);
}

VEG_FN uint64_t veg_fuzz_role_value(uint64_t seed, uint32_t role, uint64_t addr, uint64_t hl) {
  int64_t d = (int64_t)(addr - VEG_FZ_REGION);
  switch (role) {
    case 0: return 0;
    case 1: return 0x2A;
    case 2: return (uint32_t)(int32_t)(3 * (d / 4) - 7);
    case 3: return (uint32_t)(int32_t)((int64_t)(hl % 102) - 1);
    case 4: return (hl % 10 == 9) ? veg_f32_small(hl >> 8) : 0x3F800000u;
    case 5: return 0x3F800000u + (uint32_t)(((hl >> 4) % 4096) << 2);
    case 6: return (uint32_t)(hl >> 16);
    case 7: return veg_tenth_f64((uint32_t)(hl % 10) + 1);
    case 8: return 0;
    case 9: return veg_pool64((uint32_t)(hl >> 3));
    case 10: return (uint64_t)(-5 * d + 1);
    case 11: return veg_f64_of_int(d / 8 + 64);
    case 12: return veg_pool_bf16((uint32_t)(hl >> 5));
    case 13: return veg_pool_f16((uint32_t)(hl >> 5));
    case 14: return veg_f32_of_int((int64_t)(hl % 256));
    default: return (hl >> 9) & 0xFFu;
  }
}

/* address of lane l of a "role group" on object o starting at element s */
VEG_FN void veg_fuzz_role_lane(uint64_t seed, uint64_t hg, uint64_t r, uint32_t lane, int shared,
                               uint32_t pc_lo, uint32_t pc_span, veg_record* out) {
  uint32_t pc = pc_lo + (uint32_t)(hg % pc_span);
  uint32_t role = pc % 16;
  uint32_t meta = veg_fuzz_role_meta(role);
  uint32_t w = 1u << (meta & 3u);
  uint64_t hl = veg_h(seed, 1002, r);
  uint64_t addr;
  if (shared) {
    addr = ((hg >> 20) % 4096) * 8 + (uint64_t)lane * w;
    meta |= VEG_SHARED_BIT;
  } else {
    veg_object o = veg_fuzz_object((uint32_t)((hg >> 8) % VEG_FZ_NOBJ));
    uint64_t nel = o.size / w;
    uint64_t s = (hg >> 16) % nel;
    addr = o.base + (s + lane) * w;
  }
  out->pc = pc;
  out->meta = meta;
  out->addr = addr;
  uint64_t v = veg_fuzz_role_value(seed, role, addr, hl);
  /* unstructured roles sometimes carry the pre bytes (eq_pre coverage) */
  if (!shared && (role == 9 || role == 15 || role == 6 || role == 3) && (hl >> 40) % 2 == 0) {
    uint32_t oi = (uint32_t)((hg >> 8) % VEG_FZ_NOBJ);
    veg_object o = veg_fuzz_object(oi);
    if (addr + w <= o.base + o.size) {
      uint64_t b = veg_fuzz_bytes(seed, oi, 0, addr - o.base, w, o.size);
      if (role == 3) b = (uint32_t)(int32_t)(int8_t)(b & 0x7F);    /* keep role 3 in range */
      if (role == 6 || role == 3 || role == 9 || role == 15) v = b;
    }
  }
  out->value = v;
}

VEG_FN void veg_fuzz_chaos_lane(uint64_t seed, uint64_t r, veg_record* out) {
  uint64_t h = veg_h(seed, 1001, r), h2 = veg_h(seed, 1003, r);
  uint32_t lg = (uint32_t)(h & 3), kind = (uint32_t)((h >> 2) & 3), st = (uint32_t)((h >> 4) & 1);
  uint32_t meta = VEG_META(lg, kind, st);
  if (((h >> 5) & 7) == 0) meta |= VEG_SHARED_BIT;
  if (((h >> 8) & 63) == 0) meta |= 1u << (6 + ((h >> 14) % 26));     /* reserved bit */
  uint32_t w = 1u << lg;
  out->pc = 48 + (uint32_t)((h >> 20) % 22);                         /* 64..69 invalid */
  out->meta = meta;
  uint64_t sel = (h >> 28) % 32;
  if (sel == 0) {
    out->addr = (1ull << 48) + (h2 & 0xFFFF);                        /* invalid address */
  } else if (sel < 4) {
    out->addr = VEG_FZ_REGION + 0x10000 + (h2 % 0x10000);            /* unmapped gap */
  } else if (meta & VEG_SHARED_BIT) {
    out->addr = h2 % 0x8000;
  } else {
    veg_object o = veg_fuzz_object((uint32_t)(h2 % VEG_FZ_NOBJ));
    out->addr = o.base + (h2 >> 8) % (o.size + 16);                 /* may straddle / overrun */
  }
  uint64_t v;
  uint64_t vs = (h2 >> 40) % 8;
  if (vs < 4 && !(meta & VEG_SHARED_BIT) && out->addr >= VEG_FZ_REGION) {
    uint64_t a = out->addr;
    v = 0;
    for (uint32_t i = 0; i < VEG_FZ_NOBJ; ++i) {
      veg_object o = veg_fuzz_object(i);
      if (a >= o.base && a < o.base + o.size) v = veg_fuzz_bytes(seed, i, 0, a - o.base, w, o.size);
    }
  } else if (vs < 7) {
    v = veg_pool64((uint32_t)(h2 >> 50));
  } else {
    v = veg_h(seed, 1004, r);
  }
  if (w < 8 && ((h >> 50) & 63) != 0) v &= (1ull << (8 * w)) - 1;   /* else: bits above 8w (invalid) */
  out->value = v;
}

VEG_FN void veg_fuzz_record(uint64_t seed, uint64_t r, veg_record* out) {
  uint64_t g = r / 32;
  uint32_t lane = (uint32_t)(r % 32);
  uint64_t hg = veg_h(seed, 1000, g);
  uint32_t mode = (uint32_t)(hg % 16);
  if (mode <= 8) {
    veg_fuzz_role_lane(seed, hg >> 4, r, lane, 0, 0, 48, out);
  } else if (mode <= 10) {                                            /* split group */
    uint32_t s = 1 + (uint32_t)((hg >> 4) % 31);
    uint64_t hsub = veg_h(seed, 1005 + (lane >= s), g);
    veg_fuzz_role_lane(seed, hsub, r, lane >= s ? lane - s : lane, 0, 0, 48, out);
  } else if (mode <= 12) {
    veg_fuzz_chaos_lane(seed, r, out);
  } else if (mode == 13) {                                            /* uniform pc, mixed meta */
    veg_fuzz_chaos_lane(seed, r, out);
    out->pc = 48 + (uint32_t)((hg >> 4) % 16);
  } else if (mode == 14) {                                            /* shared-space group */
    veg_fuzz_role_lane(seed, hg >> 4, r, lane, 1, 32, 16, out);
  } else {                                                            /* partial invalid lanes */
    veg_fuzz_role_lane(seed, hg >> 4, r, lane, 0, 0, 48, out);
    if (lane % 7 == 3) out->pc = 64 + lane % 6;
  }
}

/* =========================================================================
 * DEDUP set (SURVEY cfg5 object mix, scaled): objects of a few sizes;
 * 30% all-zero, 10% exact copies, 5% one-byte-flip copies, 55% random.
 * ========================================================================= */
#define VEG_DD_BASE 0x7d0000000000ull

/* unit > 0: 4 distinct sizes unit .. 4 unit (the scaled test sets).  unit == 0: the cfg5 recipe
 * (SURVEY 8(d) cfg5): 50 log-uniform size classes s = 0..49 over [64 KiB, 512 MiB] (64 KiB x 2^(13 s / 49),
 * 4 KiB multiples); this returns the class size, whose EQUALITY is what the content classes use --
 * veg_dedup_object rescales it so the 1000 objects total 20 GiB (ve_gen.cu). */
VEG_FN uint64_t veg_dedup_class_size(uint32_t s) {
  const double b = 65536.0 * exp2(13.0 * (double)s / 49.0);
  return ((uint64_t)b + 4095ull) & ~4095ull;
}
VEG_FN uint64_t veg_dedup_size(uint64_t seed, uint32_t i, uint64_t unit) {
  uint64_t h = veg_h(seed, 4000, i);
  if (unit == 0) return veg_dedup_class_size((uint32_t)(h % 50));
  return unit * (1 + h % 4);                                  /* 4 distinct sizes */
}
VEG_FN uint32_t veg_dedup_base_class(uint64_t seed, uint32_t i) {
  uint32_t c = (uint32_t)(veg_h(seed, 4001, i) % 100);
  return c < 30 ? 0 : c < 40 ? 1 : c < 45 ? 2 : 3;
}
/* content class: 0 zero, 1 copy of *src, 2 one-bit-flipped copy of *src, 3 random.
 * A copy's source is the nearest earlier object of the same size whose base
 * class is 0 or 3; without one the object is random.  (Host-side, O(i).) */
VEG_FN uint32_t veg_dedup_class(uint64_t seed, uint32_t i, uint32_t* src, uint64_t unit) {
  uint32_t cls = veg_dedup_base_class(seed, i);
  *src = i;
  if (cls == 1 || cls == 2) {
    uint64_t sz = veg_dedup_size(seed, i, unit);
    for (uint32_t j = i; j-- > 0;) {
      uint32_t cj = veg_dedup_base_class(seed, j);
      if (veg_dedup_size(seed, j, unit) == sz && (cj == 3 || cj == 0)) { *src = j; return cls; }
    }
    return 3;
  }
  return cls;
}
/* 8-byte word j of dedup object i with resolved (cls, src, src_cls) */
VEG_FN uint64_t veg_dedup_word(uint64_t seed, uint32_t i, uint32_t cls, uint32_t src, uint32_t src_cls,
                               uint64_t words, uint64_t j) {
  if (cls == 0) return 0;
  if (cls == 3) return veg_h(seed, 5000 + i, j);
  uint64_t v = (src_cls == 0) ? 0 : veg_h(seed, 5000 + src, j);
  if (cls == 2 && j == veg_h(seed, 4002, i) % words) v ^= 1ull << (veg_h(seed, 4003, i) % 64);
  return v;
}


/* =========================================================================
 * cfg5 records half (BASELINE.json configs[4]; SURVEY 8(d) cfg5 "Kernels"):
 * 4000 independent kernels, epoch = kernel index k.  Kernel k has P = 4..64
 * PCs whose roles are drawn from cfg1's 16 roles, touches O = 1..4 objects
 * of 4-byte elements, and has n_k records: octave-uniform raw draws in
 * [10^4, 2*10^6), rescaled in groups of 8 kernels so every group sums to
 * exactly 2*10^6 records (500 groups: 1,000,000,000 records in total).
 * The geometry (P, O, roles, n_k) is drawn from the fixed seed 5 so that it
 * does not depend on the value seed; shift s divides every n_k by 2^s.
 *
 * Record r of kernel k: warp g = r / 32 belongs to PC p = g % P (round robin,
 * like cfg1), PC p lives on object o = p % O in slot s = p / O of L elements
 * (L = 32 * ceil(ceil(n/32) / P)); its element is e = s L + (g / P) 32 + r % 32
 * and it carries veg_cfg1_value(seed, role, e).  pre follows cfg1's per-role
 * rule; post = pre + the stores (elements no record covers keep pre).
 * ========================================================================= */
#define VEG_C5_KERNELS 4000u
#define VEG_C5_GROUP 8u
#define VEG_C5_GROUP_N 2000000ull
#define VEG_C5_GEOM_SEED 5ull
#define VEG_C5_BASE 0x7c0000000000ull

VEG_FN uint64_t veg_c5_raw(uint32_t k) {              /* octave-uniform in [1e4, 2e6) */
  uint64_t h = veg_h(VEG_C5_GEOM_SEED, 500, k);
  uint64_t lo = 10000ull << (h % 8);
  uint64_t hi = 2 * lo < 2000000ull ? 2 * lo : 2000000ull;
  return lo + (h >> 8) % (hi - lo);
}
VEG_FN uint64_t veg_c5_n(uint32_t sh, uint32_t k) {
  uint32_t g0 = k - k % VEG_C5_GROUP;
  uint64_t S = 0, part = 0;
  for (uint32_t j = 0; j < VEG_C5_GROUP; ++j) S += veg_c5_raw(g0 + j);
  uint64_t n;
  if (k % VEG_C5_GROUP != VEG_C5_GROUP - 1) {
    n = veg_c5_raw(k) * VEG_C5_GROUP_N / S;
  } else {
    for (uint32_t j = 0; j + 1 < VEG_C5_GROUP; ++j) part += veg_c5_raw(g0 + j) * VEG_C5_GROUP_N / S;
    n = VEG_C5_GROUP_N - part;
  }
  return n >> sh;
}
VEG_FN uint32_t veg_c5_npcs(uint32_t k) { return 4u + (uint32_t)(veg_h(VEG_C5_GEOM_SEED, 501, k) % 61u); }
VEG_FN uint32_t veg_c5_nobj(uint32_t k) { return 1u + (uint32_t)((veg_h(VEG_C5_GEOM_SEED, 501, k) >> 8) % 4u); }
VEG_FN uint32_t veg_c5_role(uint32_t k, uint32_t p) {
  return (uint32_t)(veg_h(VEG_C5_GEOM_SEED, 502, (uint64_t)k * 64u + p) % 16u);
}
/* elements per PC slot */
VEG_FN uint64_t veg_c5_slot(uint64_t n, uint32_t P) { return 32ull * ((((n + 31) / 32) + P - 1) / P); }

VEG_FN veg_object veg_c5_object(uint32_t sh, uint32_t k, uint32_t i) {
  veg_object o;
  uint32_t P = veg_c5_npcs(k), O = veg_c5_nobj(k);
  uint64_t L = veg_c5_slot(veg_c5_n(sh, k), P);
  uint32_t slots = (P - i + O - 1) / O;                /* PCs p = i, i + O, ... */
  o.base = VEG_C5_BASE + ((uint64_t)i << 36);
  o.size = 4ull * L * slots;
  o.id = i;
  o.elem_width = 4;
  o.has_pre = 1;
  o.has_post = 1;
  return o;
}

VEG_FN void veg_cfg5_record(uint64_t seed, uint32_t sh, uint32_t k, uint64_t r, veg_record* out) {
  uint32_t P = veg_c5_npcs(k), O = veg_c5_nobj(k);
  uint64_t L = veg_c5_slot(veg_c5_n(sh, k), P);
  uint64_t g = r / 32;
  uint32_t p = (uint32_t)(g % P), o = p % O, role = veg_c5_role(k, p);
  uint64_t e = (uint64_t)(p / O) * L + (g / P) * 32 + r % 32;
  out->addr = VEG_C5_BASE + ((uint64_t)o << 36) + 4 * e;
  out->value = veg_cfg1_value(seed, role, e);
  out->pc = p;
  out->meta = veg_cfg1_meta(role);
}

/* element e of object i (pre or post) */
VEG_FN uint32_t veg_c5_elem(uint64_t seed, uint32_t sh, uint32_t k, uint32_t i, int post, uint64_t e) {
  uint32_t P = veg_c5_npcs(k), O = veg_c5_nobj(k);
  uint64_t n = veg_c5_n(sh, k), L = veg_c5_slot(n, P);
  uint32_t p = (uint32_t)(e / L) * O + i, role = veg_c5_role(k, p);
  uint64_t w = e % L;
  uint32_t v = veg_cfg1_value(seed, role, e);
  uint32_t pre = v;                                    /* cfg1's per-role pre rule */
  if (role >= 8) {
    if (role == 8 || role == 11 || role == 13) pre = 0;
    else if (role == 9) pre = (e % 2 == 0) ? v : (v ^ 1u);
    else pre = v ^ 1u;
  }
  int covered = ((w / 32) * P + p) * 32 + w % 32 < n;
  return (post && role >= 8 && covered) ? v : pre;
}

#endif /* VE_GEN_CORE_H */
