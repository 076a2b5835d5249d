/*
 * ve_gen.cu -- libvegen.so: the seeded input generator (ve_gen_core.h) on the
 * host and on the device behind a small C ABI (include/ve_gen.h).  Test and
 * bench inputs only; holds no analysis arithmetic.
 */
#include <cuda_runtime.h>
#include <stdint.h>
#include "ve_gen_core.h"
#include "../include/ve_gen.h"

VEG_FN uint64_t snap_word(int cfg, int epoch, uint64_t seed, uint32_t obj, int post, uint64_t j) {
  if (cfg == VEG_CFG1) {
    uint64_t e = 2 * j;
    uint64_t lo = post ? veg_cfg1_post(seed, e) : veg_cfg1_pre(seed, e);
    uint64_t hi = post ? veg_cfg1_post(seed, e + 1) : veg_cfg1_pre(seed, e + 1);
    return lo | (hi << 32);
  }
  if (cfg == VEG_CFG2) {
    uint64_t e = 2 * j;
    uint64_t lo = veg_cfg2_elem(seed, (uint32_t)epoch, obj, post, e);
    uint64_t hi = veg_cfg2_elem(seed, (uint32_t)epoch, obj, post, e + 1);
    return lo | (hi << 32);
  }
  if (VEG_BASE(cfg) == VEG_CFG3) {
    const uint32_t sh = VEG_SHIFT(cfg);
    if (veg_c3_object(sh, obj).elem_width == 8) return veg_c3_elem(seed, sh, obj, post, j);
    return veg_c3_elem(seed, sh, obj, post, 2 * j) | (veg_c3_elem(seed, sh, obj, post, 2 * j + 1) << 32);
  }
  if (VEG_BASE(cfg) == VEG_CFG4) return veg_c4_elem(seed, VEG_SHIFT(cfg), (uint32_t)epoch, obj, post, j);
  if (VEG_BASE(cfg) == VEG_CFG5) {
    const uint32_t sh = VEG_SHIFT(cfg);
    return (uint64_t)veg_c5_elem(seed, sh, (uint32_t)epoch, obj, post, 2 * j) |
           ((uint64_t)veg_c5_elem(seed, sh, (uint32_t)epoch, obj, post, 2 * j + 1) << 32);
  }
  if (cfg == VEG_FUZZ) return veg_fuzz_word(seed, obj, post, j);
  return 0;
}

VEG_FN void record_at(int cfg, int epoch, uint64_t seed, uint64_t r, veg_record* out) {
  if (cfg == VEG_CFG1) veg_cfg1_record(seed, r, out);
  else if (cfg == VEG_CFG2) veg_cfg2_record(seed, (uint32_t)epoch, r, out);
  else if (VEG_BASE(cfg) == VEG_CFG3) veg_cfg3_record(seed, VEG_SHIFT(cfg), r, out);
  else if (VEG_BASE(cfg) == VEG_CFG4) veg_cfg4_record(seed, VEG_SHIFT(cfg), (uint32_t)epoch, r, out);
  else if (VEG_BASE(cfg) == VEG_CFG5) veg_cfg5_record(seed, VEG_SHIFT(cfg), (uint32_t)epoch, r, out);
  else veg_fuzz_record(seed, r, out);
}

extern "C" int veg_info_get(int cfg, int epoch, veg_info* out) {
  if (!out) return -1;
  out->pad = 0;
  if (cfg == VEG_CFG1) {
    if (epoch != 0) return -1;
    out->n_records = VEG_CFG1_N; out->n_pcs = 16; out->n_obj = 1; out->n_epochs = 1;
    return 0;
  }
  if (cfg == VEG_CFG2) {
    if (epoch < 0 || epoch > 1) return -1;
    out->n_records = epoch == 0 ? VEG_C2_FILL_N : VEG_C2_GEMM_N;
    out->n_pcs = 5; out->n_obj = 4; out->n_epochs = 2;
    return 0;
  }
  if (VEG_BASE(cfg) == VEG_CFG3) {                /* one epoch per training iteration (seed 3 + it) */
    if (epoch < 0 || epoch > 3 || VEG_SHIFT(cfg) > 7 || (cfg & ~0xFFF)) return -1;
    out->n_records = veg_c3_n(VEG_SHIFT(cfg)); out->n_pcs = VEG_C3_NPCS; out->n_obj = VEG_C3_NOBJ;
    out->n_epochs = 4;
    return 0;
  }
  if (VEG_BASE(cfg) == VEG_CFG4) {                /* epoch 0 hotspot3D-like, epoch 1 Castro-like */
    if (epoch < 0 || epoch > 1 || VEG_SHIFT(cfg) > 4 || (cfg & ~0xFFF)) return -1;
    out->n_records = veg_c4_n(VEG_SHIFT(cfg), (uint32_t)epoch); out->n_pcs = VEG_C4_NPCS; out->n_obj = 6;
    out->n_epochs = 2;
    return 0;
  }
  if (VEG_BASE(cfg) == VEG_CFG5) {                /* one epoch per kernel of the 4000-kernel application */
    if (epoch < 0 || epoch >= (int)VEG_C5_KERNELS || VEG_SHIFT(cfg) > 7 || (cfg & ~0xFFF)) return -1;
    out->n_records = veg_c5_n(VEG_SHIFT(cfg), (uint32_t)epoch);
    out->n_pcs = veg_c5_npcs((uint32_t)epoch); out->n_obj = veg_c5_nobj((uint32_t)epoch);
    out->n_epochs = VEG_C5_KERNELS;
    return 0;
  }
  if (cfg == VEG_FUZZ) {
    if (epoch != 0) return -1;
    out->n_records = 0; out->n_pcs = VEG_FZ_NPCS; out->n_obj = VEG_FZ_NOBJ; out->n_epochs = 1;
    return 0;
  }
  return -1;
}

extern "C" int veg_object_get(int cfg, int epoch, uint32_t i, veg_object* out) {
  veg_info inf;
  if (veg_info_get(cfg, epoch, &inf) != 0 || i >= inf.n_obj || !out) return -1;
  if (cfg == VEG_CFG1) {
    out->base = VEG_CFG1_BASE; out->size = 4 * VEG_CFG1_N; out->id = 0; out->elem_width = 4;
    out->has_pre = 1; out->has_post = 1;
  } else if (cfg == VEG_CFG2) {
    *out = veg_cfg2_object(i);
  } else if (VEG_BASE(cfg) == VEG_CFG3) {
    *out = veg_c3_object(VEG_SHIFT(cfg), i);
  } else if (VEG_BASE(cfg) == VEG_CFG4) {
    *out = veg_c4_object(VEG_SHIFT(cfg), i);
  } else if (VEG_BASE(cfg) == VEG_CFG5) {
    *out = veg_c5_object(VEG_SHIFT(cfg), (uint32_t)epoch, i);
  } else {
    *out = veg_fuzz_object(i);
  }
  return 0;
}

extern "C" void veg_records_host(int cfg, int epoch, uint64_t seed, uint64_t r0, uint64_t n, veg_record* out) {
  for (uint64_t i = 0; i < n; ++i) record_at(cfg, epoch, seed, r0 + i, &out[i]);
}

__global__ void k_records(int cfg, int epoch, uint64_t seed, uint64_t r0, uint64_t n, veg_record* out) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    veg_record rec;
    record_at(cfg, epoch, seed, r0 + i, &rec);
    out[i] = rec;
  }
}

extern "C" int veg_records_device(int cfg, int epoch, uint64_t seed, uint64_t r0, uint64_t n, veg_record* d_out,
                                  cudaStream_t s) {
  if (n == 0) return 0;
  uint64_t blocks = (n + 255) / 256;
  if (blocks > 148 * 64) blocks = 148 * 64;
  k_records<<<(unsigned)blocks, 256, 0, s>>>(cfg, epoch, seed, r0, n, d_out);
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

extern "C" void veg_snapshot_host(int cfg, int epoch, uint64_t seed, uint32_t obj, int post, uint64_t off,
                                  uint64_t len, uint8_t* out) {
  uint64_t wj = ~0ull, w = 0;
  for (uint64_t p = 0; p < len; ++p) {
    uint64_t b = off + p;
    if (b / 8 != wj) { wj = b / 8; w = snap_word(cfg, epoch, seed, obj, post, wj); }
    out[p] = (uint8_t)(w >> (8 * (b % 8)));
  }
}

__global__ void k_snapshot(int cfg, int epoch, uint64_t seed, uint32_t obj, int post, uint64_t size, uint8_t* out) {
  uint64_t words = (size + 7) / 8;
  for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < words; j += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t v = snap_word(cfg, epoch, seed, obj, post, j);
    if (8 * j + 8 <= size) {
      reinterpret_cast<uint64_t*>(out)[j] = v;                 /* out is 8-byte aligned */
    } else {
      for (uint64_t b = 8 * j; b < size; ++b) out[b] = (uint8_t)(v >> (8 * (b % 8)));
    }
  }
}

extern "C" int veg_snapshot_device(int cfg, int epoch, uint64_t seed, uint32_t obj, int post, uint8_t* d_out,
                                   cudaStream_t s) {
  veg_object o;
  if (veg_object_get(cfg, epoch, obj, &o) != 0) return -1;
  uint64_t blocks = (o.size / 8 + 255) / 256 + 1;
  if (blocks > 148 * 64) blocks = 148 * 64;
  k_snapshot<<<(unsigned)blocks, 256, 0, s>>>(cfg, epoch, seed, obj, post, o.size, d_out);
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

/* ---- dedup object sets --------------------------------------------------- */

/* unit == 0 (the cfg5 recipe): the class sizes of objects 0..999 rescaled so that they total 20 GiB
 * (4 KiB multiples, rounded down; the same factor for every object) */
static uint64_t dedup_scaled(uint64_t seed, uint32_t i) {
  static uint64_t cached_seed = ~0ull;
  static double factor = 1.0;
  if (cached_seed != seed) {
    double tot = 0;
    for (uint32_t j = 0; j < 1000; ++j) tot += (double)veg_dedup_size(seed, j, 0);
    factor = (double)(20ull << 30) / tot;
    cached_seed = seed;
  }
  const uint64_t v = (uint64_t)((double)veg_dedup_size(seed, i, 0) * factor) & ~4095ull;
  return v ? v : 4096;
}

extern "C" int veg_dedup_object(uint64_t seed, uint32_t i, uint64_t unit, veg_object* out, uint32_t* cls,
                                uint32_t* src) {
  if (!out || unit % 8) return -1;
  out->id = i;
  out->base = VEG_DD_BASE + (uint64_t)i * 0x100000000ull;
  out->size = unit ? veg_dedup_size(seed, i, unit) : dedup_scaled(seed, i);
  out->elem_width = 8;
  out->has_pre = 1;
  out->has_post = 1;
  uint32_t s;
  uint32_t c = veg_dedup_class(seed, i, &s, unit);
  if (cls) *cls = c;
  if (src) *src = s;
  return 0;
}

extern "C" void veg_dedup_host(uint64_t seed, uint32_t i, uint64_t unit, uint8_t* out) {
  veg_object o;
  uint32_t cls, src, ssrc;
  veg_dedup_object(seed, i, unit, &o, &cls, &src);
  uint32_t scls = veg_dedup_class(seed, src, &ssrc, unit);
  uint64_t words = o.size / 8;
  for (uint64_t j = 0; j < words; ++j) {
    uint64_t v = veg_dedup_word(seed, i, cls, src, scls, words, j);
    memcpy(out + 8 * j, &v, 8);
  }
}

__global__ void k_dedup(uint64_t seed, uint32_t i, uint32_t cls, uint32_t src, uint32_t scls, uint64_t words,
                        uint64_t* out) {
  for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < words; j += (uint64_t)gridDim.x * blockDim.x)
    out[j] = veg_dedup_word(seed, i, cls, src, scls, words, j);
}

extern "C" int veg_dedup_device(uint64_t seed, uint32_t i, uint64_t unit, uint8_t* d_out, cudaStream_t s) {
  veg_object o;
  uint32_t cls, src, ssrc;
  if (veg_dedup_object(seed, i, unit, &o, &cls, &src) != 0) return -1;
  uint32_t scls = veg_dedup_class(seed, src, &ssrc, unit);
  uint64_t words = o.size / 8;
  uint64_t blocks = (words + 255) / 256;
  if (blocks > 148 * 64) blocks = 148 * 64;
  k_dedup<<<(unsigned)blocks, 256, 0, s>>>(seed, i, cls, src, scls, words, reinterpret_cast<uint64_t*>(d_out));
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}
