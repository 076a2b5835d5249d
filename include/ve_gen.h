/*
 * ve_gen.h -- C ABI of libvegen.so, the seeded synthetic-input generator.
 *
 * TEST / BENCH INPUTS ONLY.  Not part of the analysis boundary (include/ve.h).
 * Produces the value traces and object snapshots of DESIGN.md section 4
 * (the configs of BASELINE.json, shapes of SURVEY.md 8(d)) as pure
 * functions of (cfg, epoch, seed, index), bit-identically on host and device.
 *
 *   cfg: VEG_CFG1 (1)  single kernel, 2^20 4-byte records, 16 PCs, one 4 MiB object
 *        VEG_CFG2 (2)  Darknet YOLOv4 conv layer; epoch 0 fill_ongpu, epoch 1 gemm
 *        VEG_CFG3 (3)  PyTorch op mix (4 epochs = iterations, seed 3 + iteration)
 *        VEG_CFG4 (4)  f64 stencils; epoch 0 hotspot3D-like, epoch 1 Castro-like
 *                      (cfg3 / cfg4 | s << 8: tensors 2^s times smaller)
 *        VEG_FUZZ (100) adversarial mixed trace (unbounded record stream)
 *   Dedup sets: veg_dedup_* (object i of a set keyed by seed and size unit; unit 0 = the cfg5
 *   recipe: 50 log-uniform size classes over [64 KiB, 512 MiB], rescaled to 20 GiB per 1000 objects).
 *
 * Return 0 on success, -1 on bad arguments / launch failure.  Device calls are
 * asynchronous on stream s; d_out is caller-owned device memory (8-byte
 * aligned).  Host calls write caller-owned host memory.
 */
#ifndef VE_GEN_H
#define VE_GEN_H
#include <stdint.h>
#include <cuda_runtime_api.h>
#include "../gen/ve_gen_core.h"

#ifdef __cplusplus
extern "C" {
#endif

int veg_info_get(int cfg, int epoch, veg_info* out);
int veg_object_get(int cfg, int epoch, uint32_t i, veg_object* out);
void veg_records_host(int cfg, int epoch, uint64_t seed, uint64_t r0, uint64_t n, veg_record* out);
int veg_records_device(int cfg, int epoch, uint64_t seed, uint64_t r0, uint64_t n, veg_record* d_out,
                       cudaStream_t s);
void veg_snapshot_host(int cfg, int epoch, uint64_t seed, uint32_t obj, int post, uint64_t off, uint64_t len,
                       uint8_t* out);
int veg_snapshot_device(int cfg, int epoch, uint64_t seed, uint32_t obj, int post, uint8_t* d_out,
                        cudaStream_t s);
int veg_dedup_object(uint64_t seed, uint32_t i, uint64_t unit, veg_object* out, uint32_t* cls, uint32_t* src);
void veg_dedup_host(uint64_t seed, uint32_t i, uint64_t unit, uint8_t* out);
int veg_dedup_device(uint64_t seed, uint32_t i, uint64_t unit, uint8_t* d_out, cudaStream_t s);

#ifdef __cplusplus
}
#endif
#endif
