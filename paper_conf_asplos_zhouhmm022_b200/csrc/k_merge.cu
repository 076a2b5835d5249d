// k_merge.cu -- S12 / C12: merging statistics of two contexts on one device.
//
// The statistics are a commutative monoid (SUM adds, MIN/MAX, line states
// under (+), histogram counts add per (key, value) before top-k, bitmaps OR),
// so analyzing A then B, analyzing A u B, and merging the stats of A and B all
// give the same report (the paper's chunked buffer flushes).
#include <cuda_runtime.h>

#include "ve_internal.cuh"

namespace ve {

__global__ void k_merge_tables(DevTables d, DevTables s, uint32_t n_keys, uint64_t bm_words) {
  const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = tid; i < (uint64_t)n_keys * NSUM; i += stride) d.sum[i] += s.sum[i];
  for (uint64_t i = tid; i < (uint64_t)n_keys * NMM; i += stride) {
    if (s.mn[i] < d.mn[i]) d.mn[i] = s.mn[i];
    if (s.mx[i] > d.mx[i]) d.mx[i] = s.mx[i];
  }
  for (uint64_t k = tid; k < n_keys; k += stride) {
    LinePts r = line_merge(line_load(d.line[k]), line_load(s.line[k]));
    line_store(d.line[k], r);
  }
  for (uint64_t i = tid; i < bm_words; i += stride) {
    d.W[i] |= s.W[i];
    d.L[i] |= s.L[i];
  }
  if (tid < 3) d.glob[tid] += s.glob[tid];
  if (tid == 3 && s.glob[G_OVERFLOW]) d.glob[G_OVERFLOW] = 1;
}

__global__ void k_merge_hist(DevTables d, const HSlot* shs, const unsigned long long* shc, uint64_t scap) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < scap; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t tag = shs[i].tag;
    if (tag != EMPTY_TAG) hist_insert_global_rf(d, tag, shs[i].bits, shc[i]);
  }
}

ve_status merge_local(ve_ctx* dst, const ve_ctx* src, cudaStream_t s) {
  if (dst->n_keys != src->n_keys || dst->n_obj != src->n_obj || dst->bm_words != src->bm_words ||
      dst->device != src->device)
    return fail(dst, VE_ERR_INVALID, "ve_merge_stats: contexts differ in config, objects or device");
  for (uint32_t i = 0; i < dst->n_obj; ++i)
    if (dst->objs[i].base != src->objs[i].base || dst->objs[i].size != src->objs[i].size ||
        dst->objs[i].ew != src->objs[i].ew || dst->objs[i].id != src->objs[i].id)
      return fail(dst, VE_ERR_INVALID, "ve_merge_stats: object tables differ");
  // dense per-element counts move into each side's exact histogram first
  ve_status st = dense_flush(dst, s);
  if (st != VE_OK) return st;
  st = dense_flush(const_cast<ve_ctx*>(src), s);
  if (st != VE_OK) return fail(dst, st, "ve_merge_stats: src: " + src->err);
  const int grid = dst->num_sms * 4;
  count_launch();
  k_merge_tables<<<grid, 256, 0, s>>>(dst->t, src->t, dst->n_keys, dst->bm_words);
  count_launch();
  k_merge_hist<<<grid, 256, 0, s>>>(dst->t, src->t.hslot, src->t.hcount, src->hcap);
  cudaError_t e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(dst, e, "ve_merge_stats (local)");
  if (src->poisoned) dst->poisoned = true;
  return VE_OK;
}

}  // namespace ve
