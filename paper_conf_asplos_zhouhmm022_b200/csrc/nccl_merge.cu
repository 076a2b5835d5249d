// nccl_merge.cu -- S12 across ranks; placeholder until the
// collective merge lands: NCCL is loaded at run time (dlopen) so libve.so has
// no link-time NCCL dependency.
#include <cuda_runtime.h>
#include <dlfcn.h>

#include "ve_internal.cuh"

namespace ve {
ve_status merge_nccl(ve_ctx* c, void* comm, cudaStream_t s) {
  (void)comm;
  (void)s;
  return fail(c, VE_ERR_NCCL, "ve_merge_stats: NCCL merge not built yet");
}
}  // namespace ve

extern "C" {
ve_status ve_nccl_get_unique_id(void* out128) {
  (void)out128;
  return VE_ERR_NCCL;
}
ve_status ve_nccl_comm_init(void** comm_out, int nranks, const void* id128, int rank) {
  (void)comm_out; (void)nranks; (void)id128; (void)rank;
  return VE_ERR_NCCL;
}
ve_status ve_nccl_comm_destroy(void* comm) {
  (void)comm;
  return VE_ERR_NCCL;
}
}
