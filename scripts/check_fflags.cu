// Exhaustive equivalence check of the closed-form float flags used by the K1 fast
// path against the generic definition (float_flags) -- every binary32 pattern and
// every binary16 / bfloat16 pattern.  Run on a GPU box:
//   nvcc -gencode arch=compute_100a,code=sm_100a -std=c++17 -Iinclude \
//        -Ipaper_conf_asplos_zhouhmm022_b200/csrc scripts/check_fflags.cu -o /tmp/chk && /tmp/chk
#include <cstdio>

#include "ve_internal.cuh"

using namespace ve;

__global__ void k_check32(unsigned long long* bad, unsigned long long* first) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < (1ull << 32); i += stride) {
    const uint32_t b = (uint32_t)i;
    int64_t iv;
    const uint32_t g = float_flags(b, 2u, 2u, iv);
    if (g != fflags_f32(b)) {
      atomicAdd(bad, 1ull);
      atomicMin(first, (unsigned long long)b);
    }
  }
}

int main() {
  unsigned long long *bad, *first;
  cudaMallocManaged(&bad, 8);
  cudaMallocManaged(&first, 8);
  *bad = 0;
  *first = ~0ull;
  k_check32<<<148 * 8, 256>>>(bad, first);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { printf("cuda error %s\n", cudaGetErrorString(e)); return 2; }
  printf("fflags_f32: %llu mismatches over 2^32 patterns (first 0x%llx)\n", *bad, *first);
  return *bad ? 1 : 0;
}
