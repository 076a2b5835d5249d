// k_diff.cu -- K5: snapshot diff (C10).
//
// Def 3.1 and section 5.1: compare the pre and post value
// snapshots of an object element by element, restricted to the addresses the
// API wrote (the written-element bitmap W) or to all elements or a
// caller mask.  HBM-bound: each warp streams 512 contiguous bytes of pre and
// of post per instruction (128-bit coalesced loads, 4 in flight per thread),
// compares per element, and counts masked / unchanged elements with popcounts.
#include <cuda_runtime.h>

#include <cstring>
#include <vector>

#include "ve_internal.cuh"

namespace ve {

// per-16-byte equality bits of its 16/ew elements, LSB = first element
__device__ __forceinline__ uint32_t eq_bits16(const uint4& a, const uint4& b, uint32_t ew_lg) {
  const uint32_t x[4] = {a.x ^ b.x, a.y ^ b.y, a.z ^ b.z, a.w ^ b.w};
  uint32_t r = 0;
  if (ew_lg == 3) {
    r = ((x[0] | x[1]) == 0) | (((x[2] | x[3]) == 0) << 1);
  } else if (ew_lg == 2) {
#pragma unroll
    for (int i = 0; i < 4; ++i) r |= (uint32_t)(x[i] == 0) << i;
  } else if (ew_lg == 1) {
#pragma unroll
    for (int i = 0; i < 4; ++i)
      r |= ((uint32_t)((x[i] & 0xFFFFu) == 0) | ((uint32_t)((x[i] >> 16) == 0) << 1)) << (2 * i);
  } else {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const uint32_t z = __vcmpeq4(x[i], 0u);  // 0xFF per equal byte
      r |= (((z >> 0) & 1u) | ((z >> 7) & 2u) | ((z >> 14) & 4u) | ((z >> 21) & 8u)) << (4 * i);
    }
  }
  return r;
}

// vector part: bytes [0, nvec*16) of 16-byte aligned pre/post
__global__ void __launch_bounds__(256) k_diff_vec(const uint4* __restrict__ pre, const uint4* __restrict__ post,
                                                  uint64_t nvec, uint32_t ew_lg, const uint32_t* __restrict__ mask,
                                                  unsigned long long* out /* [2] masked, unchanged */) {
  const uint32_t per = 16u >> ew_lg;  // elements per 16 bytes
  unsigned long long cm = 0, cu = 0;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  constexpr int U = 4;
  // the mask bits of a 16-byte block are read first: blocks without masked elements load nothing
  // (B_diff = 2 x masked bytes + mask)
  const uint32_t full = (per == 32u) ? 0xFFFFFFFFu : ((1u << per) - 1u);
  if (mask) {
    // warp-level pass: a warp takes 32 mask words (1024 elements) at a time, skips them at once when
    // none is set (an unwritten object's W-mode diff read its mask 16 times per word: 0.18 ms per
    // GiB), else diffs their 16-byte blocks lane-strided (coalesced)
    const int lane = threadIdx.x & 31;
    const uint64_t nwd = (nvec * per) / 32;              // whole mask words inside the vector part
    const uint64_t nchunk = nwd / 32;
    const uint64_t wst = stride / 32;
    for (uint64_t c = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) / 32; c < nchunk; c += wst) {
      const uint32_t mw = __ldg(mask + c * 32 + lane);
      if (!__any_sync(0xFFFFFFFFu, mw != 0u)) continue;
      const uint64_t b0 = c * 32 * 32 / per, nb = 32u * 32u / per;   // the chunk's 16-byte blocks
      for (uint64_t k = lane; k < nb; k += 32) {
        const uint64_t bi = b0 + k, e0 = bi * per;
        const uint32_t m = full & (__ldg(mask + (e0 >> 5)) >> (e0 & 31));
        if (!m) continue;
        const uint4 a = __ldcs(pre + bi), b = __ldcs(post + bi);
        const uint32_t q = eq_bits16(a, b, ew_lg);
        cm += __popc(m);
        cu += __popc(m & q);
      }
    }
    i = nchunk * 32 * 32 / per + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;   // the rest below
  }
  for (; i + (U - 1) * stride < nvec; i += U * stride) {
    uint32_t m[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t e0 = (i + u * stride) * per;
      m[u] = mask ? full & (__ldg(mask + (e0 >> 5)) >> (e0 & 31)) : full;
    }
    uint4 a[U], b[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      a[u] = b[u] = make_uint4(0, 0, 0, 0);
      if (m[u]) { a[u] = __ldcs(pre + i + u * stride); b[u] = __ldcs(post + i + u * stride); }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint32_t q = eq_bits16(a[u], b[u], ew_lg);
      cm += __popc(m[u]);
      cu += __popc(m[u] & q);
    }
  }
  for (; i < nvec; i += stride) {
    const uint64_t e0 = i * per;
    const uint32_t m = mask ? full & (__ldg(mask + (e0 >> 5)) >> (e0 & 31)) : full;
    if (!m) continue;
    const uint4 a = __ldcs(pre + i), b = __ldcs(post + i);
    const uint32_t q = eq_bits16(a, b, ew_lg);
    cm += __popc(m);
    cu += __popc(m & q);
  }
  for (int o = 16; o > 0; o >>= 1) {
    cm += __shfl_xor_sync(0xFFFFFFFFu, cm, o);
    cu += __shfl_xor_sync(0xFFFFFFFFu, cu, o);
  }
  __shared__ unsigned long long sm[8], su[8];
  if ((threadIdx.x & 31) == 0) { sm[threadIdx.x >> 5] = cm; su[threadIdx.x >> 5] = cu; }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long a = 0, b = 0;
    for (int w = 0; w < 8; ++w) { a += sm[w]; b += su[w]; }
    if (a) atomicAdd(&out[0], a);
    if (b) atomicAdd(&out[1], b);
  }
}

// scalar part: elements [e_begin, n_elems) byte by byte (tail, or unaligned snapshots)
__global__ void k_diff_scalar(const uint8_t* pre, const uint8_t* post, uint64_t size, uint32_t ew,
                              uint64_t e_begin, uint64_t n_elems, const uint32_t* mask,
                              unsigned long long* out) {
  unsigned long long cm = 0, cu = 0;
  for (uint64_t e = e_begin + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < n_elems;
       e += (uint64_t)gridDim.x * blockDim.x) {
    if (mask && !((mask[e >> 5] >> (e & 31)) & 1u)) continue;
    const uint64_t b0 = e * ew;
    const uint64_t b1 = (b0 + ew <= size) ? b0 + ew : size;
    bool same = true;
    for (uint64_t b = b0; b < b1; ++b) same &= (pre[b] == post[b]);
    cm += 1;
    cu += same;
  }
  if (cm) atomicAdd(&out[0], cm);
  if (cu) atomicAdd(&out[1], cu);
}

// |W u L| of one object's bitmap words (n_untouched = n_elems - this)
__global__ void __launch_bounds__(256) k_touched(const uint32_t* __restrict__ W, const uint32_t* __restrict__ L,
                                                 uint64_t nw, unsigned long long* out) {
  unsigned long long n = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nw; i += (uint64_t)gridDim.x * blockDim.x)
    n += __popc(W[i] | L[i]);
  for (int o = 16; o; o >>= 1) n += __shfl_xor_sync(0xFFFFFFFFu, n, o);
  if ((threadIdx.x & 31) == 0 && n) atomicAdd(out, n);
}

ve_status run_diff(ve_ctx* c, uint32_t oi, uint32_t mode, const uint32_t* d_mask, ve_diff* out, cudaStream_t s) {
  const HostObject& o = c->objs[oi];
  ctx_begin(c, s);
  // counted loads set their L bits when flushed: flush first, so n_untouched does not
  // depend on whether ve_report ran before this call (idempotent; ve_report skips it then)
  if (!c->hist_merged) {
    ve_status st = dense_flush(c, s);
    if (st != VE_OK) return st;
  }
  if (!o.pre || !o.post) return fail(c, VE_ERR_INVALID, "ve_snapshot_diff: object needs pre and post snapshots");
  const uint32_t* mask = nullptr;
  if (mode == VE_DIFF_WRITTEN) mask = c->t.W + o.bmoff;
  else if (mode == VE_DIFF_MASK) {
    if (!d_mask) return fail(c, VE_ERR_INVALID, "ve_snapshot_diff: VE_DIFF_MASK needs d_mask");
    mask = d_mask;
  } else if (mode != VE_DIFF_ALL) {
    return fail(c, VE_ERR_INVALID, "ve_snapshot_diff: bad mode");
  }
  const uint32_t ew_lg = o.ew == 1 ? 0 : o.ew == 2 ? 1 : o.ew == 4 ? 2 : 3;
  unsigned long long* d_out = nullptr;   // [0] masked, [1] unchanged, [2] |W u L|
  cudaError_t e = cudaMallocAsync((void**)&d_out, 24, s);
  if (e != cudaSuccess) return cuda_fail(c, e, "diff alloc");
  cudaMemsetAsync(d_out, 0, 24, s);
  const bool aligned = (o.pre % 16 == 0) && (o.post % 16 == 0);
  uint64_t e_begin = 0;
  if (aligned) {
    const uint64_t nvec = o.size / 16;
    if (nvec) {
      uint64_t blocks = (nvec + 255) / 256;
      const uint64_t cap = (uint64_t)c->num_sms * 8;
      if (blocks > cap) blocks = cap;
      count_launch();
      k_diff_vec<<<(unsigned)blocks, 256, 0, s>>>((const uint4*)o.pre, (const uint4*)o.post, nvec, ew_lg, mask,
                                                 d_out);
    }
    e_begin = nvec * 16 / o.ew;
  }
  if (e_begin < o.n_elems) {
    const uint64_t rem = o.n_elems - e_begin;
    uint64_t blocks = (rem + 255) / 256;
    if (blocks > (uint64_t)c->num_sms * 8) blocks = (uint64_t)c->num_sms * 8;
    count_launch();
    k_diff_scalar<<<(unsigned)blocks, 256, 0, s>>>((const uint8_t*)o.pre, (const uint8_t*)o.post, o.size, o.ew,
                                                  e_begin, o.n_elems, mask, d_out);
  }
  // n_untouched = n_elems - |W u L|, counted in the same stream (one read-back)
  if (o.bmwords) {
    uint64_t blocks = (o.bmwords + 255) / 256;
    if (blocks > (uint64_t)c->num_sms * 4) blocks = (uint64_t)c->num_sms * 4;
    count_launch();
    k_touched<<<(unsigned)blocks, 256, 0, s>>>(c->t.W + o.bmoff, c->t.L + o.bmoff, o.bmwords, d_out + 2);
  }
  unsigned long long h[3];
  cudaMemcpyAsync(h, d_out, 24, cudaMemcpyDeviceToHost, s);
  cudaFreeAsync(d_out, s);
  ctx_end(c, s);
  e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c, e, "ve_snapshot_diff");
  out->n_elems = o.n_elems;
  out->n_masked = h[0];
  out->n_unchanged = h[1];
  out->n_changed = h[0] - h[1];
  out->n_untouched = o.n_elems - h[2];
  out->redundant = (h[0] > 0 && (unsigned __int128)100 * h[1] > (unsigned __int128)c->cfg.t_redundant_pct * h[0]);
  out->pad = 0;
  return VE_OK;
}

}  // namespace ve

namespace ve {
// S10 of every object with both snapshots (mode WRITTEN or ALL), sharded by object over comm: the
// object at position k of the ctx's sorted table is diffed by rank k mod G; each rank's results go
// into a u64 table [n_obj][5] (zero where it does not own), SUM-allreduced, then unpacked by id.
// Objects without both snapshots report n_elems only.  Every context must hold the same objects
// (the merged state of a rank merge).
ve_status diff_ranks(const std::vector<ve_ctx*>& cs, Comm& comm, uint32_t mode, ve_diff* out_by_id, cudaStream_t s) {
  ve_ctx* c0 = cs[0];
  if (mode != VE_DIFF_WRITTEN && mode != VE_DIFF_ALL)
    return fail(c0, VE_ERR_INVALID, "ve_snapshot_diff_all: mode must be VE_DIFF_WRITTEN or VE_DIFF_ALL");
  const uint32_t n = c0->n_obj;
  for (ve_ctx* c : cs)
    if (c->n_obj != n) return fail(c0, VE_ERR_INVALID, "ve_snapshot_diff_all: contexts hold different objects");
  if (n == 0) return VE_OK;
  const int G = comm.G;
  std::vector<void*> bufs(cs.size());
  for (size_t i = 0; i < cs.size(); ++i) {
    ve_ctx* c = cs[i];
    std::vector<unsigned long long> tab((size_t)n * 5, 0ull);
    for (uint32_t k = 0; k < n; ++k) {
      if ((int)(k % G) != comm.local[i]) continue;
      const HostObject& o = c->objs[k];
      if (!o.pre || !o.post) continue;
      ve_diff d;
      ve_status st = run_diff(c, k, mode, nullptr, &d, s);
      if (st != VE_OK) return st;
      unsigned long long* r = &tab[(size_t)k * 5];
      r[0] = 1; r[1] = d.n_masked; r[2] = d.n_unchanged; r[3] = d.n_untouched; r[4] = 0;
    }
    cudaError_t e = cudaMallocAsync(&bufs[i], tab.size() * 8, s);
    if (e != cudaSuccess) return cuda_fail(c0, e, "diff_all alloc");
    cudaMemcpyAsync(bufs[i], tab.data(), tab.size() * 8, cudaMemcpyHostToDevice, s);
    e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return cuda_fail(c0, e, "diff_all");
  }
  if (!comm.allreduce(bufs, (size_t)n * 5, OP_SUM, s)) return fail(c0, VE_ERR_NCCL, "diff allreduce: " + comm.err);
  std::vector<unsigned long long> tab((size_t)n * 5);
  cudaMemcpyAsync(tab.data(), bufs[0], tab.size() * 8, cudaMemcpyDeviceToHost, s);
  for (void* b : bufs) cudaFreeAsync(b, s);
  cudaError_t e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c0, e, "diff_all");
  for (uint32_t k = 0; k < n; ++k) {
    const HostObject& o = c0->objs[k];
    const unsigned long long* r = &tab[(size_t)k * 5];
    ve_diff& d = out_by_id[o.id];
    memset(&d, 0, sizeof(d));
    d.n_elems = o.n_elems;
    if (!r[0]) continue;
    d.n_masked = r[1];
    d.n_unchanged = r[2];
    d.n_changed = r[1] - r[2];
    d.n_untouched = r[3];
    d.redundant = (r[1] > 0 && (unsigned __int128)100 * r[2] > (unsigned __int128)c0->cfg.t_redundant_pct * r[1]);
  }
  return VE_OK;
}
}  // namespace ve
