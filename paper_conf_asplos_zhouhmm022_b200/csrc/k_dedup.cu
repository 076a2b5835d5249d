// k_dedup.cu -- K7 / K8: duplicate objects (C11).
//
// Def 3.2: objects D1, D2 with the same values.  The paper groups
// SHA256 digests of the post snapshots; here a chunk-parallel,
// order-free 64-bit content hash (sum over 8-byte words of a position-keyed
// mix, so any reduction order gives the same value) only FILTERS candidates:
// every class is then byte-verified against its representative (K8), so a hash
// collision can never produce a false duplicate ("no false positives").
#include <cuda_runtime.h>

#include <algorithm>
#include <map>
#include <vector>

#include "ve_internal.cuh"

namespace ve {

__device__ __forceinline__ uint64_t word_mix(uint64_t w, uint64_t j) {
  return mix64(w ^ (j * 0x9E3779B97F4A7C15ull) ^ 0x5851F42D4C957F2Dull) + j;
}

struct HashJob {          // one chunk of one object: bytes [off, off + len) of p (size bytes in total)
  const uint8_t* p;
  uint64_t size, off, len;
  uint32_t pos, pad;     // the object's slot in the hash array
};

// K7: one CTA per chunk of <= DD_CH bytes; the hash is a sum over the object's 8-byte words of a
// position-keyed mix, so the chunks' partial sums simply add (any order, any split)
constexpr uint64_t DD_CH = 1ull << 20;
__global__ void __launch_bounds__(256) k_hash(const HashJob* jobs, unsigned long long* hash) {
  const HashJob jb = jobs[blockIdx.x];
  unsigned long long acc = 0;
  const uint64_t w0 = jb.off / 8, w1 = (jb.off + jb.len + 7) / 8;    // the chunk's words (off is 8-aligned)
  if (((uintptr_t)jb.p & 15) == 0 && (jb.off & 15) == 0) {
    const uint64_t v0 = jb.off / 16, v1 = (jb.off + jb.len) / 16 < jb.size / 16 ? (jb.off + jb.len) / 16 : jb.size / 16;
    const uint4* v = (const uint4*)jb.p;
    uint64_t i = v0 + threadIdx.x;
    for (; i + 3 * 256 < v1; i += 4 * 256) {   // four independent 16-byte loads in flight per thread
      uint4 x[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) x[u] = __ldcs(v + i + u * 256);
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const uint64_t k = i + u * 256;
        acc += word_mix(((uint64_t)x[u].y << 32) | x[u].x, 2 * k) + word_mix(((uint64_t)x[u].w << 32) | x[u].z, 2 * k + 1);
      }
    }
    for (; i < v1; i += 256) {
      const uint4 x = __ldcs(v + i);
      acc += word_mix(((uint64_t)x.y << 32) | x.x, 2 * i) + word_mix(((uint64_t)x.w << 32) | x.z, 2 * i + 1);
    }
    // the chunk's words beyond its whole 16-byte blocks (the object's tail, incl. a partial word)
    for (uint64_t j = 2 * v1 + threadIdx.x; j < w1 && j * 8 < jb.size; j += 256) {
      uint64_t w = 0;
      for (uint64_t b = 0; b < 8 && j * 8 + b < jb.size; ++b) w |= (uint64_t)jb.p[j * 8 + b] << (8 * b);
      acc += word_mix(w, j);
    }
  } else {
    for (uint64_t j = w0 + threadIdx.x; j < w1 && j * 8 < jb.size; j += 256) {
      uint64_t w = 0;
      for (uint64_t b = 0; b < 8 && j * 8 + b < jb.size; ++b) w |= (uint64_t)jb.p[j * 8 + b] << (8 * b);
      acc += word_mix(w, j);
    }
  }
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xFFFFFFFFu, acc, o);
  if ((threadIdx.x & 31) == 0 && acc) atomicAdd(&hash[jb.pos], acc);
}

struct CmpJob {
  const uint8_t* a;
  const uint8_t* b;
  uint64_t off, len;   // byte range of this chunk
  uint32_t pair;
  uint32_t pad;
};

// K8: bytewise verification of (member, representative) pairs, 256 KiB per CTA
__global__ void __launch_bounds__(256) k_compare(const CmpJob* jobs, unsigned long long* differs) {
  const CmpJob jb = jobs[blockIdx.x];
  // early exit when another chunk of the pair already differs: decided once per block (thread 0
  // reads the flag) so every thread takes the same branch before __syncthreads_or below
  __shared__ unsigned int s_skip;
  if (threadIdx.x == 0) s_skip = *(volatile unsigned long long*)&differs[jb.pair] != 0ull;
  __syncthreads();
  if (s_skip) return;
  bool diff = false;
  const uint8_t* a = jb.a + jb.off;
  const uint8_t* b = jb.b + jb.off;
  if ((((uintptr_t)a | (uintptr_t)b) & 15) == 0) {
    const uint64_t nv = jb.len / 16;
    uint64_t i = threadIdx.x;
    for (; i + 3 * blockDim.x < nv; i += 4 * blockDim.x) {   // 8 independent 16-byte loads in flight
      uint4 x[4], y[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        x[u] = __ldcs((const uint4*)a + i + u * blockDim.x);
        y[u] = __ldcs((const uint4*)b + i + u * blockDim.x);
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) diff |= (x[u].x != y[u].x) | (x[u].y != y[u].y) | (x[u].z != y[u].z) | (x[u].w != y[u].w);
    }
    for (; i < nv; i += blockDim.x) {
      const uint4 x = __ldcs((const uint4*)a + i), y = __ldcs((const uint4*)b + i);
      diff |= (x.x != y.x) | (x.y != y.y) | (x.z != y.z) | (x.w != y.w);
    }
    for (uint64_t k = nv * 16 + threadIdx.x; k < jb.len; k += blockDim.x) diff |= a[k] != b[k];
  } else {
    for (uint64_t k = threadIdx.x; k < jb.len; k += blockDim.x) diff |= a[k] != b[k];
  }
  if (__syncthreads_or(diff) && threadIdx.x == 0) atomicOr(&differs[jb.pair], 1ull);
}

// K7 of the eligible objects k (positions in elig) with k mod G == rank into d_hash[k]: every owned
// object cut into DD_CH-byte chunk jobs, one CTA each (sizes from KiB to hundreds of MiB balance)
static ve_status hash_launch(ve_ctx* c, const ve_object* objs, const std::vector<uint32_t>& elig, int G, int rank,
                             unsigned long long* d_hash, cudaStream_t s) {
  std::vector<HashJob> hj;
  for (size_t k = 0; k < elig.size(); ++k) {
    if ((int)(k % G) != rank) continue;
    const ve_object& o = objs[elig[k]];
    for (uint64_t off = 0; off < o.size; off += DD_CH)
      hj.push_back(HashJob{(const uint8_t*)o.post, o.size, off, std::min(DD_CH, o.size - off), (uint32_t)k, 0});
  }
  if (hj.empty()) return VE_OK;
  HashJob* d_jobs = nullptr;
  cudaError_t e = cudaMallocAsync((void**)&d_jobs, hj.size() * sizeof(HashJob), s);
  if (e != cudaSuccess) return cuda_fail(c, e, "dedup hash jobs");
  cudaMemcpyAsync(d_jobs, hj.data(), hj.size() * sizeof(HashJob), cudaMemcpyHostToDevice, s);
  for (size_t j0 = 0; j0 < hj.size(); j0 += (1u << 30)) {
    count_launch();
    k_hash<<<(unsigned)std::min<size_t>(hj.size() - j0, 1u << 30), 256, 0, s>>>(d_jobs + j0, d_hash);
  }
  cudaFreeAsync(d_jobs, s);
  e = cudaStreamSynchronize(s);      // (hj is a host vector of this call)
  return e == cudaSuccess ? VE_OK : cuda_fail(c, e, "dedup hash");
}

ve_status dedup_ranks(const std::vector<ve_ctx*>& cs, Comm& comm, const ve_object* objs, uint32_t n,
                      uint32_t* group_of, cudaStream_t s) {
  ve_ctx* c0 = cs[0];
  const int G = comm.G;
  for (uint32_t i = 0; i < n; ++i) group_of[i] = objs[i].id;
  std::vector<uint32_t> elig;
  for (uint32_t i = 0; i < n; ++i)
    if (objs[i].size > 0 && objs[i].post) elig.push_back(i);
  if (elig.size() < 2) return VE_OK;
  const size_t ne = elig.size();
  // K7 on the owned objects, then a SUM allreduce: every rank holds every hash
  std::vector<void*> hb(cs.size());
  for (size_t i = 0; i < cs.size(); ++i) {
    cudaError_t e = cudaMallocAsync(&hb[i], ne * 8, s);
    if (e != cudaSuccess) return cuda_fail(c0, e, "dedup alloc");
    cudaMemsetAsync(hb[i], 0, ne * 8, s);
    ve_status st = hash_launch(cs[i], objs, elig, G, comm.local[i], (unsigned long long*)hb[i], s);
    if (st != VE_OK) return st;
  }
  if (!comm.allreduce(hb, ne, OP_SUM, s)) return fail(c0, VE_ERR_NCCL, "dedup hash allreduce: " + comm.err);
  std::vector<unsigned long long> h(ne);
  cudaMemcpyAsync(h.data(), hb[0], ne * 8, cudaMemcpyDeviceToHost, s);
  for (size_t i = 0; i < cs.size(); ++i) cudaFreeAsync(hb[i], s);
  cudaError_t e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c0, e, "dedup hash");

  // candidate groups: equal (size, hash); members ordered by id (the same on every rank)
  std::map<std::pair<uint64_t, uint64_t>, std::vector<uint32_t>> groups;
  for (size_t k = 0; k < ne; ++k) groups[{objs[elig[k]].size, h[k]}].push_back(elig[k]);
  std::vector<std::vector<uint32_t>> pending;
  for (auto& g : groups) {
    if (g.second.size() < 2) continue;
    std::sort(g.second.begin(), g.second.end(), [&](uint32_t a, uint32_t b) { return objs[a].id < objs[b].id; });
    pending.push_back(g.second);
  }
  // K8: verify every member against its class representative (lowest id); pair p is checked by rank
  // p mod G, the flags are SUM-allreduced; mismatches form a new pending group
  const uint64_t CH = 1 << 18;   // 256 KiB per verification CTA
  while (!pending.empty()) {
    std::vector<std::pair<uint32_t, uint32_t>> pairs;  // (group index, member index)
    for (uint32_t gi = 0; gi < pending.size(); ++gi)
      for (uint32_t mi = 1; mi < pending[gi].size(); ++mi) pairs.push_back({gi, mi});
    const size_t np = pairs.size();
    std::vector<void*> db(cs.size());
    for (size_t i = 0; i < cs.size(); ++i) {
      std::vector<CmpJob> jobs;
      for (size_t p = 0; p < np; ++p) {
        if ((int)(p % G) != comm.local[i]) continue;
        const auto& g = pending[pairs[p].first];
        const ve_object& rep = objs[g[0]];
        const ve_object& m = objs[g[pairs[p].second]];
        for (uint64_t off = 0; off < m.size; off += CH)
          jobs.push_back(CmpJob{(const uint8_t*)m.post, (const uint8_t*)rep.post, off, std::min(CH, m.size - off),
                                (uint32_t)p, 0});
      }
      e = cudaMallocAsync(&db[i], np * 8 + jobs.size() * sizeof(CmpJob), s);
      if (e != cudaSuccess) return cuda_fail(c0, e, "dedup verify alloc");
      unsigned long long* d_diff = (unsigned long long*)db[i];
      CmpJob* d_cj = (CmpJob*)((uint8_t*)db[i] + np * 8);
      cudaMemsetAsync(d_diff, 0, np * 8, s);
      if (!jobs.empty()) {
        cudaMemcpyAsync(d_cj, jobs.data(), jobs.size() * sizeof(CmpJob), cudaMemcpyHostToDevice, s);
        for (size_t j0 = 0; j0 < jobs.size(); j0 += (1u << 30)) {
          const unsigned gxx = (unsigned)std::min<size_t>(jobs.size() - j0, 1u << 30);
          count_launch();
          k_compare<<<gxx, 256, 0, s>>>(d_cj + j0, d_diff);
        }
      }
      cudaStreamSynchronize(s);   // (jobs is a host vector of this iteration)
    }
    if (!comm.allreduce(db, np, OP_SUM, s)) return fail(c0, VE_ERR_NCCL, "dedup verify allreduce: " + comm.err);
    std::vector<unsigned long long> diff(np);
    cudaMemcpyAsync(diff.data(), db[0], np * 8, cudaMemcpyDeviceToHost, s);
    for (size_t i = 0; i < cs.size(); ++i) cudaFreeAsync(db[i], s);
    e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return cuda_fail(c0, e, "dedup verify");
    std::vector<std::vector<uint32_t>> next(pending.size());
    for (size_t p = 0; p < np; ++p) {
      const auto& g = pending[pairs[p].first];
      const uint32_t mem = g[pairs[p].second];
      if (!diff[p]) group_of[mem] = objs[g[0]].id;
      else next[pairs[p].first].push_back(mem);
    }
    pending.clear();
    for (auto& g : next)
      if (g.size() >= 2) pending.push_back(g);
  }
  return VE_OK;
}

ve_status run_dedup(ve_ctx* c, const ve_object* objs, uint32_t n, uint32_t* group_of, cudaStream_t s) {
  LocalComm one;
  return dedup_ranks({c}, one, objs, n, group_of, s);
}

}  // namespace ve
