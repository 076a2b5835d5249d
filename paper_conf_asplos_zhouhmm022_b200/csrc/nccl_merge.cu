// nccl_merge.cu -- S12 across ranks: every rank ends with the
// merged statistics of all ranks.
//
//   1. SUM / MIN / MAX blocks and globals          -> allreduce
//   2. line states                                 -> allgather, folded with (+) in rank order
//   3. W / L element bitmaps                       -> allgather, OR
//   4. exact value histogram: each rank builds its per-PC / per-object view
//      entries, hash-partitions them to owner ranks (all-to-all), owners sum the
//      counts of a disjoint key space, compute per-key partial n_distinct and
//      top-k; allreduce of n_distinct, allgather of the owners' top-k, re-rank.
//      Exact, because the partitions are disjoint and their counts global.
//
// One algorithm, two transports: NCCL (one rank per process/GPU; NCCL is
// dlopen'ed so libve has no link-time dependency) and same-device simulated
// ranks (ve_merge_group), which the single-GPU tests use to check the partition
// logic bit-for-bit against the oracle.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <vector>

#include "ve_internal.cuh"

namespace ve {

// ---- transports (Comm: ve_internal.cuh) --------------------------------------------
__global__ void k_reduce_u64(unsigned long long* dst, const unsigned long long* src, size_t n, int op) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    const unsigned long long a = dst[i], b = src[i];
    dst[i] = op == OP_SUM ? a + b : op == OP_MIN ? (a < b ? a : b) : (a > b ? a : b);
  }
}

// same-device simulated ranks: local i is global rank i
struct SimComm : Comm {
  bool allreduce(const std::vector<void*>& bufs, size_t count, int op, cudaStream_t s) override {
    for (size_t i = 1; i < bufs.size(); ++i) {
      count_launch();
      k_reduce_u64<<<256, 256, 0, s>>>((unsigned long long*)bufs[0], (const unsigned long long*)bufs[i], count, op);
    }
    for (size_t i = 1; i < bufs.size(); ++i) cudaMemcpyAsync(bufs[i], bufs[0], count * 8, cudaMemcpyDeviceToDevice, s);
    return cudaGetLastError() == cudaSuccess;
  }
  bool allgather(const std::vector<const void*>& send, const std::vector<void*>& recv, size_t bytes,
                 cudaStream_t s) override {
    for (size_t i = 0; i < recv.size(); ++i)
      for (size_t g = 0; g < send.size(); ++g)
        if (bytes) cudaMemcpyAsync((uint8_t*)recv[i] + g * bytes, send[g], bytes, cudaMemcpyDeviceToDevice, s);
    return cudaGetLastError() == cudaSuccess;
  }
  bool alltoallv(const std::vector<const uint8_t*>& send, const std::vector<std::vector<size_t>>& soff,
                 const std::vector<std::vector<size_t>>& sbytes, const std::vector<uint8_t*>& recv,
                 const std::vector<std::vector<size_t>>& roff, const std::vector<std::vector<size_t>>& rbytes,
                 cudaStream_t s) override {
    for (size_t r = 0; r < recv.size(); ++r)
      for (size_t g = 0; g < send.size(); ++g) {
        if (sbytes[g][r] != rbytes[r][g]) return false;
        if (sbytes[g][r]) cudaMemcpyAsync(recv[r] + roff[r][g], send[g] + soff[g][r], sbytes[g][r],
                                          cudaMemcpyDeviceToDevice, s);
      }
    return cudaGetLastError() == cudaSuccess;
  }
};

// ---- NCCL, loaded at run time ------------------------------------------------------
struct NcclApi {
  bool ok = false;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*CommCount)(const ncclComm_t, int*) = nullptr;
  ncclResult_t (*CommUserRank)(const ncclComm_t, int*) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

static NcclApi& nccl() {
  static NcclApi api;
  static bool tried = false;
  if (tried) return api;
  tried = true;
  void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
  if (!h) return api;
#define VE_SYM(name, field) api.field = reinterpret_cast<decltype(api.field)>(dlsym(h, name))
  VE_SYM("ncclGetUniqueId", GetUniqueId);
  VE_SYM("ncclCommInitRank", CommInitRank);
  VE_SYM("ncclCommDestroy", CommDestroy);
  VE_SYM("ncclCommCount", CommCount);
  VE_SYM("ncclCommUserRank", CommUserRank);
  VE_SYM("ncclAllReduce", AllReduce);
  VE_SYM("ncclAllGather", AllGather);
  VE_SYM("ncclSend", Send);
  VE_SYM("ncclRecv", Recv);
  VE_SYM("ncclGroupStart", GroupStart);
  VE_SYM("ncclGroupEnd", GroupEnd);
  VE_SYM("ncclGetErrorString", GetErrorString);
#undef VE_SYM
  api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.CommCount && api.CommUserRank &&
           api.AllReduce && api.AllGather && api.Send && api.Recv && api.GroupStart && api.GroupEnd;
  return api;
}

struct NcclComm : Comm {
  ncclComm_t comm;
  bool check(ncclResult_t r) {
    if (r != ncclSuccess) err = nccl().GetErrorString ? nccl().GetErrorString(r) : "nccl error";
    return r == ncclSuccess;
  }
  bool allreduce(const std::vector<void*>& bufs, size_t count, int op, cudaStream_t s) override {
    const ncclRedOp_t o = op == OP_SUM ? ncclSum : op == OP_MIN ? ncclMin : ncclMax;
    return check(nccl().AllReduce(bufs[0], bufs[0], count, ncclUint64, o, comm, s));
  }
  bool allgather(const std::vector<const void*>& send, const std::vector<void*>& recv, size_t bytes,
                 cudaStream_t s) override {
    return check(nccl().AllGather(send[0], recv[0], bytes, ncclUint8, comm, s));
  }
  bool alltoallv(const std::vector<const uint8_t*>& send, const std::vector<std::vector<size_t>>& soff,
                 const std::vector<std::vector<size_t>>& sbytes, const std::vector<uint8_t*>& recv,
                 const std::vector<std::vector<size_t>>& roff, const std::vector<std::vector<size_t>>& rbytes,
                 cudaStream_t s) override {
    if (!check(nccl().GroupStart())) return false;
    for (int g = 0; g < G; ++g) {
      if (sbytes[0][g] && !check(nccl().Send(send[0] + soff[0][g], sbytes[0][g], ncclUint8, g, comm, s))) break;
      if (rbytes[0][g] && !check(nccl().Recv(recv[0] + roff[0][g], rbytes[0][g], ncclUint8, g, comm, s))) break;
    }
    return check(nccl().GroupEnd()) && err.empty();
  }
};

// ---- merge kernels ------------------------------------------------------------------
__global__ void k_fold_lines(LineState* out, const LineState* all, uint32_t n_keys, int G) {
  for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < n_keys; k += gridDim.x * blockDim.x) {
    LinePts r = line_load(all[k]);
    for (int g = 1; g < G; ++g) r = line_merge(r, line_load(all[(size_t)g * n_keys + k]));
    LineState& o = out[k];
    line_store(o, r);
    o.lock = 0;
  }
}

__global__ void k_or_words(uint32_t* out, const uint32_t* all, uint64_t words, int G) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < words; i += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t v = 0;
    for (int g = 0; g < G; ++g) v |= all[(size_t)g * words + i];
    out[i] = v;
  }
}

struct Entry {            // one (view key, value) count
  uint64_t bits, count;
  uint32_t key, pad;
};

__device__ __forceinline__ uint32_t owner_of(uint32_t key, uint64_t bits, int G) {
  return (uint32_t)(mix64(bits ^ ((uint64_t)key << 40) ^ 0x7A3C5E1F00000000ull) % (uint64_t)G);
}

__global__ void k_owner_count(const HSlot* vs, const unsigned long long* vc, uint64_t vcap, int G,
                              unsigned long long* counts) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < vcap; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t tag = vs[i].tag;
    if (tag != EMPTY_TAG) atomicAdd(&counts[owner_of(tag, vs[i].bits, G)], 1ull);
  }
}

__global__ void k_owner_scatter(const HSlot* vs, const unsigned long long* vc, uint64_t vcap, int G,
                                unsigned long long* cursor, Entry* out) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < vcap; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t tag = vs[i].tag;
    if (tag == EMPTY_TAG) continue;
    const uint64_t b = vs[i].bits;
    const unsigned long long p = atomicAdd(&cursor[owner_of(tag, b, G)], 1ull);
    Entry e;
    e.bits = b;
    e.count = vc[i];
    e.key = tag;
    e.pad = 0;
    out[p] = e;
  }
}

__global__ void k_insert_entries(const Entry* in, uint64_t n, HSlot* vs, unsigned long long* vc, uint64_t vmask,
                                 unsigned long long* overflow) {
  DevTables t{};
  t.hslot = vs;
  t.hcount = vc;
  t.hmask = vmask;
  t.glob = overflow - G_OVERFLOW;   // hist_insert_global flags glob[G_OVERFLOW]
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    hist_insert_global_rf(t, in[i].key, in[i].bits, in[i].count);
}

static bool same_layout(const ve_ctx* a, const ve_ctx* b) {
  if (a->n_keys != b->n_keys || a->n_obj != b->n_obj || a->bm_words != b->bm_words || a->cfg.topk != b->cfg.topk)
    return false;
  for (uint32_t i = 0; i < a->n_obj; ++i)
    if (a->objs[i].base != b->objs[i].base || a->objs[i].size != b->objs[i].size || a->objs[i].ew != b->objs[i].ew ||
        a->objs[i].id != b->objs[i].id)
      return false;
  return true;
}

// The merge algorithm over the local contexts cs (1 for NCCL, all G for simulated ranks).
static ve_status merge_ranks(const std::vector<ve_ctx*>& cs, Comm& comm, cudaStream_t s) {
  ve_ctx* c0 = cs[0];
  const int G = comm.G;
  const size_t L = cs.size();
  for (ve_ctx* c : cs) {
    if (c->poisoned || c->hist_merged) return fail(c0, VE_ERR_STATE, "merge: a context is poisoned or merged");
    if (!same_layout(c0, c)) return fail(c0, VE_ERR_INVALID, "merge: contexts differ in config or objects");
  }
  for (ve_ctx* c : cs) {
    ve_status st = dense_flush(c, s);
    if (st != VE_OK) return st;
  }
  const uint32_t nk = c0->n_keys, K = c0->cfg.topk;
  auto nccl_fail = [&](const char* what) { return fail(c0, VE_ERR_NCCL, std::string(what) + ": " + comm.err); };
  // 1. SUM / MIN / MAX blocks and globals
  {
    std::vector<void*> b;
    for (ve_ctx* c : cs) b.push_back(c->t.sum);
    if (!comm.allreduce(b, (size_t)nk * NSUM, OP_SUM, s)) return nccl_fail("allreduce sum");
    b.clear();
    for (ve_ctx* c : cs) b.push_back(c->t.mn);
    if (!comm.allreduce(b, (size_t)nk * NMM, OP_MIN, s)) return nccl_fail("allreduce min");
    b.clear();
    for (ve_ctx* c : cs) b.push_back(c->t.mx);
    if (!comm.allreduce(b, (size_t)nk * NMM, OP_MAX, s)) return nccl_fail("allreduce max");
    b.clear();
    for (ve_ctx* c : cs) b.push_back(c->t.glob);
    if (!comm.allreduce(b, 4, OP_SUM, s)) return nccl_fail("allreduce globals");
  }
  // 2. line states, 3. bitmaps: allgather then fold
  {
    std::vector<void*> gl(L), gw(L), gL(L);
    const size_t lb = (size_t)nk * sizeof(LineState), wb = c0->bm_words * 4;
    for (size_t i = 0; i < L; ++i) {
      if (cudaMallocAsync(&gl[i], lb * G, s) != cudaSuccess || cudaMallocAsync(&gw[i], wb * G + 4, s) != cudaSuccess ||
          cudaMallocAsync(&gL[i], wb * G + 4, s) != cudaSuccess)
        return fail(c0, VE_ERR_NOMEM, "merge buffers");
    }
    std::vector<const void*> sl, sw, sL;
    for (ve_ctx* c : cs) { sl.push_back(c->t.line); sw.push_back(c->t.W); sL.push_back(c->t.L); }
    if (!comm.allgather(sl, gl, lb, s)) return nccl_fail("allgather lines");
    if (wb && (!comm.allgather(sw, gw, wb, s) || !comm.allgather(sL, gL, wb, s))) return nccl_fail("allgather bitmaps");
    for (size_t i = 0; i < L; ++i) {
      count_launch();
      k_fold_lines<<<64, 256, 0, s>>>(cs[i]->t.line, (const LineState*)gl[i], nk, G);
      if (wb) {
        count_launch();
        k_or_words<<<cs[i]->num_sms * 4, 256, 0, s>>>(cs[i]->t.W, (const uint32_t*)gw[i], cs[i]->bm_words, G);
        count_launch();
        k_or_words<<<cs[i]->num_sms * 4, 256, 0, s>>>(cs[i]->t.L, (const uint32_t*)gL[i], cs[i]->bm_words, G);
      }
      cudaFreeAsync(gl[i], s);
      cudaFreeAsync(gw[i], s);
      cudaFreeAsync(gL[i], s);
    }
  }
  // 4. exact histogram: partition view entries to owners
  std::vector<ViewTable> V(L), V2(L);
  std::vector<Entry*> sendb(L, nullptr), recvb(L, nullptr);
  std::vector<std::vector<size_t>> soff(L, std::vector<size_t>(G)), sbytes(L, std::vector<size_t>(G)),
      roff(L, std::vector<size_t>(G)), rbytes(L, std::vector<size_t>(G));
  std::vector<unsigned long long*> dcnt(L);
  std::vector<void*> cnt_all(L);
  for (size_t i = 0; i < L; ++i) {
    ve_status st = build_views(cs[i], s, V[i]);
    if (st != VE_OK) return st;
    cudaMallocAsync((void**)&dcnt[i], 8 * G * 2, s);
    cudaMemsetAsync(dcnt[i], 0, 8 * G * 2, s);
    count_launch();
    k_owner_count<<<cs[i]->num_sms * 4, 256, 0, s>>>(V[i].vs, V[i].vc, V[i].vcap, G, dcnt[i]);
    cudaMallocAsync(&cnt_all[i], 8 * G * G, s);
  }
  {
    std::vector<const void*> snd;
    for (size_t i = 0; i < L; ++i) snd.push_back(dcnt[i]);
    if (!comm.allgather(snd, cnt_all, 8 * G, s)) return nccl_fail("allgather counts");
  }
  for (size_t i = 0; i < L; ++i) {
    std::vector<unsigned long long> m((size_t)G * G);
    cudaMemcpyAsync(m.data(), cnt_all[i], 8 * G * G, cudaMemcpyDeviceToHost, s);
    if (cudaStreamSynchronize(s) != cudaSuccess) return cuda_fail(c0, cudaGetLastError(), "merge counts");
    const int me = comm.local[i];
    size_t so = 0, ro = 0;
    for (int g = 0; g < G; ++g) {
      soff[i][g] = so * sizeof(Entry);
      sbytes[i][g] = m[(size_t)me * G + g] * sizeof(Entry);   // row me: what I send to g
      so += m[(size_t)me * G + g];
      roff[i][g] = ro * sizeof(Entry);
      rbytes[i][g] = m[(size_t)g * G + me] * sizeof(Entry);   // what g sends to me
      ro += m[(size_t)g * G + me];
    }
    cudaMallocAsync((void**)&sendb[i], so * sizeof(Entry) + 8, s);
    cudaMallocAsync((void**)&recvb[i], ro * sizeof(Entry) + 8, s);
    std::vector<unsigned long long> cur(G);
    for (int g = 0; g < G; ++g) cur[g] = soff[i][g] / sizeof(Entry);
    cudaMemcpyAsync(dcnt[i] + G, cur.data(), 8 * G, cudaMemcpyHostToDevice, s);
    count_launch();
    k_owner_scatter<<<cs[i]->num_sms * 4, 256, 0, s>>>(V[i].vs, V[i].vc, V[i].vcap, G, dcnt[i] + G, sendb[i]);
    ve_status st = alloc_views(cs[i], s, ro, V2[i]);
    if (st != VE_OK) return st;
    rbytes[i].push_back(ro);   // remember the received entry count at the end
  }
  {
    std::vector<const uint8_t*> snd;
    std::vector<uint8_t*> rcv;
    std::vector<std::vector<size_t>> rb(L);
    for (size_t i = 0; i < L; ++i) {
      snd.push_back((const uint8_t*)sendb[i]);
      rcv.push_back((uint8_t*)recvb[i]);
      rb[i].assign(rbytes[i].begin(), rbytes[i].begin() + G);
    }
    if (!comm.alltoallv(snd, soff, sbytes, rcv, roff, rb, s)) return nccl_fail("all-to-all entries");
  }
  std::vector<std::vector<uint64_t>> nd(L);
  std::vector<std::vector<ve_topk_entry>> tk(L);
  for (size_t i = 0; i < L; ++i) {
    const uint64_t ro = rbytes[i][G];
    unsigned long long* ovf = dcnt[i];      // reuse as an overflow flag slot
    cudaMemsetAsync(ovf, 0, 8, s);
    if (ro) {
      count_launch();
      k_insert_entries<<<cs[i]->num_sms * 4, 256, 0, s>>>(recvb[i], ro, V2[i].vs, V2[i].vc, V2[i].vcap - 1, ovf);
    }
    ve_status st = view_topk(cs[i], V2[i], s, nd[i], tk[i]);
    if (st != VE_OK) return st;
    free_views(V[i], s);
    free_views(V2[i], s);
    cudaFreeAsync(sendb[i], s);
    cudaFreeAsync(recvb[i], s);
  }
  // n_distinct: allreduce of the owners' partial counts; top-k: allgather + re-rank
  std::vector<void*> ndb(L), tkb(L), tka(L);
  for (size_t i = 0; i < L; ++i) {
    cudaMallocAsync(&ndb[i], 8 * nk, s);
    cudaMemcpyAsync(ndb[i], nd[i].data(), 8 * nk, cudaMemcpyHostToDevice, s);
    cudaMallocAsync(&tkb[i], sizeof(ve_topk_entry) * nk * K, s);
    cudaMemcpyAsync(tkb[i], tk[i].data(), sizeof(ve_topk_entry) * nk * K, cudaMemcpyHostToDevice, s);
    cudaMallocAsync(&tka[i], sizeof(ve_topk_entry) * nk * K * G, s);
  }
  if (!comm.allreduce(ndb, nk, OP_SUM, s)) return nccl_fail("allreduce n_distinct");
  {
    std::vector<const void*> snd(tkb.begin(), tkb.end());
    if (!comm.allgather(snd, tka, sizeof(ve_topk_entry) * nk * K, s)) return nccl_fail("allgather top-k");
  }
  for (size_t i = 0; i < L; ++i) {
    ve_ctx* c = cs[i];
    c->merged_ndistinct.assign(nk, 0);
    std::vector<ve_topk_entry> all((size_t)nk * K * G);
    cudaMemcpyAsync(c->merged_ndistinct.data(), ndb[i], 8 * nk, cudaMemcpyDeviceToHost, s);
    cudaMemcpyAsync(all.data(), tka[i], all.size() * sizeof(ve_topk_entry), cudaMemcpyDeviceToHost, s);
    unsigned long long ovf = 0;
    cudaMemcpyAsync(&ovf, dcnt[i], 8, cudaMemcpyDeviceToHost, s);
    if (cudaStreamSynchronize(s) != cudaSuccess) return cuda_fail(c0, cudaGetLastError(), "merge results");
    if (ovf) return fail(c0, VE_ERR_CAPACITY, "merge: owner view table overflow");
    c->merged_topk.assign((size_t)nk * K, ve_topk_entry{0, 0});
    std::vector<ve_topk_entry> cand;
    for (uint32_t k = 0; k < nk; ++k) {
      cand.clear();
      for (int g = 0; g < G; ++g)
        for (uint32_t j = 0; j < K; ++j) {
          const ve_topk_entry& e = all[((size_t)g * nk + k) * K + j];
          if (e.count) cand.push_back(e);
        }
      std::sort(cand.begin(), cand.end(), [](const ve_topk_entry& a, const ve_topk_entry& b) {
        return a.count > b.count || (a.count == b.count && a.bits < b.bits);
      });
      for (size_t j = 0; j < cand.size() && j < K; ++j) c->merged_topk[(size_t)k * K + j] = cand[j];
    }
    c->hist_merged = true;
    cudaFreeAsync(ndb[i], s);
    cudaFreeAsync(tkb[i], s);
    cudaFreeAsync(tka[i], s);
    cudaFreeAsync(dcnt[i], s);
    cudaFreeAsync(cnt_all[i], s);
  }
  cudaError_t e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c0, e, "merge");
  return VE_OK;
}

ve_status merge_nccl(ve_ctx* c, void* comm_ptr, cudaStream_t s) {
  if (!nccl().ok) return fail(c, VE_ERR_NCCL, "NCCL library not available");
  NcclComm comm;
  comm.comm = (ncclComm_t)comm_ptr;
  int G = 0, me = 0;
  if (nccl().CommCount(comm.comm, &G) != ncclSuccess || nccl().CommUserRank(comm.comm, &me) != ncclSuccess)
    return fail(c, VE_ERR_NCCL, "bad NCCL communicator");
  comm.G = G;
  comm.local = {me};
  return merge_ranks({c}, comm, s);
}

}  // namespace ve

using namespace ve;

extern "C" {

ve_status ve_merge_group(ve_ctx** ctxs, uint32_t n, cudaStream_t s) {
  if (!ctxs || n == 0) return VE_ERR_INVALID;
  std::vector<ve_ctx*> cs(ctxs, ctxs + n);
  for (ve_ctx* c : cs)
    if (!c || c->device != cs[0]->device) return VE_ERR_INVALID;
  cudaSetDevice(cs[0]->device);
  SimComm comm;
  comm.G = (int)n;
  for (uint32_t i = 0; i < n; ++i) comm.local.push_back((int)i);
  for (ve_ctx* c : cs) ctx_begin(c, s);
  const ve_status st = merge_ranks(cs, comm, s);
  for (ve_ctx* c : cs) ctx_end(c, s);
  return st;
}

// S10 / S11 sharded by object: see diff_ranks / dedup_ranks
static ve_status comm_of(ve_ctx* c, void* comm_ptr, NcclComm& comm) {
  if (!nccl().ok) return fail(c, VE_ERR_NCCL, "NCCL library not available");
  comm.comm = (ncclComm_t)comm_ptr;
  int G = 0, me = 0;
  if (nccl().CommCount(comm.comm, &G) != ncclSuccess || nccl().CommUserRank(comm.comm, &me) != ncclSuccess)
    return fail(c, VE_ERR_NCCL, "bad NCCL communicator");
  comm.G = G;
  comm.local = {me};
  return VE_OK;
}

ve_status ve_snapshot_diff_all(ve_ctx* ctx, uint32_t mode, void* nccl_comm_or_null, ve_diff* h_out, cudaStream_t s) {
  if (!ctx || !h_out) return VE_ERR_INVALID;
  cudaSetDevice(ctx->device);
  if (!nccl_comm_or_null) {
    LocalComm one;
    return diff_ranks({ctx}, one, mode, h_out, s);
  }
  NcclComm comm;
  ve_status st = comm_of(ctx, nccl_comm_or_null, comm);
  return st != VE_OK ? st : diff_ranks({ctx}, comm, mode, h_out, s);
}

ve_status ve_object_dedup_comm(ve_ctx* ctx, const ve_object* objs, uint32_t n, void* nccl_comm, uint32_t* h_group_of,
                               cudaStream_t s) {
  if (!ctx || !nccl_comm || (n && (!objs || !h_group_of))) return VE_ERR_INVALID;
  cudaSetDevice(ctx->device);
  NcclComm comm;
  ve_status st = comm_of(ctx, nccl_comm, comm);
  ctx_begin(ctx, s);
  return st != VE_OK ? st : dedup_ranks({ctx}, comm, objs, n, h_group_of, s);
}

ve_status ve_snapshot_diff_all_group(ve_ctx** ctxs, uint32_t n, uint32_t mode, ve_diff* h_out, cudaStream_t s) {
  if (!ctxs || n == 0 || !h_out) return VE_ERR_INVALID;
  std::vector<ve_ctx*> cs(ctxs, ctxs + n);
  for (ve_ctx* c : cs)
    if (!c || c->device != cs[0]->device) return VE_ERR_INVALID;
  cudaSetDevice(cs[0]->device);
  SimComm comm;
  comm.G = (int)n;
  for (uint32_t i = 0; i < n; ++i) comm.local.push_back((int)i);
  return diff_ranks(cs, comm, mode, h_out, s);
}

ve_status ve_object_dedup_group(ve_ctx** ctxs, uint32_t n, const ve_object* objs, uint32_t n_objs, uint32_t* h_group_of,
                                cudaStream_t s) {
  if (!ctxs || n == 0 || (n_objs && (!objs || !h_group_of))) return VE_ERR_INVALID;
  std::vector<ve_ctx*> cs(ctxs, ctxs + n);
  for (ve_ctx* c : cs)
    if (!c || c->device != cs[0]->device) return VE_ERR_INVALID;
  cudaSetDevice(cs[0]->device);
  SimComm comm;
  comm.G = (int)n;
  for (uint32_t i = 0; i < n; ++i) comm.local.push_back((int)i);
  for (ve_ctx* c : cs) ctx_begin(c, s);
  return dedup_ranks(cs, comm, objs, n_objs, h_group_of, s);
}

ve_status ve_nccl_get_unique_id(void* out128) {
  if (!out128) return VE_ERR_INVALID;
  if (!nccl().ok) return VE_ERR_NCCL;
  ncclUniqueId id;
  if (nccl().GetUniqueId(&id) != ncclSuccess) return VE_ERR_NCCL;
  memcpy(out128, &id, sizeof(id));
  return VE_OK;
}

ve_status ve_nccl_comm_init(void** comm_out, int nranks, const void* id128, int rank) {
  if (!comm_out || !id128 || nranks < 1 || rank < 0 || rank >= nranks) return VE_ERR_INVALID;
  if (!nccl().ok) return VE_ERR_NCCL;
  ncclUniqueId id;
  memcpy(&id, id128, sizeof(id));
  ncclComm_t comm;
  if (nccl().CommInitRank(&comm, nranks, id, rank) != ncclSuccess) return VE_ERR_NCCL;
  *comm_out = comm;
  return VE_OK;
}

ve_status ve_nccl_comm_destroy(void* comm) {
  if (!comm) return VE_ERR_INVALID;
  if (!nccl().ok) return VE_ERR_NCCL;
  return nccl().CommDestroy((ncclComm_t)comm) == ncclSuccess ? VE_OK : VE_ERR_NCCL;
}

}  // extern "C"
