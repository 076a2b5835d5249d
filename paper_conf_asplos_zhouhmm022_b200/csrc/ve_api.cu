// ve_api.cu -- the C ABI of include/ve.h: context lifecycle, argument
// validation, the host side of the five hot-path calls, and the report (R1:
// integer threshold tests and the heavy-type lattice).
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <vector>

#include "ve_internal.cuh"

#include <atomic>

namespace ve {

static std::atomic<unsigned long long> g_launches{0};
void count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }

ve_status fail(ve_ctx* c, ve_status s, const std::string& msg) {
  if (c) c->err = msg;
  return s;
}
ve_status cuda_fail(ve_ctx* c, cudaError_t e, const char* where) {
  if (c) c->err = std::string(where) + ": " + cudaGetErrorString(e);
  return VE_ERR_CUDA;
}

static void free_dev(ve_ctx* c) {
  cudaFree(c->t.sum);
  cudaFree(c->t.mn);
  cudaFree(c->t.mx);
  cudaFree(c->t.line);
  cudaFree(c->t.lcta);
  cudaFree(c->t.glob);
  cudaFree(c->t.W);
  cudaFree(c->t.L);
  cudaFree(c->t.hslot);
  cudaFree(c->t.hcount);
  cudaFree(c->t.occ_bm);
  cudaFree(c->obj_block);
  cudaFree(c->scratch);
  cudaFree(c->occ_flat);
  if (c->pin) cudaFreeHost(c->pin);
  if (c->rpin) cudaFreeHost(c->rpin);
  cudaFree(c->dense_pool);
  cudaFree(c->hstage);
  for (int i = 0; i < 2; ++i) {
    if (c->stage[i]) cudaFree(c->stage[i]);
    if (c->stage_ev[i]) cudaEventDestroy(c->stage_ev[i]);
    if (c->copied_ev[i]) cudaEventDestroy(c->copied_ev[i]);
  }
  if (c->copy_stream) cudaStreamDestroy(c->copy_stream);
  if (c->ord_ev) cudaEventDestroy(c->ord_ev);
  if (c->cs) cudaStreamDestroy(c->cs);
}

// grow-only device buffers: freed and allocated stream-ordered on the ctx stream after the ctx's queued
// work (cudaFree / cudaMalloc would synchronise the whole device and stall every other context), then
// one wait on the ctx stream so the new block is valid for whatever stream the caller uses next
cudaError_t ctx_realloc(ve_ctx* c, void** p, size_t bytes) {
  ctx_begin(c, c->cs);
  if (*p) cudaFreeAsync(*p, c->cs);
  *p = nullptr;
  cudaError_t e = cudaMallocAsync(p, bytes, c->cs);
  if (e == cudaSuccess) e = cudaStreamSynchronize(c->cs);
  if (e != cudaSuccess) {
    cudaGetLastError();
    *p = nullptr;
  }
  return e;
}

// make the dense counter pool hold the current object set's claims (dense_want counters), allocated
// on first need; false when there is no memory for it (the calls then count through the hash path)
bool dense_reserve(ve_ctx* c) {
  if (c->dense_want == 0) return false;
  if (c->dense_pool && c->dense_cap >= c->dense_want) return true;
  c->dense_cap = 0;
  c->dense_dirty = false;
  if (ctx_realloc(c, &c->dense_pool, c->dense_want * 4) != cudaSuccess ||
      cudaMemsetAsync(c->dense_pool, 0, c->dense_want * 4, c->cs) != cudaSuccess) {
    cudaGetLastError();
    if (c->dense_pool) cudaFreeAsync(c->dense_pool, c->cs);
    c->dense_pool = nullptr;
    c->dense_want = 0;                                 // no memory: this object set uses the hash path
    return false;
  }
  if (cudaStreamSynchronize(c->cs) != cudaSuccess) return false;   // (rare: the caller's launch follows)
  c->dense_cap = c->dense_want;
  c->o.dense_pool = (uint32_t*)c->dense_pool;
  c->o.dense_cap = c->dense_cap;
  return true;
}

void ctx_begin(ve_ctx* c, cudaStream_t s) {
  if (c->ord_ev) cudaStreamWaitEvent(s, c->ord_ev, 0);
}
void ctx_end(ve_ctx* c, cudaStream_t s) {
  if (c->ord_ev) cudaEventRecord(c->ord_ev, s);
}
cudaError_t ctx_quiesce(ve_ctx* c) {
  return c->ord_ev ? cudaEventSynchronize(c->ord_ev) : cudaSuccess;
}

// empty the slots marked in the occupancy bitmap (the table's only non-empty slots), and the bitmap
__global__ void k_reset_occ(DevTables t) {
  const uint64_t nw = (t.hmask + 1) >> 5;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nw; i += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t w = t.occ_bm[i];
    if (!w) continue;
    t.occ_bm[i] = 0;
    for (; w; w &= w - 1) {
      const uint64_t h = (i << 5) + (uint32_t)(__ffs(w) - 1);
      t.hslot[h].bits = ~0ull;
      t.hslot[h].tag = EMPTY_TAG;
      t.hslot[h].pad = EMPTY_TAG;
      t.hcount[h] = 0;
    }
  }
}

ve_status launch_reset(ve_ctx* c, cudaStream_t s) {
  ctx_begin(c, s);
  const uint64_t nk_max = (uint64_t)c->cfg.n_pcs + c->cfg.max_objects + 1;
  cudaMemsetAsync(c->t.sum, 0, nk_max * NSUM * 8, s);
  cudaMemsetAsync(c->t.mn, 0xFF, nk_max * NMM * 8, s);
  cudaMemsetAsync(c->t.mx, 0, nk_max * NMM * 8, s);
  cudaMemsetAsync(c->t.line, 0, nk_max * sizeof(LineState), s);
  // counts claimed arrays still hold (analysed, never flushed): clear the used pool
  if (c->dense_dirty && c->dense_pool) {
    unsigned long long used = 0;
    cudaMemcpyAsync(&used, c->t.glob + G_DENSE_NEXT, 8, cudaMemcpyDeviceToHost, s);
    cudaStreamSynchronize(s);
    if (used > c->dense_cap) used = c->dense_cap;
    if (used) cudaMemsetAsync(c->dense_pool, 0, used * 4, s);
    c->dense_dirty = false;
  }
  // the value table: a fresh table is filled whole; afterwards only the slots claimed since the last
  // reset (marked in t.occ_bm) are emptied -- O(entries + hist_capacity / 32), per epoch
  const bool full = !c->table_clean;
  if (!full) {
    count_launch();
    k_reset_occ<<<c->num_sms * 4, 256, 0, s>>>(c->t);
  } else {
    cudaMemsetAsync(c->t.occ_bm, 0, c->hcap / 8, s);
  }
  cudaMemsetAsync(c->t.glob, 0, 8 * 8, s);
  if (c->bm_words) {
    cudaMemsetAsync(c->t.W, 0, c->bm_words * 4, s);
    cudaMemsetAsync(c->t.L, 0, c->bm_words * 4, s);
  }
  if (full) cudaMemsetAsync(c->t.hslot, 0xFF, c->hcap * sizeof(HSlot), s);
  if (c->n_obj) {
    cudaMemcpyAsync(c->o.dense_pc, c->dense_pc_init.data(), 4ull * DENSE_PER_OBJ * c->n_obj, cudaMemcpyHostToDevice, s);
    cudaMemsetAsync(c->o.dense_off, 0xFF, 8ull * DENSE_PER_OBJ * c->n_obj, s);   // DENSE_NOT_READY
  }
  c->records_analyzed = 0;
  cudaError_t e = full ? cudaMemsetAsync(c->t.hcount, 0, c->hcap * 8, s) : cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(c, e, "reset");
  c->table_clean = true;
  ctx_end(c, s);
  c->poisoned = false;
  c->hist_merged = false;
  c->merged_ndistinct.clear();
  c->merged_topk.clear();
  return VE_OK;
}

// ---- R1: heavy type from the raw fields (C6) --------------------------------
static int64_t float_int_of_ord(uint64_t ord, uint32_t tc) {
  // invert the orderable key, then decode the (integral) float exactly
  const uint32_t w = (tc == 8 || tc == 11) ? 2 : (tc == 9) ? 4 : 8;
  const uint32_t nb = 8 * w;
  const uint64_t mask = nb == 64 ? ~0ull : ((1ull << nb) - 1);
  const uint64_t sign = 1ull << (nb - 1);
  const uint64_t b = (ord & sign) ? (ord & ~sign) : (~ord & mask);
  int eb, mb;
  if (tc == 11) { eb = 8; mb = 7; } else if (w == 2) { eb = 5; mb = 10; } else if (w == 4) { eb = 8; mb = 23; }
  else { eb = 11; mb = 52; }
  const bool neg = (b >> (nb - 1)) & 1;
  const uint64_t E = (b >> mb) & ((1ull << eb) - 1), M = b & ((1ull << mb) - 1);
  const uint64_t sig = E ? (M | (1ull << mb)) : M;
  const int ex = (E ? (int)E : 1) - ((1 << (eb - 1)) - 1) - mb;
  uint64_t mag;
  if (sig == 0) mag = 0;
  else if (ex >= 0) mag = sig << ex;
  else mag = (-ex >= 64) ? 0 : (sig >> -ex);
  return neg ? -(int64_t)mag : (int64_t)mag;
}

static uint32_t heavy_of(const ve_key_stats& k, uint32_t tc) {
  static const uint32_t wid[12] = {1, 2, 4, 8, 1, 2, 4, 8, 2, 4, 8, 2};
  const uint32_t w = wid[tc];
  const uint32_t cand[3] = {1, 2, 4};
  if (tc <= 3) {
    for (uint32_t v : cand) {
      if (v >= w) break;
      if (k.ord_max <= ((1ull << (8 * v)) - 1)) return v == 1 ? 0 : v == 2 ? 1 : 2;
    }
    return 255;
  }
  if (tc <= 7) {
    const int64_t mn = (int64_t)(k.ord_min ^ (1ull << 63)), mx = (int64_t)(k.ord_max ^ (1ull << 63));
    for (uint32_t v : cand) {
      if (v >= w) break;
      const int64_t lo = -(1ll << (8 * v - 1)), hi = (1ll << (8 * v - 1)) - 1;
      if (mn >= lo && mx <= hi) return v == 1 ? 4 : v == 2 ? 5 : 6;
    }
    return 255;
  }
  for (uint32_t v : cand) {
    if (v >= w) break;
    if (k.n_nonint == 0) {
      const int64_t mn = float_int_of_ord(k.ord_min, tc), mx = float_int_of_ord(k.ord_max, tc);
      if (mn >= 0) {
        if ((uint64_t)mx <= ((1ull << (8 * v)) - 1)) return v == 1 ? 0 : v == 2 ? 1 : 2;
      } else {
        const int64_t lo = -(1ll << (8 * v - 1)), hi = (1ll << (8 * v - 1)) - 1;
        if (mn >= lo && mx <= hi) return v == 1 ? 4 : v == 2 ? 5 : 6;
      }
    }
    if (v == 2 && k.n_not_f16 == 0) return 8;
    if (v == 2 && k.n_not_bf16 == 0) return 11;
    if (v == 4 && k.n_not_f32 == 0) return 9;
  }
  return 255;
}

static void derive(const ve_config& cfg, ve_key_stats& k, const ve_topk_entry* top) {
  static const uint32_t wid[12] = {1, 2, 4, 8, 1, 2, 4, 8, 2, 4, 8, 2};
  const uint64_t n = k.n_ld + k.n_st;
  uint32_t nt = 0, tc = 0;
  for (uint32_t t = 0; t < 12; ++t)
    if (k.n_type[t]) { ++nt; tc = t; }
  k.single_type = nt == 1;
  k.single_value = n > 0 && k.raw_min == k.raw_max;
  k.single_zero = n > 0 && k.n_zero == n;
  k.frequent = k.n_top > 0 && (unsigned __int128)100 * top[0].count > (unsigned __int128)cfg.t_frequent_pct * n;
  k.structured = k.approx = k.dict8 = 0;
  k.heavy = 255;
  if (!k.single_type) return;
  const __int128 py = (__int128)(((unsigned __int128)(uint64_t)k.p_yhi << 64) | k.p_ylo);
  const __int128 qy = (__int128)(((unsigned __int128)(uint64_t)k.q_yhi << 64) | k.q_ylo);
  k.structured = k.line_state == VE_LINE_LINE && py != qy;
  k.approx = tc >= 8 && k.n_nan == 0 && n > 0 && k.trunc_min == k.trunc_max && !k.single_value;
  k.dict8 = k.n_distinct <= 256 && wid[tc] > 1;
  k.heavy = heavy_of(k, tc);
}

static bool ctx_ok(const ve_ctx* c) { return c != nullptr; }

}  // namespace ve

using namespace ve;

extern "C" {

ve_status ve_create(const ve_config* cfg, int cuda_device, ve_ctx** out) {
  if (!cfg || !out) return VE_ERR_INVALID;
  *out = nullptr;
  if (cfg->n_pcs == 0 || cfg->n_pcs > 65535 || cfg->max_objects > 65534 || cfg->topk == 0 || cfg->topk > 64 ||
      cfg->hist_capacity == 0)
    return VE_ERR_INVALID;
  ve_ctx* c = new (std::nothrow) ve_ctx();
  if (!c) return VE_ERR_NOMEM;
  c->cfg = *cfg;
  c->device = cuda_device;
  cudaError_t e = cudaSetDevice(cuda_device);
  if (e != cudaSuccess) { delete c; return VE_ERR_CUDA; }
  cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, cuda_device);
  {
    // keep stream-ordered scratch allocations cached in the pool across synchronizations
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, cuda_device) == cudaSuccess) {
      uint64_t thr = ~0ull;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
  }
  if (cfg->hist_capacity > (1ull << 32)) return VE_ERR_INVALID;   // (slot indices are 32-bit)
  uint64_t hcap = 1024;
  while (hcap < cfg->hist_capacity) hcap <<= 1;
  c->hcap = hcap;
  c->t.hmask = hcap - 1;
  const uint64_t nk_max = (uint64_t)cfg->n_pcs + cfg->max_objects + 1;
  bool ok = cudaMalloc(&c->t.sum, nk_max * NSUM * 8) == cudaSuccess &&
            cudaMalloc(&c->t.mn, nk_max * NMM * 8) == cudaSuccess &&
            cudaMalloc(&c->t.mx, nk_max * NMM * 8) == cudaSuccess &&
            cudaMalloc(&c->t.line, nk_max * sizeof(LineState)) == cudaSuccess &&
            cudaMalloc(&c->t.lcta, (size_t)c->num_sms * K1_NSK * sizeof(LineState)) == cudaSuccess &&
            cudaMalloc(&c->t.glob, 8 * 8) == cudaSuccess &&
            cudaMalloc(&c->t.hslot, hcap * sizeof(HSlot)) == cudaSuccess &&
            cudaMalloc(&c->t.hcount, hcap * 8) == cudaSuccess &&
            cudaMalloc(&c->t.occ_bm, hcap / 8) == cudaSuccess;
  if (!ok) {
    cudaGetLastError();
    free_dev(c);
    delete c;
    return VE_ERR_NOMEM;
  }
  c->n_obj = 0;
  c->n_keys = cfg->n_pcs + 1;
  if (cudaEventCreateWithFlags(&c->ord_ev, cudaEventDisableTiming) != cudaSuccess ||
      cudaStreamCreateWithFlags(&c->cs, cudaStreamNonBlocking) != cudaSuccess) {
    cudaGetLastError();
    free_dev(c);
    delete c;
    return VE_ERR_CUDA;
  }
  if (launch_reset(c, c->cs) != VE_OK || cudaStreamSynchronize(c->cs) != cudaSuccess) {
    free_dev(c);
    delete c;
    return VE_ERR_CUDA;
  }
  *out = c;
  return VE_OK;
}

ve_status ve_destroy(ve_ctx* c) {
  if (!c) return VE_ERR_INVALID;
  cudaSetDevice(c->device);
  ctx_quiesce(c);
  if (c->cs) cudaStreamSynchronize(c->cs);
  free_dev(c);
  delete c;
  return VE_OK;
}

const char* ve_last_error(const ve_ctx* c) { return c ? c->err.c_str() : "null context"; }

// the object table of n objects in units (unit u = the next unit_nobj[u] entries of objs; one unit
// holding all of them for ve_set_objects): sorted by (unit, base), overlaps rejected within a unit
static ve_status set_objects_units(ve_ctx* c, const ve_object* objs, uint32_t n, const uint32_t* unit_nobj,
                                   uint32_t n_units) {
  if (!ctx_ok(c)) return VE_ERR_INVALID;
  if (n > c->cfg.max_objects) return fail(c, VE_ERR_INVALID, "ve_set_objects: n > max_objects");
  if (n && !objs) return fail(c, VE_ERR_INVALID, "ve_set_objects: null objects");
  std::vector<uint32_t> unit_of(n, 0), ustart(n_units + 1, 0);
  if (unit_nobj) {
    uint64_t tot = 0;
    for (uint32_t u = 0; u < n_units; ++u) {
      ustart[u] = (uint32_t)std::min<uint64_t>(tot, n);
      for (uint64_t i = tot; i < tot + unit_nobj[u] && i < n; ++i) unit_of[i] = u;
      tot += unit_nobj[u];
    }
    if (tot != n) return fail(c, VE_ERR_INVALID, "ve_set_units: unit object counts do not sum to n");
    ustart[n_units] = n;
  } else {
    ustart[n_units] = n;       // one unit of every object
  }
  std::vector<HostObject> v(n);
  std::vector<uint32_t> vu(n);
  std::vector<char> seen(n, 0);
  for (uint32_t i = 0; i < n; ++i) {
    const ve_object& o = objs[i];
    const uint32_t ew = o.elem_width;
    if (o.size == 0 || o.id >= n || seen[o.id] || !(ew == 1 || ew == 2 || ew == 4 || ew == 8) ||
        o.base >= (1ull << 48) || o.size > (1ull << 48) - o.base)
      return fail(c, VE_ERR_INVALID, "ve_set_objects: bad object " + std::to_string(i));
    seen[o.id] = 1;
    v[i] = HostObject{o.base, o.size, (uint64_t)(uintptr_t)o.pre, (uint64_t)(uintptr_t)o.post, o.id, ew,
                      (o.size + ew - 1) / ew, 0, 0};
  }
  {
    std::vector<uint32_t> ord(n);
    for (uint32_t i = 0; i < n; ++i) ord[i] = i;
    std::sort(ord.begin(), ord.end(), [&](uint32_t a, uint32_t b) {
      return unit_of[a] != unit_of[b] ? unit_of[a] < unit_of[b] : v[a].base < v[b].base;
    });
    std::vector<HostObject> w(n);
    for (uint32_t i = 0; i < n; ++i) { w[i] = v[ord[i]]; vu[i] = unit_of[ord[i]]; }
    v.swap(w);
  }
  for (uint32_t i = 1; i < n; ++i)
    if (vu[i - 1] == vu[i] && v[i - 1].base + v[i - 1].size > v[i].base)
      return fail(c, VE_ERR_INVALID, "ve_set_objects: overlap");
  uint64_t words = 0;
  for (auto& o : v) {
    o.bmoff = words;
    o.bmwords = (o.n_elems + 31) / 32;
    words += o.bmwords;
  }
  cudaSetDevice(c->device);
  // the buffers below are reused or replaced: the ctx's queued work (any stream) must be done
  // (a wait on this ctx's work only -- other contexts and the application keep running)
  cudaError_t qe = ctx_quiesce(c);
  if (qe != cudaSuccess) return cuda_fail(c, qe, "ve_set_objects (pending work)");
  if (words > c->bm_cap || !c->t.W) {
    const uint64_t alloc = words ? words : 1;
    c->bm_cap = 0;
    if (ctx_realloc(c, (void**)&c->t.W, alloc * 4) != cudaSuccess ||
        ctx_realloc(c, (void**)&c->t.L, alloc * 4) != cudaSuccess)
      return fail(c, VE_ERR_NOMEM, "ve_set_objects: bitmaps");
    c->bm_cap = alloc;
  }
  c->bm_words = words;
  // dense per-element counters: up to DENSE_PER_OBJ arrays per object with a pre
  // snapshot, allocated from one pool when a (pc, access type) first claims one
  // (k_analyze's dense_lookup); the pool holds min(2^31, DENSE_PER_OBJ * sum of the
  // objects' elements) counters (<= 8 GiB), claims beyond it take the hash path
  // (VE_DENSE_BUDGET: a smaller pool, for tests of the pool-exhausted path)
  const uint64_t DENSE_BUDGET = getenv("VE_DENSE_BUDGET") ? strtoull(getenv("VE_DENSE_BUDGET"), nullptr, 10)
                                                          : (1ull << 31);
  c->dense_pc_init.assign((size_t)DENSE_PER_OBJ * n, DENSE_OFF);
  uint64_t want = 0;
  uint64_t pre_elems = 0;
  for (uint32_t i = 0; i < n; ++i) {
    if (!v[i].pre && !v[i].post) continue;
    for (int j = 0; j < DENSE_PER_OBJ; ++j) c->dense_pc_init[DENSE_PER_OBJ * i + j] = DENSE_FREE;
    want += DENSE_PER_OBJ * v[i].n_elems;
    if (v[i].pre) pre_elems += v[i].n_elems;
  }
  c->pre_elems = pre_elems;
  if (want > DENSE_BUDGET) want = DENSE_BUDGET;
  // the pool itself is allocated by the first analysis call that may count densely (dense_reserve):
  // a ctx whose calls never carry a record per pre element (cfg5's kernels) holds no pool
  c->dense_want = want;
  // device object table (SoA, sorted by base); the block is reused when it is large
  // enough (after the device is idle: earlier launches may still read the old table)
  const size_t nn = n ? n : 1;
  const size_t nb = nn * (8 * 5 + 8 * DENSE_PER_OBJ + 4 * 2 + 4 * DENSE_PER_OBJ) + 64;
  if (nb > c->obj_block_bytes) {
    c->obj_block_bytes = 0;
    if (ctx_realloc(c, &c->obj_block, nb) != cudaSuccess) return fail(c, VE_ERR_NOMEM, "objects");
    c->obj_block_bytes = nb;
  }   // (else: the block is reused -- the ctx's work was waited for above)
  std::vector<uint8_t> host(nb, 0);
  uint64_t* hb = (uint64_t*)host.data();
  uint64_t* he = hb + n;
  uint64_t* hp = he + n;
  uint64_t* hm = hp + n;
  uint64_t* hq = hm + n;
  uint64_t* hdo = hq + n;
  uint32_t* hid = (uint32_t*)(hdo + DENSE_PER_OBJ * n);
  uint32_t* hew = hid + n;
  uint32_t* hdp = hew + n;
  c->sorted_of_id.assign(n, 0);
  for (uint32_t i = 0; i < n; ++i) {
    hb[i] = v[i].base; he[i] = v[i].base + v[i].size; hp[i] = v[i].pre; hm[i] = v[i].bmoff; hq[i] = v[i].post;
    hid[i] = v[i].id; hew[i] = v[i].ew;
    c->sorted_of_id[v[i].id] = i;
  }
  for (size_t k = 0; k < (size_t)DENSE_PER_OBJ * n; ++k) { hdo[k] = DENSE_NOT_READY; hdp[k] = c->dense_pc_init[k]; }
  cudaMemcpyAsync(c->obj_block, host.data(), nb, cudaMemcpyHostToDevice, c->cs);   // (pageable: staged before return)
  uint64_t* db = (uint64_t*)c->obj_block;
  c->o.base = db;
  c->o.end = db + n;
  c->o.pre = db + 2 * n;
  c->o.bmoff = db + 3 * n;
  c->o.post = db + 4 * n;
  c->o.dense_off = (unsigned long long*)(db + 5 * n);
  c->o.id = (const uint32_t*)(db + 5 * n + DENSE_PER_OBJ * n);
  c->o.ew = c->o.id + n;
  c->o.dense_pc = const_cast<uint32_t*>(c->o.ew + n);
  c->o.dense_pool = (uint32_t*)c->dense_pool;
  c->o.dense_cap = c->dense_pool ? std::min(c->dense_cap, c->dense_want) : 0;
  c->o.dense_next = c->t.glob + G_DENSE_NEXT;
  c->o.n = n;
  c->objs = v;
  c->n_obj = n;
  c->n_keys = c->cfg.n_pcs + n + 1;
  c->n_units = n_units;
  c->unit_obj = ustart;
  // the reset runs on the ctx stream; the analysis / diff calls wait for it on their stream
  // (no host synchronisation per object set)
  return launch_reset(c, c->cs);
}

ve_status ve_set_objects(ve_ctx* c, const ve_object* objs, uint32_t n) {
  return set_objects_units(c, objs, n, nullptr, 1u);
}

ve_status ve_set_units(ve_ctx* c, const ve_object* objs, uint32_t n, const uint32_t* unit_nobj, uint32_t n_units) {
  if (!ctx_ok(c)) return VE_ERR_INVALID;
  if (n_units == 0 || n_units > 65535 || !unit_nobj) return fail(c, VE_ERR_INVALID, "ve_set_units: 1..65535 units");
  return set_objects_units(c, objs, n, unit_nobj, n_units);
}

ve_status ve_reset(ve_ctx* c) {
  if (!ctx_ok(c)) return VE_ERR_INVALID;
  cudaSetDevice(c->device);
  // the reset is ordered after the ctx's queued work on any stream (ctx_begin in launch_reset)
  ve_status st = launch_reset(c, c->cs);
  if (st != VE_OK) return st;
  cudaError_t e = cudaStreamSynchronize(c->cs);
  return e == cudaSuccess ? VE_OK : cuda_fail(c, e, "ve_reset");
}

ve_status ve_analyze_records(ve_ctx* c, const ve_record* d, uint64_t n, cudaStream_t s) {
  if (!ctx_ok(c)) return VE_ERR_INVALID;
  if (c->poisoned || c->hist_merged) return fail(c, VE_ERR_STATE, "ve_analyze_records: ctx poisoned or merged; ve_reset first");
  if (n == 0) return VE_OK;
  if (!d || ((uintptr_t)d & 7)) return fail(c, VE_ERR_INVALID, "ve_analyze_records: d_records null or not 8-byte aligned");
  // per-CTA shared counters are 32-bit: keep each launch below 2^31 records per CTA (the
  // grid is one CTA per SM, so the cap scales with the SM count: MIG slices have few SMs)
  const uint64_t CH = (uint64_t)(c->num_sms > 0 ? c->num_sms : 1) << 31;
  for (uint64_t off = 0; off < n; off += CH) {
    ve_status st = launch_analyze(c, d + off, std::min(CH, n - off), s);
    if (st != VE_OK) return st;
  }
  return VE_OK;
}

ve_status ve_analyze_records_host(ve_ctx* c, const ve_record* h, uint64_t n, cudaStream_t s) {
  if (!ctx_ok(c)) return VE_ERR_INVALID;
  if (c->poisoned || c->hist_merged) return fail(c, VE_ERR_STATE, "ve_analyze_records_host: ctx poisoned or merged");
  if (n == 0) return VE_OK;
  if (!h) return fail(c, VE_ERR_INVALID, "ve_analyze_records_host: null records");
  const uint64_t CH = 1ull << 21;  // 2 Mi records = 48 MiB per staging buffer
  if (!c->stage[0] || !c->stage[1] || !c->stage_ev[0] || !c->stage_ev[1]) {
    // all or nothing: a partial allocation is released, so a later call retries from scratch
    bool ok = true;
    for (int i = 0; i < 2 && ok; ++i) {
      ok = cudaMalloc(&c->stage[i], CH * sizeof(ve_record)) == cudaSuccess &&
           cudaEventCreateWithFlags(&c->stage_ev[i], cudaEventDisableTiming) == cudaSuccess;
    }
    if (!ok) {
      cudaGetLastError();
      for (int i = 0; i < 2; ++i) {
        if (c->stage[i]) cudaFree(c->stage[i]);
        if (c->stage_ev[i]) cudaEventDestroy(c->stage_ev[i]);
        c->stage[i] = nullptr;
        c->stage_ev[i] = nullptr;
      }
      return fail(c, VE_ERR_NOMEM, "staging buffers");
    }
    c->stage_bytes = CH * sizeof(ve_record);
  }
  if (!c->copy_stream) {
    if (cudaStreamCreateWithFlags(&c->copy_stream, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->copied_ev[0], cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->copied_ev[1], cudaEventDisableTiming) != cudaSuccess) {
      cudaGetLastError();
      return fail(c, VE_ERR_NOMEM, "copy stream");
    }
  }
  // chunk i: the copy stream fills stage[i%2] once that buffer's previous analysis is done,
  // and stream s analyses it once the copy is done -- copy i+1 overlaps analysis i.
  // stage_ev[b] always marks the last analysis that read stage[b], on whatever stream an
  // earlier call used: the copy stream waits on it before overwriting (cross-call and
  // cross-stream safe); the first copy of this call also waits for earlier work on s.
  cudaError_t e0 = cudaStreamWaitEvent(c->copy_stream, c->stage_ev[0], 0);
  if (e0 == cudaSuccess) e0 = cudaStreamWaitEvent(c->copy_stream, c->stage_ev[1], 0);
  if (e0 == cudaSuccess) e0 = cudaEventRecord(c->copied_ev[0], s);
  if (e0 == cudaSuccess) e0 = cudaStreamWaitEvent(c->copy_stream, c->copied_ev[0], 0);
  if (e0 != cudaSuccess) return cuda_fail(c, e0, "ve_analyze_records_host order");
  for (uint64_t off = 0, i = 0; off < n; off += CH, ++i) {
    const int b = (int)(i & 1);
    const uint64_t m = std::min(CH, n - off);
    cudaError_t e = cudaStreamWaitEvent(c->copy_stream, c->stage_ev[b], 0);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(c->stage[b], h + off, m * sizeof(ve_record), cudaMemcpyHostToDevice, c->copy_stream);
    if (e == cudaSuccess) e = cudaEventRecord(c->copied_ev[b], c->copy_stream);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(s, c->copied_ev[b], 0);
    if (e != cudaSuccess) return cuda_fail(c, e, "ve_analyze_records_host copy");
    ve_status st = launch_analyze(c, (const ve_record*)c->stage[b], m, s);
    if (st != VE_OK) return st;
    cudaEventRecord(c->stage_ev[b], s);
  }
  return VE_OK;
}

ve_status ve_snapshot_diff(ve_ctx* c, uint32_t obj_id, uint32_t mode, const uint32_t* d_mask, ve_diff* h_out,
                           cudaStream_t s) {
  if (!ctx_ok(c) || !h_out) return VE_ERR_INVALID;
  if (obj_id >= c->n_obj) return fail(c, VE_ERR_INVALID, "ve_snapshot_diff: bad object id");
  return run_diff(c, c->sorted_of_id[obj_id], mode, d_mask, h_out, s);
}

ve_status ve_object_dedup(ve_ctx* c, const ve_object* objs, uint32_t n, uint32_t* h_group_of, cudaStream_t s) {
  if (!ctx_ok(c) || (n && (!objs || !h_group_of))) return VE_ERR_INVALID;
  ctx_begin(c, s);
  const ve_status st = run_dedup(c, objs, n, h_group_of, s);
  ctx_end(c, s);
  return st;
}

ve_status ve_merge_stats(ve_ctx* dst, const ve_ctx* src, void* comm, cudaStream_t s) {
  if (!ctx_ok(dst) || (!src && !comm) || (src && comm)) return VE_ERR_INVALID;
  if (dst->hist_merged) return fail(dst, VE_ERR_STATE, "ve_merge_stats: ctx already merged over ranks");
  cudaSetDevice(dst->device);
  ctx_begin(dst, s);
  if (src) ctx_begin(const_cast<ve_ctx*>(src), s);   // (waits for src's queued work; src's order is unchanged)
  const ve_status st = src ? merge_local(dst, src, s) : merge_nccl(dst, comm, s);
  ctx_end(dst, s);
  return st;
}

ve_status ve_report(ve_ctx* c, ve_rep** out) {
  if (!ctx_ok(c) || !out) return VE_ERR_INVALID;
  *out = nullptr;
  cudaSetDevice(c->device);
  cudaStream_t cs = c->cs;
  ctx_begin(c, cs);                 // after the ctx's analyses, on whatever stream they ran
  unsigned long long glob[8];
  cudaError_t e = cudaMemcpyAsync(glob, c->t.glob, sizeof(glob), cudaMemcpyDeviceToHost, cs);
  if (e == cudaSuccess) e = cudaStreamSynchronize(cs);
  if (e != cudaSuccess) return cuda_fail(c, e, "ve_report (pending work)");
  if (c->poisoned) return fail(c, VE_ERR_STATE, "ve_report: ctx poisoned by histogram overflow; ve_reset");
  if (glob[G_OVERFLOW]) {
    c->poisoned = true;
    return fail(c, VE_ERR_CAPACITY, "value histogram capacity exceeded (hist_capacity)");
  }
  if (glob[G_DENSE_NEXT] == 0) c->dense_dirty = false;   // no dense array was claimed: nothing to flush
  // counted loads contribute their value statistics and histogram entries first
  const bool tm = getenv("VE_TIMING") != nullptr;
  auto t0 = std::chrono::steady_clock::now();
  if (!c->hist_merged) {
    ve_status st = dense_flush(c, cs);
    if (st != VE_OK) return st;
    if (tm) {
      cudaStreamSynchronize(cs);
      fprintf(stderr, "[ve] dense_flush %.3f ms\n",
              std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count());
      t0 = std::chrono::steady_clock::now();
    }
  }
  const uint32_t nk = c->n_keys, K = c->cfg.topk;
  std::vector<uint64_t> sum((size_t)nk * NSUM), mn((size_t)nk * NMM), mx((size_t)nk * NMM);
  std::vector<LineState> line(nk);
  {   // the four tables through one pinned staging area, one synchronisation
    const size_t bs = sum.size() * 8, bm = mn.size() * 8, bl = nk * sizeof(LineState);
    const size_t need = bs + 2 * bm + bl;
    if (c->rpin_bytes < need) {
      if (c->rpin) cudaFreeHost(c->rpin);
      c->rpin = nullptr;
      c->rpin_bytes = 0;
      e = cudaMallocHost(&c->rpin, need);
      if (e != cudaSuccess) { c->rpin = nullptr; return cuda_fail(c, e, "ve_report staging"); }
      c->rpin_bytes = need;
    }
    uint8_t* hp = (uint8_t*)c->rpin;
    cudaMemcpyAsync(hp, c->t.sum, bs, cudaMemcpyDeviceToHost, cs);
    cudaMemcpyAsync(hp + bs, c->t.mn, bm, cudaMemcpyDeviceToHost, cs);
    cudaMemcpyAsync(hp + bs + bm, c->t.mx, bm, cudaMemcpyDeviceToHost, cs);
    cudaMemcpyAsync(hp + bs + 2 * bm, c->t.line, bl, cudaMemcpyDeviceToHost, cs);
    e = cudaStreamSynchronize(cs);
    if (e != cudaSuccess) return cuda_fail(c, e, "ve_report copy");
    memcpy(sum.data(), hp, bs);
    memcpy(mn.data(), hp + bs, bm);
    memcpy(mx.data(), hp + bs + bm, bm);
    memcpy(line.data(), hp + bs + 2 * bm, bl);
  }
  ve_rep* r = new (std::nothrow) ve_rep();
  if (!r) return VE_ERR_NOMEM;
  r->n_keys = nk;
  r->n_obj = c->n_obj;
  r->topk = K;
  std::vector<uint64_t> nd;
  ve_status st;
  if (c->hist_merged) {
    nd = c->merged_ndistinct;
    r->top = c->merged_topk;
  } else {
    st = finalize_hist(c, cs, nd, r->top);
    if (tm) {
      cudaStreamSynchronize(cs);
      fprintf(stderr, "[ve] finalize_hist %.3f ms\n",
              std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count());
    }
    if (st != VE_OK) { delete r; return st; }
  }
  st = bitmap_counts(c, cs, r->objs);
  if (st != VE_OK) { delete r; return st; }
  r->keys.assign(nk, ve_key_stats{});
  for (uint32_t k = 0; k < nk; ++k) {
    ve_key_stats& ks = r->keys[k];
    memset(&ks, 0, sizeof(ks));
    const uint64_t* sv = &sum[(size_t)k * NSUM];
    ks.n_ld = sv[F_LD]; ks.n_st = sv[F_ST]; ks.n_zero = sv[F_ZERO];
    ks.n_ld_eq_pre = sv[F_LDEQ]; ks.n_st_eq_pre = sv[F_STEQ]; ks.n_nosnap = sv[F_NOSNAP];
    for (int t = 0; t < 12; ++t) ks.n_type[t] = sv[F_TYPE0 + t];
    ks.n_nan = sv[F_NAN]; ks.n_nonint = sv[F_NONINT]; ks.n_not_f16 = sv[F_NF16];
    ks.n_not_bf16 = sv[F_NBF16]; ks.n_not_f32 = sv[F_NF32];
    ks.raw_min = mn[(size_t)k * NMM + M_RAW]; ks.ord_min = mn[(size_t)k * NMM + M_ORD];
    ks.trunc_min = mn[(size_t)k * NMM + M_TRUNC];
    ks.raw_max = mx[(size_t)k * NMM + M_RAW]; ks.ord_max = mx[(size_t)k * NMM + M_ORD];
    ks.trunc_max = mx[(size_t)k * NMM + M_TRUNC];
    const LineState& L = line[k];
    ks.line_state = L.state;
    if (L.state == VE_LINE_POINT || L.state == VE_LINE_LINE) {
      ks.p_x = L.px; ks.p_ylo = L.pylo; ks.p_yhi = L.pyhi;
      ks.q_x = L.qx; ks.q_ylo = L.qylo; ks.q_yhi = L.qyhi;
    }
    ks.n_distinct = nd[k];
    ks.n_top = std::min<uint64_t>(nd[k], K);
    derive(c->cfg, ks, &r->top[(size_t)k * K]);
  }
  for (uint32_t i = 0; i < c->n_obj; ++i) {
    ve_obj_stats& os = r->objs[i];
    const uint64_t eq = r->keys[c->cfg.n_pcs + i].n_ld_eq_pre;
    os.n_ld_reload = eq - os.n_loaded_eq;
  }
  r->glob.n_records = glob[G_RECORDS];
  r->glob.n_invalid = glob[G_INVALID];
  r->glob.n_unmapped = glob[G_UNMAPPED];
  r->glob.hist_entries = 0;
  if (!c->hist_merged) {   // occupied value-table slots after the dense flush (implementation statistic)
    r->glob.hist_entries = c->last_nocc;   // (counted by finalize_hist's occupancy compaction)
  }
  ctx_end(c, cs);
  *out = r;
  return VE_OK;
}

// approximate frequent values (C16; Def 3.3 over Def 3.8's truncation)
ve_status ve_approx_topk(ve_ctx* c, uint64_t* h_ndistinct, ve_topk_entry* h_top, cudaStream_t s) {
  if (!ctx_ok(c) || !h_ndistinct || !h_top) return VE_ERR_INVALID;
  cudaSetDevice(c->device);
  if (c->poisoned) return fail(c, VE_ERR_STATE, "ve_approx_topk: ctx poisoned by histogram overflow; ve_reset");
  if (c->hist_merged)
    return fail(c, VE_ERR_STATE, "ve_approx_topk: the histogram of a rank-merged ctx is partitioned over ranks");
  ctx_begin(c, s);
  ve_status st = dense_flush(c, s);   // counted loads -> exact histogram (idempotent)
  if (st != VE_OK) return st;
  const uint32_t nk = c->n_keys, K = c->cfg.topk;
  std::vector<uint64_t> sum((size_t)nk * NSUM);
  cudaError_t e = cudaMemcpyAsync(sum.data(), c->t.sum, sum.size() * 8, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(c, e, "ve_approx_topk");
  // keys whose records all have one float type (Q15): type codes 8 f16, 9 f32, 10 f64, 11 bf16
  std::vector<uint8_t> akind(nk, 0xFF);
  static const uint8_t code[4] = {(2u << 2) | 1u, (2u << 2) | 2u, (2u << 2) | 3u, (3u << 2) | 1u};
  for (uint32_t k = 0; k < nk; ++k) {
    int nt = 0, tc = -1;
    for (int t = 0; t < 12; ++t)
      if (sum[(size_t)k * NSUM + F_TYPE0 + t]) { ++nt; tc = t; }
    if (nt == 1 && tc >= 8) akind[k] = code[tc - 8];
  }
  std::vector<uint64_t> nd;
  std::vector<ve_topk_entry> top;
  st = approx_topk(c, s, akind, nd, top);
  if (st != VE_OK) return st;
  for (uint32_t k = 0; k < nk; ++k) h_ndistinct[k] = nd[k];
  memcpy(h_top, top.data(), (size_t)nk * K * sizeof(ve_topk_entry));
  return VE_OK;
}

void ve_report_free(ve_rep* r) { delete r; }
uint64_t ve_kernel_launches(void) { return g_launches.load(std::memory_order_relaxed); }
uint32_t ve_report_n_keys(const ve_rep* r) { return r ? r->n_keys : 0; }
uint32_t ve_report_n_objects(const ve_rep* r) { return r ? r->n_obj : 0; }
uint32_t ve_report_topk(const ve_rep* r) { return r ? r->topk : 0; }

ve_status ve_report_keys(const ve_rep* r, ve_key_stats* out) {
  if (!r || !out) return VE_ERR_INVALID;
  memcpy(out, r->keys.data(), r->keys.size() * sizeof(ve_key_stats));
  return VE_OK;
}
ve_status ve_report_topk_entries(const ve_rep* r, ve_topk_entry* out) {
  if (!r || !out) return VE_ERR_INVALID;
  memcpy(out, r->top.data(), r->top.size() * sizeof(ve_topk_entry));
  return VE_OK;
}
ve_status ve_report_objects(const ve_rep* r, ve_obj_stats* out) {
  if (!r || !out) return VE_ERR_INVALID;
  memcpy(out, r->objs.data(), r->objs.size() * sizeof(ve_obj_stats));
  return VE_OK;
}
ve_status ve_report_globals(const ve_rep* r, ve_globals* out) {
  if (!r || !out) return VE_ERR_INVALID;
  *out = r->glob;
  return VE_OK;
}

ve_status ve_report_dump(const ve_rep* r, const char* path, int format) {
  if (!r || !path || (format != 0 && format != 1)) return VE_ERR_INVALID;
  FILE* f = fopen(path, format == 0 ? "wb" : "w");
  if (!f) return VE_ERR_INVALID;
  if (format == 0) {
    const uint32_t hdr[4] = {0x50524556u /* "VERP" */, 1u, r->n_keys, r->n_obj};
    fwrite(hdr, 4, 4, f);
    fwrite(&r->topk, 4, 1, f);
    fwrite(&r->glob, sizeof(r->glob), 1, f);
    fwrite(r->keys.data(), sizeof(ve_key_stats), r->keys.size(), f);
    fwrite(r->top.data(), sizeof(ve_topk_entry), r->top.size(), f);
    fwrite(r->objs.data(), sizeof(ve_obj_stats), r->objs.size(), f);
  } else {
    static const char* tn[12] = {"u8", "u16", "u32", "u64", "i8", "i16", "i32", "i64", "f16", "f32", "f64", "bf16"};
    fprintf(f, "{\"n_records\": %llu, \"n_invalid\": %llu, \"n_unmapped\": %llu, \"keys\": [\n",
            (unsigned long long)r->glob.n_records, (unsigned long long)r->glob.n_invalid,
            (unsigned long long)r->glob.n_unmapped);
    for (uint32_t k = 0; k < r->n_keys; ++k) {
      const ve_key_stats& s = r->keys[k];
      typedef unsigned long long ull;
      fprintf(f,
              "  {\"key\": %u, \"n_ld\": %llu, \"n_st\": %llu, \"n_zero\": %llu, \"n_ld_eq_pre\": %llu, "
              "\"n_st_eq_pre\": %llu, \"n_nosnap\": %llu, \"n_distinct\": %llu, \"single_value\": %u, "
              "\"single_zero\": %u, \"frequent\": %u, \"structured\": %u, \"approx\": %u, \"dict8\": %u, "
              "\"heavy\": \"%s\", \"single_type\": %u, ",
              k, (ull)s.n_ld, (ull)s.n_st, (ull)s.n_zero, (ull)s.n_ld_eq_pre, (ull)s.n_st_eq_pre, (ull)s.n_nosnap,
              (ull)s.n_distinct, s.single_value, s.single_zero, s.frequent, s.structured, s.approx, s.dict8,
              s.heavy < 12 ? tn[s.heavy] : "none", s.single_type);
      // C5 float flags, C4 / C5 / C7 ranges, C8 line (y as signed 128-bit: hi, lo words), n_type
      fprintf(f,
              "\"n_nan\": %llu, \"n_nonint\": %llu, \"n_not_f16\": %llu, \"n_not_bf16\": %llu, \"n_not_f32\": %llu, "
              "\"raw_min\": %llu, \"raw_max\": %llu, \"ord_min\": %llu, \"ord_max\": %llu, \"trunc_min\": %llu, "
              "\"trunc_max\": %llu, \"line_state\": %llu, \"p\": [%llu, %lld, %llu], \"q\": [%llu, %lld, %llu], "
              "\"n_type\": [",
              (ull)s.n_nan, (ull)s.n_nonint, (ull)s.n_not_f16, (ull)s.n_not_bf16, (ull)s.n_not_f32, (ull)s.raw_min,
              (ull)s.raw_max, (ull)s.ord_min, (ull)s.ord_max, (ull)s.trunc_min, (ull)s.trunc_max,
              (ull)s.line_state, (ull)s.p_x, (long long)s.p_yhi, (ull)s.p_ylo, (ull)s.q_x, (long long)s.q_yhi,
              (ull)s.q_ylo);
      for (int t = 0; t < 12; ++t) fprintf(f, "%s%llu", t ? ", " : "", (ull)s.n_type[t]);
      fprintf(f, "], \"top\": [");
      for (uint64_t j = 0; j < s.n_top; ++j)
        fprintf(f, "%s[%llu, %llu]", j ? ", " : "", (unsigned long long)r->top[(size_t)k * r->topk + j].bits,
                (unsigned long long)r->top[(size_t)k * r->topk + j].count);
      fprintf(f, "]}%s\n", k + 1 < r->n_keys ? "," : "");
    }
    fprintf(f, "], \"objects\": [\n");
    for (uint32_t i = 0; i < r->n_obj; ++i) {
      const ve_obj_stats& o = r->objs[i];
      fprintf(f,
              "  {\"id\": %u, \"n_elems\": %llu, \"n_written\": %llu, \"n_loaded_eq\": %llu, \"n_ld_reload\": %llu, "
              "\"n_touched\": %llu}%s\n",
              i, (unsigned long long)o.n_elems, (unsigned long long)o.n_written, (unsigned long long)o.n_loaded_eq,
              (unsigned long long)o.n_ld_reload, (unsigned long long)o.n_touched, i + 1 < r->n_obj ? "," : "");
    }
    fprintf(f, "]}\n");
  }
  fclose(f);
  return VE_OK;
}

}  // extern "C"
