// vfg.cu -- SURVEY 8(f) f4: the value flow graph and its two subgraphs (PAPER.md
// section 5.2, Defs 5.1-5.3).  Host-side bookkeeping over an
// API-event log: one pass in program order with a "last writer" table per data
// object builds every edge e_{i,j,k} (v_i the last writer of D_k before v_j's
// access); invocations of one vertex id (one call path) merge.  No
// device work: the graph has one edge per (writer, accessor, object) and is
// orders of magnitude smaller than the value trace.  Readings R7-R9: DESIGN.md 3.
#include <algorithm>
#include <map>
#include <new>
#include <set>
#include <tuple>
#include <unordered_map>
#include <vector>

#include "ve_internal.cuh"

struct ve_vfg {
  std::vector<ve_vfg_vertex> v;   // sorted by id
  std::vector<ve_vfg_edge> e;     // sorted by (src, dst, object)
};

namespace {

using EdgeKey = std::tuple<uint32_t, uint32_t, uint32_t>;

struct EdgeAcc {
  uint32_t label = 0;
  uint64_t bytes = 0, count = 0, last_seq = ~0ull;
};

void add_edge(std::map<EdgeKey, EdgeAcc>& E, uint32_t src, uint32_t dst, uint32_t obj, uint32_t label, uint64_t bytes,
              uint64_t seq) {
  EdgeAcc& a = E[EdgeKey{src, dst, obj}];
  a.label |= label;
  a.bytes += bytes;
  if (a.last_seq != seq) {   // one count per invocation
    ++a.count;
    a.last_seq = seq;
  }
}

ve_vfg* make(const std::map<EdgeKey, EdgeAcc>& E, const std::map<uint32_t, uint64_t>& inv) {
  ve_vfg* g = new (std::nothrow) ve_vfg();
  if (!g) return nullptr;
  for (const auto& kv : inv) g->v.push_back(ve_vfg_vertex{kv.first, 0, kv.second});
  for (const auto& kv : E)
    g->e.push_back(ve_vfg_edge{std::get<0>(kv.first), std::get<1>(kv.first), std::get<2>(kv.first), kv.second.label,
                               kv.second.bytes, kv.second.count});
  return g;
}

uint64_t invocations_of(const ve_vfg* g, uint32_t v) {
  auto it = std::lower_bound(g->v.begin(), g->v.end(), v,
                             [](const ve_vfg_vertex& a, uint32_t x) { return a.vertex < x; });
  return (it != g->v.end() && it->vertex == v) ? it->invocations : 0;
}

}  // namespace

extern "C" {

ve_status ve_vfg_build(const ve_api_access* log, uint64_t n, ve_vfg** out) {
  if (!out || (n && !log)) return VE_ERR_INVALID;
  *out = nullptr;
  std::unordered_map<uint32_t, uint32_t> writer;          // D_k -> its last writer
  std::map<EdgeKey, EdgeAcc> E;
  std::map<uint32_t, uint64_t> inv;                       // vertex -> invocations
  std::vector<std::pair<uint32_t, uint32_t>> pending;     // (object, writer) of the current invocation
  uint64_t i = 0;
  while (i < n) {
    const uint64_t seq = log[i].seq;
    uint64_t j = i;
    while (j < n && log[j].seq == seq) ++j;
    if (j < n && log[j].seq < seq) return VE_ERR_INVALID;  // program order
    pending.clear();
    std::set<uint32_t> seen_v;
    for (uint64_t k = i; k < j; ++k) {
      const ve_api_access& a = log[k];
      if (a.vertex == VE_HOST_VERTEX || a.object == 0xFFFFFFFFu || a.kind > VE_EV_D2H) return VE_ERR_INVALID;
      if (seen_v.insert(a.vertex).second) inv[a.vertex]++;
      if (a.kind == VE_EV_ALLOC) {                         // the allocation: D_k's first writer
        pending.push_back({a.object, a.vertex});
        continue;
      }
      auto w = writer.find(a.object);
      if (w == writer.end()) return VE_ERR_INVALID;        // accessed before its allocation
      uint32_t mode = a.mode & (VE_ACC_READ | VE_ACC_WRITE);
      if (a.kind == VE_EV_H2D) mode = VE_ACC_WRITE;
      if (a.kind == VE_EV_D2H) mode = VE_ACC_READ;
      if (!mode) return VE_ERR_INVALID;
      add_edge(E, w->second, a.vertex, a.object, mode, a.bytes, seq);
      if (a.kind == VE_EV_H2D) add_edge(E, VE_HOST_VERTEX, a.vertex, a.object, VE_ACC_WRITE, a.bytes, seq);
      if (a.kind == VE_EV_D2H) add_edge(E, a.vertex, VE_HOST_VERTEX, a.object, VE_ACC_READ, a.bytes, seq);
      if (mode & VE_ACC_WRITE) pending.push_back({a.object, a.vertex});
    }
    for (const auto& p : pending) writer[p.first] = p.second;   // writes take effect after the invocation
    i = j;
  }
  ve_vfg* g = make(E, inv);
  if (!g) return VE_ERR_NOMEM;
  *out = g;
  return VE_OK;
}

ve_status ve_vfg_slice(const ve_vfg* g, uint32_t v, ve_vfg** out) {
  if (!g || !out) return VE_ERR_INVALID;
  *out = nullptr;
  if (!invocations_of(g, v)) return VE_ERR_INVALID;
  // objects v reads or writes: edges into v (its accesses) or out of v (it was a writer)
  std::set<uint32_t> objs;
  for (const auto& e : g->e)
    if (e.dst == v || e.src == v) objs.insert(e.object);
  std::map<EdgeKey, EdgeAcc> E;
  std::map<uint32_t, uint64_t> inv;
  for (uint32_t k : objs) {
    std::vector<const ve_vfg_edge*> ek;
    for (const auto& e : g->e)
      if (e.object == k) ek.push_back(&e);
    // vertices reaching v / reached from v over D_k's edges (BFS both ways)
    std::set<uint32_t> to_v{v}, from_v{v};
    std::vector<uint32_t> st{v};
    while (!st.empty()) {
      const uint32_t x = st.back();
      st.pop_back();
      for (const auto* e : ek)
        if (e->dst == x && to_v.insert(e->src).second) st.push_back(e->src);
    }
    st.assign(1, v);
    while (!st.empty()) {
      const uint32_t x = st.back();
      st.pop_back();
      for (const auto* e : ek)
        if (e->src == x && from_v.insert(e->dst).second) st.push_back(e->dst);
    }
    for (const auto* e : ek) {
      if (!to_v.count(e->dst) && !from_v.count(e->src)) continue;
      EdgeAcc& a = E[EdgeKey{e->src, e->dst, e->object}];
      a.label = e->label;
      a.bytes = e->bytes;
      a.count = e->count;
      for (uint32_t x : {e->src, e->dst})
        if (x != VE_HOST_VERTEX) inv[x] = invocations_of(g, x);
    }
  }
  ve_vfg* r = make(E, inv);
  if (!r) return VE_ERR_NOMEM;
  *out = r;
  return VE_OK;
}

ve_status ve_vfg_important(const ve_vfg* g, uint64_t min_edge_bytes, uint64_t min_vertex_invocations,
                           ve_vfg** out) {
  if (!g || !out) return VE_ERR_INVALID;
  ve_vfg* r = new (std::nothrow) ve_vfg();
  if (!r) return VE_ERR_NOMEM;
  std::set<uint32_t> keep;
  for (const auto& e : g->e)
    if (e.bytes >= min_edge_bytes) {
      r->e.push_back(e);
      if (e.src != VE_HOST_VERTEX) keep.insert(e.src);
      if (e.dst != VE_HOST_VERTEX) keep.insert(e.dst);
    }
  for (const auto& v : g->v)
    if (keep.count(v.vertex) || v.invocations >= min_vertex_invocations) r->v.push_back(v);
  *out = r;
  return VE_OK;
}

ve_status ve_vfg_size(const ve_vfg* g, uint64_t* nv, uint64_t* ne) {
  if (!g || !nv || !ne) return VE_ERR_INVALID;
  *nv = g->v.size();
  *ne = g->e.size();
  return VE_OK;
}

ve_status ve_vfg_vertices(const ve_vfg* g, ve_vfg_vertex* out) {
  if (!g || (!out && !g->v.empty())) return VE_ERR_INVALID;
  std::copy(g->v.begin(), g->v.end(), out);
  return VE_OK;
}

ve_status ve_vfg_edges(const ve_vfg* g, ve_vfg_edge* out) {
  if (!g || (!out && !g->e.empty())) return VE_ERR_INVALID;
  std::copy(g->e.begin(), g->e.end(), out);
  return VE_OK;
}

void ve_vfg_free(ve_vfg* g) { delete g; }

}  // extern "C"
