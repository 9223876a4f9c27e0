// plan.cpp — layout propagation over an operator DAG: Algorithm 1
// (§4.2) run for every tuned tensor in topological (edge) order,
// plus the multi-producer rule of §6, settled in topological
// order (reading A31).
//
// Deviation that is this library's point: where Alg. 1 line 4
// inserts a conversion op (complex -> complex edge), the producer's fused
// epilogue writes the consumer's layout instead, so the conversion is
// recorded (conversion[e] = 1) but never launched as a separate kernel.
#include <algorithm>
#include <deque>
#include <vector>

#include "alt.h"
#include "layout.h"

namespace alt {

// Reading A9: pad(0,0), unfold with B == D (one tile) or B == S dividing D
// are trivial; any other pad / unfold is a non-trivial advanced primitive.
static bool nontrivial_advanced(const Layout &L) {
  for (int s = 0; s < L.np; s++) {
    const alt_prim &p = L.prims[s];
    const int64_t D = L.desc.shp[s][p.dim];
    if (p.kind == ALT_PAD && (p.v[0] != 0 || p.v[1] != 0)) return true;
    if (p.kind == ALT_UNFOLD) {
      const int64_t B = p.v[0], S = p.v[1];
      if (B == D) continue;
      if (B == S && D % S == 0) continue;
      return true;
    }
  }
  return false;
}

}  // namespace alt

using namespace alt;

extern "C" alt_status alt_plan_chain(int32_t n_ops, const int32_t *op_kind, int32_t n_edges,
                                     const int32_t *edge_src, const int32_t *edge_dst,
                                     const int32_t *edge_in_idx, const int64_t *edge_numel,
                                     const alt_layout *edge_layout, int32_t *src_edge,
                                     int32_t *conversion) {
  if (n_ops < 0 || n_edges < 0 || (n_ops && !op_kind) ||
      (n_edges && (!edge_src || !edge_dst || !edge_in_idx || !edge_numel || !edge_layout ||
                   !src_edge || !conversion))) {
    set_error("alt_plan_chain: NULL argument");
    return ALT_E_INVALID;
  }
  for (int e = 0; e < n_edges; e++) {
    if (edge_src[e] < -1 || edge_src[e] >= n_ops || edge_dst[e] < -1 || edge_dst[e] >= n_ops) {
      set_error("alt_plan_chain: edge %d references a bad op", e);
      return ALT_E_INVALID;
    }
    src_edge[e] = -1;
    conversion[e] = 0;
  }
  for (int o = 0; o < n_ops; o++)
    if (op_kind[o] < 0 || op_kind[o] > 2) { set_error("alt_plan_chain: bad op kind"); return ALT_E_INVALID; }
  enum { COMPLEX = 0, ELEMWISE = 1 };
  // 1. Alg. 1 for every tuned tensor (edge order): reach[T] = the edges its
  //    layout propagates to (lines 6-12), or a recorded conversion (lines 3-5)
  std::vector<int> tuned;
  for (int e = 0; e < n_edges; e++) if (edge_layout[e]) tuned.push_back(e);
  std::vector<std::vector<char>> reach(tuned.size(), std::vector<char>(n_edges, 0));
  for (size_t k = 0; k < tuned.size(); k++) {
    const int eT = tuned[k];
    const Layout &L = edge_layout[eT]->impl;
    const int o2 = edge_dst[eT];
    reach[k][eT] = 1;  // line 2: P <- {p_T}
    const bool empty = (L.flags & ALT_IDENTITY) != 0;
    if (empty || nontrivial_advanced(L) || (o2 >= 0 && op_kind[o2] == COMPLEX)) {  // lines 3-5
      if (!empty && o2 >= 0) conversion[eT] = 1;  // A21: identity conversion elided
      continue;
    }
    std::deque<int> Q{eT};  // lines 6-12
    while (!Q.empty()) {
      const int s = Q.front();
      Q.pop_front();
      const int so2 = edge_dst[s];
      if (so2 < 0 || op_kind[so2] != ELEMWISE) continue;
      for (int t = 0; t < n_edges; t++) {
        if (edge_src[t] != so2 || reach[k][t]) continue;
        const int o3 = edge_dst[t];
        if (edge_numel[t] != edge_numel[s]) continue;     // shape check (line 10)
        if (o3 >= 0 && op_kind[o3] == COMPLEX) continue;  // o3 converts itself
        reach[k][t] = 1;                                  // line 11
        Q.push_back(t);                                   // line 12
      }
    }
  }
  // 2. multi-producer rule (X0; reading A31): in topological
  //    order, an edge reached by several tuned layouts takes the one its
  //    elementwise producer receives through the lowest input slot, judged by
  //    the layout that input finally carries (inputs are settled first)
  std::vector<int> indeg(n_ops, 0), rank(n_ops, 0);
  for (int e = 0; e < n_edges; e++)
    if (edge_src[e] >= 0 && edge_dst[e] >= 0) indeg[edge_dst[e]]++;
  {
    std::deque<int> ready;
    for (int o = 0; o < n_ops; o++) if (!indeg[o]) ready.push_back(o);
    int r = 0;
    while (!ready.empty()) {
      const int o = ready.front();
      ready.pop_front();
      rank[o] = r++;
      for (int e = 0; e < n_edges; e++)
        if (edge_src[e] == o && edge_dst[e] >= 0 && --indeg[edge_dst[e]] == 0) ready.push_back(edge_dst[e]);
    }
  }
  std::vector<int> order(n_edges);
  for (int e = 0; e < n_edges; e++) order[e] = e;
  std::stable_sort(order.begin(), order.end(), [&](int a, int b) {
    const int ra = edge_src[a] < 0 ? -1 : rank[edge_src[a]], rb = edge_src[b] < 0 ? -1 : rank[edge_src[b]];
    return ra < rb;
  });
  for (int e : order) {
    if (edge_layout[e]) { src_edge[e] = e; continue; }  // a tuned tensor keeps its own layout
    bool any = false;
    for (size_t k = 0; k < tuned.size() && !any; k++) any = reach[k][e] != 0;
    if (!any) continue;
    const int producer = edge_src[e];
    int best_slot = 1 << 30;
    for (int i = 0; i < n_edges; i++) {
      if (edge_dst[i] != producer || producer < 0 || src_edge[i] < 0 || edge_in_idx[i] >= best_slot) continue;
      // the layout input i carries must itself reach e
      size_t k = 0;
      while (k < tuned.size() && tuned[k] != src_edge[i]) k++;
      if (k == tuned.size() || !reach[k][e]) continue;
      best_slot = edge_in_idx[i];
      src_edge[e] = src_edge[i];
    }
  }
  return ALT_OK;
}
