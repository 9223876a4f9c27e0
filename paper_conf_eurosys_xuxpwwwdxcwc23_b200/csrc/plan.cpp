// plan.cpp — layout propagation over an operator DAG: Algorithm 1
// (§4.2) run for every tuned tensor in topological (edge) order,
// plus the multi-producer rule of §6.
//
// Deviation that is this library's point: where Alg. 1 line 4
// inserts a conversion op (complex -> complex edge), the producer's fused
// epilogue writes the consumer's layout instead, so the conversion is
// recorded (conversion[e] = 1) but never launched as a separate kernel.
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
  // slot through which the propagated layout entered the producer of e
  std::vector<int32_t> entry_slot(n_edges, 1 << 30);
  for (int eT = 0; eT < n_edges; eT++) {
    if (!edge_layout[eT]) continue;
    const Layout &L = edge_layout[eT]->impl;
    const int o2 = edge_dst[eT];
    // line 2: P <- {p_T}
    if (src_edge[eT] < 0 || entry_slot[eT] > 0) { src_edge[eT] = eT; entry_slot[eT] = -1; }
    const bool empty = (L.flags & ALT_IDENTITY) != 0;
    // line 3-5
    if (empty || nontrivial_advanced(L) || (o2 >= 0 && op_kind[o2] == COMPLEX)) {
      if (!empty && o2 >= 0) conversion[eT] = 1;  // A21: identity conversion elided
      continue;
    }
    // line 6-12
    std::deque<int> Q{eT};
    while (!Q.empty()) {
      const int s = Q.front();
      Q.pop_front();
      const int so2 = edge_dst[s];
      if (so2 < 0 || op_kind[so2] != ELEMWISE) continue;
      for (int t = 0; t < n_edges; t++) {
        if (edge_src[t] != so2) continue;
        const int o3 = edge_dst[t];
        if (edge_numel[t] != edge_numel[s]) continue;        // shape check (line 10)
        if (o3 >= 0 && op_kind[o3] == COMPLEX) continue;     // o3 converts itself
        // multi-producer rule: the layout entering through the lowest input
        // slot of the elementwise op wins (X0)
        const int32_t slot = edge_in_idx[s];
        if (src_edge[t] >= 0 && entry_slot[t] <= slot) continue;
        src_edge[t] = src_edge[s] >= 0 ? src_edge[s] : eT;   // line 11
        entry_slot[t] = slot;
        Q.push_back(t);                                      // line 12
      }
    }
  }
  return ALT_OK;
}
