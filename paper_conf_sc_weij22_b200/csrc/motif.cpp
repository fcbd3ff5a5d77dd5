// motif.cpp -- size-k motif census (PAPER.md:25 motivates
// counting many patterns, "pattern merging [16]").
//
// stm_motif_catalog enumerates the connected graphs on k <= 6 vertices up to isomorphism
// (2, 6, 21, 112 of them for k = 3..6); stm_motif_census counts every one of them on a
// resident graph with the same counting kernel (one persistent launch per motif on the
// caller's stream; the graph, its degree-ranked copy and hub bitmaps are built once and
// shared; given graph statistics, every motif gets its cost-based order).  Counts are
// distinct subgraphs (Grochow-Kellis restrictions); with STM_VERTEX_INDUCED they are the
// induced motif frequencies, which sum to the number of connected induced k-vertex subsets.
#include <algorithm>
#include <cstring>
#include <mutex>
#include <vector>

#include "internal.h"

namespace {

constexpr int kMotifKMax = 6;

struct Motif {
  int n_edges;
  std::vector<std::pair<int, int>> edges;
  unsigned code;  // canonical edge mask (minimum over vertex permutations)
};

// edge index of (a < b) inside the upper triangle of a k x k adjacency matrix
int edge_bit(int k, int a, int b) {
  if (a > b) std::swap(a, b);
  return a * k - a * (a + 1) / 2 + (b - a - 1);
}

bool connected(int k, unsigned mask) {
  unsigned seen = 1, frontier = 1;
  while (frontier) {
    unsigned next = 0;
    for (int u = 0; u < k; ++u) {
      if (!(frontier >> u & 1)) continue;
      for (int v = 0; v < k; ++v)
        if (v != u && (mask >> edge_bit(k, u, v) & 1) && !(seen >> v & 1)) next |= 1u << v;
    }
    seen |= next;
    frontier = next;
  }
  return seen == (1u << k) - 1;
}

std::vector<Motif> build_catalog(int k) {
  const int ne = k * (k - 1) / 2;
  std::vector<std::vector<int>> perms;
  std::vector<int> p(k);
  for (int i = 0; i < k; ++i) p[i] = i;
  do perms.push_back(p); while (std::next_permutation(p.begin(), p.end()));
  // remap[perm][bit] = image of edge bit under the permutation
  std::vector<std::vector<int>> remap(perms.size(), std::vector<int>(ne));
  for (size_t q = 0; q < perms.size(); ++q)
    for (int a = 0; a < k; ++a)
      for (int b = a + 1; b < k; ++b) remap[q][edge_bit(k, a, b)] = edge_bit(k, perms[q][a], perms[q][b]);
  std::vector<unsigned> codes;
  for (unsigned mask = 1; mask < (1u << ne); ++mask) {
    if (!connected(k, mask)) continue;
    unsigned best = ~0u;
    for (size_t q = 0; q < perms.size() && best != 0; ++q) {
      unsigned img = 0;
      for (int e = 0; e < ne; ++e)
        if (mask >> e & 1) img |= 1u << remap[q][e];
      best = std::min(best, img);
    }
    if (best == mask) codes.push_back(mask);  // mask is its own canonical form
  }
  std::vector<Motif> out;
  for (unsigned c : codes) {
    Motif m{__builtin_popcount(c), {}, c};
    for (int a = 0; a < k; ++a)
      for (int b = a + 1; b < k; ++b)
        if (c >> edge_bit(k, a, b) & 1) m.edges.push_back({a, b});
    out.push_back(m);
  }
  std::stable_sort(out.begin(), out.end(), [](const Motif& x, const Motif& y) {
    return x.n_edges != y.n_edges ? x.n_edges < y.n_edges : x.code < y.code;
  });
  return out;
}

const std::vector<Motif>& catalog(int k) {
  static std::once_flag once[kMotifKMax + 1];
  static std::vector<Motif> cat[kMotifKMax + 1];
  std::call_once(once[k], [k] { cat[k] = build_catalog(k); });
  return cat[k];
}

}  // namespace

extern "C" stm_status stm_motif_catalog(int k, int capacity, int32_t* n_edges, int32_t* edges,
                                        int* n_motifs) {
  if (k < 2 || k > kMotifKMax) return stm_fail(STM_EUNSUPPORTED, "motif size k=%d outside 2..%d", k, kMotifKMax);
  if (!n_motifs) return stm_fail(STM_EINVAL, "n_motifs is NULL");
  if (capacity < 0 || (capacity > 0 && (!n_edges || !edges))) return stm_fail(STM_EINVAL, "bad output arrays");
  const auto& cat = catalog(k);
  const int stride = k * (k - 1);
  for (int i = 0; i < (int)cat.size() && i < capacity; ++i) {
    n_edges[i] = cat[i].n_edges;
    for (int e = 0; e < cat[i].n_edges; ++e) {
      edges[i * stride + 2 * e] = cat[i].edges[e].first;
      edges[i * stride + 2 * e + 1] = cat[i].edges[e].second;
    }
  }
  *n_motifs = (int)cat.size();
  return STM_OK;
}

extern "C" stm_status stm_motif_census(const stm_graph* g, int k, uint32_t flags, const stm_graph_stats* stats,
                                       const stm_tuning* t, void* stream, int capacity, uint64_t* counts,
                                       int* n_motifs) {
  if (!g) return stm_fail(STM_EINVAL, "graph is NULL");
  if (k < 2 || k > kMotifKMax) return stm_fail(STM_EUNSUPPORTED, "motif size k=%d outside 2..%d", k, kMotifKMax);
  if (!n_motifs || !counts) return stm_fail(STM_EINVAL, "NULL output");
  if (flags & ~(uint32_t)(STM_VERTEX_INDUCED | STM_NO_CODE_MOTION | STM_LAZY_UNBOUNDED | STM_AUTO_ORDER))
    return stm_fail(STM_EINVAL,
                    "census flags: only STM_VERTEX_INDUCED, STM_NO_CODE_MOTION, STM_LAZY_UNBOUNDED, STM_AUTO_ORDER");
  // cost-based orders by default: the caller's statistics, else the graph's own (computed
  // at load); STM_AUTO_ORDER keeps the compiler's greedy order
  stm_graph_stats gstats;
  if (!stats && !(flags & STM_AUTO_ORDER) && stm_graph_get_stats(g, &gstats) == STM_OK) stats = &gstats;
  flags &= ~(uint32_t)STM_AUTO_ORDER;
  const auto& cat = catalog(k);
  if (capacity < (int)cat.size())
    return stm_fail(STM_EINVAL, "capacity %d < %zu motifs of size %d", capacity, cat.size(), k);
  for (size_t i = 0; i < cat.size(); ++i) {
    std::vector<int32_t> e;
    for (auto& pr : cat[i].edges) { e.push_back(pr.first); e.push_back(pr.second); }
    int32_t order[kMotifKMax];
    stm_status s = STM_OK;
    if (stats) {  // cost-based matching order (order.cpp, NEXT-2)
      s = stm_order_optimize(k, cat[i].n_edges, e.data(), nullptr, 0, nullptr, flags | STM_AUTO_RESTRICT, stats,
                             order, nullptr, nullptr);
      if (s != STM_OK) return s;
    }
    stm_plan* P = nullptr;
    s = stm_pattern_compile(k, cat[i].n_edges, e.data(), nullptr, stats ? order : nullptr, 0, nullptr,
                            flags | STM_AUTO_RESTRICT, &P);
    if (s != STM_OK) return s;
    uint64_t c = 0;
    s = stm_match_count_ex(g, P, t, nullptr, stream, &c);
    stm_plan_free(P);
    if (s != STM_OK) return s;
    counts[i] = c;
  }
  *n_motifs = (int)cat.size();
  return STM_OK;
}
