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
#include <cstdio>
#include <cstring>
#include <map>
#include <string>
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

// ---------------------------------------------------------------------------------
// Pattern merging ("pattern merging [16]"): the per-motif plans are merged
// into a trie of matching levels (kernel.h StmMVert / StmMNode).  A level signature is
// everything the kernel reads for one level of one plan: the candidate source (a raw
// neighbour list or a set node, by its full recursive definition), the filter (label,
// bounds, exclusions) and `need`; at the last level, the counting operation.  Motifs
// with equal signatures on levels 0..d share one trie vertex at depth d -- one DFS
// frame, and every set node built on the way (by definition, deduplicated).
// ---------------------------------------------------------------------------------
namespace {

std::string node_def(const StmPlan& P, int s) {
  const StmNode& n = P.nodes[s];
  std::string a = n.a_kind == STM_SRC_RAW ? "r" + std::to_string(n.a) : "(" + node_def(P, n.a) + ")";
  char buf[96];
  snprintf(buf, sizeof buf, "L%d:%s%c%d|%u|%u|%u", n.level, a.c_str(), n.op == STM_OP_AND ? '&' : '-', n.b,
           (unsigned)n.lab, (unsigned)n.lo, (unsigned)n.hi);
  return buf;
}

std::string src_def(const StmPlan& P, StmSrc x) {
  return x.kind == STM_SRC_RAW ? "r" + std::to_string(x.idx) : "(" + node_def(P, x.idx) + ")";
}

std::string filt_def(const StmFilter& f) {
  char buf[48];
  snprintf(buf, sizeof buf, "%u/%u/%u/%u", (unsigned)f.lab, (unsigned)f.lo, (unsigned)f.hi, (unsigned)f.excl);
  return buf;
}

std::string level_sig(const StmPlan& P, int d) {
  const int k = P.k;
  if (d == 0) return "F" + filt_def(P.filt[0]);
  if (d < k - 1) return "C" + src_def(P, P.cand[d]) + "#" + filt_def(P.filt[d]) + "#" + std::to_string(P.need[d]);
  return "K" + src_def(P, P.cnt_a) + (P.cnt_op == STM_OP_NONE ? std::string("")
                                                                 : std::string(P.cnt_op == STM_OP_AND ? "&" : "-") +
                                                                       std::to_string(P.cnt_b)) +
         "#" + filt_def(P.filt[k - 1]);
}

struct TNodeH {            // host trie vertex
  int depth = 0, parent = -1;
  std::map<std::string, int> child;  // signature -> host id
  std::vector<int> motifs;           // motifs in the subtree
  int leaf_motif = -1;
};

}  // namespace

// Merge the plans of `pats` (all of size k) into one trie.  Returns STM_EUNSUPPORTED when
// a build set exceeds the kernel's per-level limit (the caller then splits the group).
static stm_status merge_plans(const std::vector<const stm_plan*>& pats, stm_merged& M) {
  const int k = pats[0]->k;
  M = stm_merged();
  M.k = k;
  M.n_patterns = (int)pats.size();
  std::vector<TNodeH> T(1);
  const std::string root_sig = level_sig(pats[0]->dev, 0);
  for (size_t i = 0; i < pats.size(); ++i) {
    const StmPlan& P = pats[i]->dev;
    if (P.k != k || level_sig(P, 0) != root_sig) return stm_fail(STM_EUNSUPPORTED, "patterns differ at the root");
    M.order_free = M.order_free && pats[i]->order_free;
    int t = 0;
    T[0].motifs.push_back((int)i);
    for (int d = 1; d < k; ++d) {
      std::string sg = level_sig(P, d);
      if (d == k - 1) sg += "#m" + std::to_string(i);  // one leaf per pattern
      auto it = T[t].child.find(sg);
      if (it == T[t].child.end()) {
        TNodeH c;
        c.depth = d;
        c.parent = t;
        T.push_back(c);
        const int id = (int)T.size() - 1;
        T[t].child[sg] = id;
        t = id;
      } else {
        t = it->second;
      }
      T[t].motifs.push_back((int)i);
    }
    T[t].leaf_motif = (int)i;
  }
  // BFS numbering: the children of every vertex are contiguous
  std::vector<int> order = {0}, newid(T.size(), -1);
  newid[0] = 0;
  for (size_t q = 0; q < order.size(); ++q)
    for (auto& kv : T[order[q]].child) {
      newid[kv.second] = (int)order.size();
      order.push_back(kv.second);
    }
  // build sets: nodes of level d+1 used by any motif under a depth-d vertex, by definition
  std::vector<std::vector<std::pair<int, std::string>>> bset(T.size());  // (stage, def)
  std::vector<std::map<std::string, int>> bset_index(T.size());
  std::vector<int> maxslots(k + 1, 0);
  for (size_t h = 0; h < T.size(); ++h) {
    const int d = T[h].depth;
    if (d > k - 2) continue;
    std::map<std::string, int> seen;  // def -> stage
    for (int i : T[h].motifs) {
      const StmPlan& P = pats[i]->dev;
      for (int s = 0; s < P.n_nodes; ++s)
        if (P.nodes[s].level == d + 1) seen[node_def(P, s)] = P.nodes[s].stage;
    }
    for (auto& kv : seen) bset[h].push_back({kv.second, kv.first});
    std::stable_sort(bset[h].begin(), bset[h].end());
    if ((int)bset[h].size() > STM_MAX_NODES)
      return stm_fail(STM_EUNSUPPORTED, "merged level needs %zu set nodes > %d", bset[h].size(), STM_MAX_NODES);
    for (size_t j = 0; j < bset[h].size(); ++j) bset_index[h][bset[h][j].second] = (int)j;
    maxslots[d + 1] = std::max(maxslots[d + 1], (int)bset[h].size());
  }
  std::vector<int> level_base(k + 1, 0);
  for (int l = 1; l <= k; ++l) level_base[l] = level_base[l - 1] + maxslots[l - 1];
  M.n_regions = level_base[k] + maxslots[k];
  // every region costs 2 x 8 ints of each warp's shared-memory stack
  if (M.n_regions > 64) return stm_fail(STM_EUNSUPPORTED, "merged plan needs %d set regions > 64", M.n_regions);
  // pool: vertices in BFS order, each vertex's build set contiguous
  std::vector<int> pool_begin(T.size(), -1);
  // ancestor of host vertex h at depth a
  auto ancestor = [&](int h, int a) {
    while (T[h].depth > a) h = T[h].parent;
    return h;
  };
  // pool index of a node definition `def` (level L) seen from host vertex h (depth >= L-1)
  auto pool_of = [&](int h, const std::string& def, int L) -> int {
    const int a = ancestor(h, L - 1);
    auto it = bset_index[a].find(def);
    if (it == bset_index[a].end() || pool_begin[a] < 0) return -1;
    return pool_begin[a] + it->second;
  };
  for (int h : order) {
    const int d = T[h].depth;
    if (d > k - 2) continue;
    pool_begin[h] = (int)M.nodes.size();
    // any motif under h that has the node gives its fields (identical by definition)
    for (size_t j = 0; j < bset[h].size(); ++j) {
      const std::string& def = bset[h][j].second;
      StmMNode mn;
      memset(&mn, 0, sizeof mn);
      bool found = false;
      for (int i : T[h].motifs) {
        const StmPlan& P = pats[i]->dev;
        for (int s = 0; s < P.n_nodes && !found; ++s) {
          if (P.nodes[s].level != d + 1 || node_def(P, s) != def) continue;
          mn.nd = P.nodes[s];
          if (mn.nd.a_kind == STM_SRC_NODE) {
            const int pa = pool_of(h, node_def(P, P.nodes[s].a), P.nodes[P.nodes[s].a].level);
            if (pa < 0) return stm_fail(STM_EUNSUPPORTED, "merge: unresolved operand");
            mn.nd.a = (int16_t)pa;
          }
          found = true;
        }
        if (found) break;
      }
      if (!found) return stm_fail(STM_EUNSUPPORTED, "merge: lost node definition");
      mn.region = (int16_t)(level_base[d + 1] + (int)j);
      M.nodes.push_back(mn);
    }
  }
  if (M.nodes.size() > 32767)
    return stm_fail(STM_EUNSUPPORTED, "merged plan needs %zu pool nodes", M.nodes.size());
  // vertices
  M.verts.resize(order.size());
  for (int h : order) {
    StmMVert v;
    memset(&v, 0, sizeof v);
    const int d = T[h].depth;
    v.depth = (int16_t)d;
    v.n_children = (int16_t)T[h].child.size();
    v.child_begin = T[h].child.empty() ? 0 : (int16_t)newid[T[h].child.begin()->second];
    v.build_begin = (int16_t)std::max(0, pool_begin[h]);
    v.n_build = (int16_t)(d <= k - 2 ? bset[h].size() : 0);
    int nst = 0;
    if (d <= k - 2)
      for (auto& x : bset[h]) nst = std::max(nst, x.first + 1);
    v.n_stages = (int8_t)nst;
    const StmPlan& P = pats[T[h].motifs[0]]->dev;  // representative: levels 0..d are shared
    v.need = (int8_t)(d >= 1 && d < k ? P.need[d] : 1);
    v.motif = -1;
    auto resolve = [&](StmSrc x) -> StmSrc {
      if (x.kind == STM_SRC_NODE) {
        const int pi = pool_of(h, node_def(P, x.idx), P.nodes[x.idx].level);
        x.idx = (int16_t)pi;
      }
      return x;
    };
    if (d == 0) {
      v.filt = P.filt[0];
    } else if (d < k - 1) {
      v.cand = resolve(P.cand[d]);
      v.filt = P.filt[d];
    } else {
      v.cand = resolve(P.cnt_a);
      v.cnt_b = P.cnt_b;
      v.cnt_op = P.cnt_op;
      v.filt = P.filt[k - 1];
      v.motif = (int16_t)T[h].leaf_motif;
    }
    if (v.cand.kind == STM_SRC_NODE && v.cand.idx < 0) return stm_fail(STM_EUNSUPPORTED, "merge: unresolved source");
    M.verts[newid[h]] = v;
  }
  return STM_OK;
}

// Count the motifs pats[idx[..]] with merged launches, splitting a group in halves when
// its merged plan exceeds the kernel's limits.
static stm_status census_merged(const stm_graph* g, const std::vector<const stm_plan*>& pats,
                                const std::vector<int>& idx, const stm_tuning* t, void* stream, uint64_t* counts,
                                int* launches) {
  std::vector<const stm_plan*> group;
  for (int i : idx) group.push_back(pats[i]);
  stm_merged M;
  stm_status s = merge_plans(group, M);
  if (s == STM_EUNSUPPORTED && idx.size() > 1) {
    std::vector<int> a(idx.begin(), idx.begin() + idx.size() / 2), b(idx.begin() + idx.size() / 2, idx.end());
    s = census_merged(g, pats, a, t, stream, counts, launches);
    if (s == STM_OK) s = census_merged(g, pats, b, t, stream, counts, launches);
    return s;
  }
  if (s != STM_OK) return s;
  std::vector<uint64_t> c(idx.size(), 0);
  s = stm_launch_merged(g, M, t, stream, c.data());
  if (s != STM_OK) return s;
  ++*launches;
  for (size_t j = 0; j < idx.size(); ++j) counts[idx[j]] = c[j];
  return STM_OK;
}

static thread_local int g_census_launches = 0;

extern "C" stm_status stm_motif_census_launches(int* launches) {
  if (!launches) return stm_fail(STM_EINVAL, "NULL argument");
  *launches = g_census_launches;
  return STM_OK;
}

extern "C" stm_status stm_motif_census(const stm_graph* g, int k, uint32_t flags, const stm_graph_stats* stats,
                                       const stm_tuning* t, void* stream, int capacity, uint64_t* counts,
                                       int* n_motifs) {
  if (!g) return stm_fail(STM_EINVAL, "graph is NULL");
  if (k < 2 || k > kMotifKMax) return stm_fail(STM_EUNSUPPORTED, "motif size k=%d outside 2..%d", k, kMotifKMax);
  if (!n_motifs || !counts) return stm_fail(STM_EINVAL, "NULL output");
  const uint32_t allowed = STM_VERTEX_INDUCED | STM_NO_CODE_MOTION | STM_LAZY_UNBOUNDED | STM_AUTO_ORDER |
                           STM_CENSUS_PER_MOTIF;
  if (flags & ~allowed)
    return stm_fail(STM_EINVAL, "census flags: only STM_VERTEX_INDUCED, STM_NO_CODE_MOTION, STM_LAZY_UNBOUNDED, "
                                "STM_AUTO_ORDER, STM_CENSUS_PER_MOTIF");
  const bool per_motif = flags & STM_CENSUS_PER_MOTIF;
  // cost-based orders by default: the caller's statistics, else the graph's own (computed
  // at load); STM_AUTO_ORDER keeps the compiler's greedy order
  stm_graph_stats gstats;
  if (!stats && !(flags & STM_AUTO_ORDER) && stm_graph_get_stats(g, &gstats) == STM_OK) stats = &gstats;
  flags &= ~(uint32_t)(STM_AUTO_ORDER | STM_CENSUS_PER_MOTIF);
  const auto& cat = catalog(k);
  if (capacity < (int)cat.size())
    return stm_fail(STM_EINVAL, "capacity %d < %zu motifs of size %d", capacity, cat.size(), k);
  std::vector<stm_plan*> plans(cat.size(), nullptr);
  auto free_all = [&] {
    for (auto* P : plans) stm_plan_free(P);
  };
  for (size_t i = 0; i < cat.size(); ++i) {
    std::vector<int32_t> e;
    for (auto& pr : cat[i].edges) { e.push_back(pr.first); e.push_back(pr.second); }
    int32_t order[kMotifKMax];
    stm_status s = STM_OK;
    if (stats) {  // cost-based matching order (order.cpp, NEXT-2)
      s = stm_order_optimize(k, cat[i].n_edges, e.data(), nullptr, 0, nullptr, flags | STM_AUTO_RESTRICT, stats,
                             order, nullptr, nullptr);
      if (s != STM_OK) { free_all(); return s; }
    }
    s = stm_pattern_compile(k, cat[i].n_edges, e.data(), nullptr, stats ? order : nullptr, 0, nullptr,
                            flags | STM_AUTO_RESTRICT, &plans[i]);
    if (s != STM_OK) { free_all(); return s; }
  }
  std::vector<uint64_t> out(cat.size(), 0);
  int launches = 0;
  stm_status s = STM_OK;
  if (per_motif || k < 3) {  // one counting launch per motif (A/B baseline; k = 2 has one motif)
    // the generic kernel unless specialised kernels are asked for explicitly (one NVRTC
    // compile per motif would dominate the census)
    stm_tuning tt;
    if (t) tt = *t;
    else stm_tuning_default(&tt);
    if (tt.jit != 1) tt.jit = -1;
    for (size_t i = 0; i < cat.size() && s == STM_OK; ++i) {
      s = stm_match_count_ex(g, plans[i], &tt, nullptr, stream, &out[i]);
      ++launches;
    }
  } else {
    std::vector<const stm_plan*> cp(plans.begin(), plans.end());
    std::vector<int> idx(cat.size());
    for (size_t i = 0; i < idx.size(); ++i) idx[i] = (int)i;
    s = census_merged(g, cp, idx, t, stream, out.data(), &launches);
  }
  free_all();
  if (s != STM_OK) return s;
  for (size_t i = 0; i < cat.size(); ++i) counts[i] = out[i];
  g_census_launches = launches;
  *n_motifs = (int)cat.size();
  return STM_OK;
}

// (debug/test) describe the merged trie of the size-k census: vertices per depth, pool
// nodes, regions -- "depth0 depth1 ... | nodes | regions"
extern "C" stm_status stm_motif_merge_stats(int k, uint32_t flags, int* verts_per_depth, int* n_nodes,
                                            int* n_regions) {
  if (k < 3 || k > kMotifKMax || !verts_per_depth || !n_nodes || !n_regions)
    return stm_fail(STM_EINVAL, "bad arguments");
  const auto& cat = catalog(k);
  std::vector<stm_plan*> plans;
  for (size_t i = 0; i < cat.size(); ++i) {
    std::vector<int32_t> e;
    for (auto& pr : cat[i].edges) { e.push_back(pr.first); e.push_back(pr.second); }
    stm_plan* P = nullptr;
    stm_status s = stm_pattern_compile(k, cat[i].n_edges, e.data(), nullptr, nullptr, 0, nullptr,
                                       (flags & STM_VERTEX_INDUCED) | STM_AUTO_RESTRICT, &P);
    if (s != STM_OK) {
      for (auto* q : plans) stm_plan_free(q);
      return s;
    }
    plans.push_back(P);
  }
  stm_merged M;
  std::vector<const stm_plan*> cp(plans.begin(), plans.end());
  stm_status s = merge_plans(cp, M);
  for (auto* q : plans) stm_plan_free(q);
  if (s != STM_OK) return s;
  for (int d = 0; d < k; ++d) verts_per_depth[d] = 0;
  for (auto& v : M.verts) verts_per_depth[v.depth]++;
  *n_nodes = (int)M.nodes.size();
  *n_regions = M.n_regions;
  return STM_OK;
}
