// order.cpp -- cost-based matching-order optimiser (host only, product code).
//
// SURVEY.md 8(f) NEXT-2.  The paper adopts Dryadic's matching order and
// only requires that pi[l+1] be adjacent to some of pi[0..l].  The order
// changes the work, never the count, so this module only chooses the `order` argument
// of stm_pattern_compile.  Cost model (reading R15):
//
//   * data graph = Chung-Lu random graph with the observed expected degrees
//     w(v) = min(d(v), sqrt(2m)), P(x ~ y) = w(x) w(y) / 2m;
//   * the expected number of homomorphisms of a pattern subgraph H = (S, E_S) is then
//     exactly  prod_{u in S} (n M_{deg_H(u)}) / (2m)^{|E_S|},  M_j = (1/n) sum_v w(v)^j,
//     times prod_u freq(label(u)) (labels independent of degree) and times the fraction
//     ext(S) / |S|! of value orders that satisfy the restrictions among S (ext = number
//     of linear extensions of the restriction partial order restricted to S);
//   * extending one level-l prefix costs the summed expected neighbour-list lengths of
//     the set operands: the backward neighbours b of pi[l] (and, vertex-induced, the
//     backward non-neighbours), E[w(f(b))] = M_{j+1} / M_j with j = deg_{H_l}(b) --
//     except with a single operand, where the candidates are a bounded view of one row
//     (cost 1 + log2(1 + E[w])); inner-level candidates are then visited one by one;
//   * cost(pi) = n + sum_{l=1}^{k-1} N(S_l) * work_l + sum_{l=2}^{k-1} N(S_l).
//
// The search is exhaustive over connected orders (k <= 8: at most 8! = 40320), and the
// compiler's greedy order is kept unless the best order is predicted at least
// kMinGain cheaper (so cliques compile exactly as before, and near-ties -- which the
// model cannot rank, e.g. rotations of a labeled cycle that differ only by label
// frequencies -- do not move the order; trees keep it too; DESIGN.md 8b2 has the
// measurements).
#include <algorithm>
#include <cmath>
#include <cstring>
#include <map>
#include <vector>

#include "internal.h"

namespace {

constexpr double kMinGain = 0.10;  // leave the greedy order only for a >= 10% predicted saving

struct Model {
  int k = 0;
  int n_edges = 0;
  int adj[STM_KMAX][STM_KMAX] = {};
  double lab_factor[STM_KMAX] = {};
  double ext[1 << STM_KMAX] = {};  // linear extensions of the restriction order on each subset
  bool vi = false;
  double n = 0, nnz = 0;
  double M[STM_STATS_MOMENTS] = {};
};

// Evaluates cost(pi) and the estimated count N(S_k); false if pi is not a connected order.
bool eval(const Model& m, const int* pi, double* cost, double* est) {
  const int k = m.k;
  double c = m.n;  // level 0: the root loop touches every vertex once
  unsigned S = 0;
  int degH[STM_KMAX] = {};  // degree of each placed pattern vertex inside H_l
  int edgesH = 0;
  double N = 0;
  bool visit_next = false;
  auto count_of = [&](unsigned set) {  // N(S) from the closed form above
    if (m.nnz <= 0) return 0.0;
    double v = 1.0;
    for (int u = 0; u < k; ++u)
      if (set >> u & 1) v *= m.n * m.M[degH[u]] * m.lab_factor[u];
    v /= std::pow(m.nnz, edgesH);
    int sz = __builtin_popcount(set);
    double fact = 1;
    for (int i = 2; i <= sz; ++i) fact *= i;
    return v * m.ext[set] / fact;
  };
  for (int l = 0; l < k; ++l) {
    const int u = pi[l];
    if (u < 0 || u >= k || (S >> u & 1)) return false;
    if (l > 0) {
      bool con = false;
      double work = 0;
      int ops = 0;
      for (int b = 0; b < k; ++b) {
        if (!(S >> b & 1)) continue;
        const bool nb = m.adj[u][b];
        con |= nb;
        if (nb || m.vi) {
          work += m.M[degH[b]] > 0 ? m.M[degH[b] + 1] / m.M[degH[b]] : 0;
          ++ops;
        }
      }
      if (!con) return false;
      // One operand: the candidates are a bounded view of one row (no set operation),
      // a binary search for the bounds; at the last level its size is the count.
      if (ops == 1) work = 1 + std::log2(1 + work);
      c += N * work;
      visit_next = l < k - 1;  // candidates of inner levels are iterated one by one
      for (int b = 0; b < k; ++b)
        if ((S >> b & 1) && m.adj[u][b]) { ++degH[b]; ++degH[u]; ++edgesH; }
    }
    S |= 1u << u;
    N = count_of(S);
    if (visit_next) c += N;
  }
  *cost = c;
  *est = N;
  return true;
}

stm_status build_model(int k, int n_edges, const int32_t* edges, const int32_t* labels, int n_restr,
                       const int32_t* restr, uint32_t flags, const stm_graph_stats* s, Model* m,
                       std::vector<int>* greedy) {
  if (flags & STM_DIRECTED)
    return stm_fail(STM_EUNSUPPORTED, "cost-based orders model undirected patterns only (directed: greedy order)");
  if (!s) return stm_fail(STM_EINVAL, "stats is NULL");
  if (s->n < 0 || s->nnz < 0) return stm_fail(STM_EINVAL, "stats: negative n or nnz");
  if (s->n_labels < 0 || s->n_labels > STM_STATS_LABELS) return stm_fail(STM_EINVAL, "stats: bad n_labels");
  // Compiling validates the pattern and yields the restriction set (given or Grochow-Kellis)
  // and the greedy order the optimiser must beat.
  stm_plan* P = nullptr;
  stm_status st = stm_pattern_compile(k, n_edges, edges, labels, nullptr, n_restr, restr,
                                      flags | STM_AUTO_ORDER, &P);
  if (st != STM_OK) return st;
  m->k = k;
  m->vi = flags & STM_VERTEX_INDUCED;
  m->n = (double)s->n;
  m->nnz = (double)s->nnz;
  for (int j = 0; j < STM_STATS_MOMENTS; ++j) m->M[j] = s->moment[j];
  for (auto& e : P->edges) m->adj[e.first][e.second] = m->adj[e.second][e.first] = 1;
  m->n_edges = (int)P->edges.size();
  for (int u = 0; u < k; ++u) {
    m->lab_factor[u] = 1.0;
    if (!P->labels.empty() && P->labels[u] >= 0 && s->n_labels > 0) {
      double f = 0;
      for (int i = 0; i < s->n_labels; ++i)
        if (s->label_value[i] == P->labels[u]) f = s->label_freq[i];
      m->lab_factor[u] = f;
    }
  }
  int less[STM_KMAX][STM_KMAX] = {};
  for (auto& r : P->restr) less[r.first][r.second] = 1;
  for (int x = 0; x < k; ++x)
    for (int i = 0; i < k; ++i)
      for (int j = 0; j < k; ++j)
        if (less[i][x] && less[x][j]) less[i][j] = 1;
  // ext[S] by the subset recursion: the last element of an extension of S is a
  // maximal element of S (nothing in S above it).
  m->ext[0] = 1;
  for (unsigned S = 1; S < (1u << k); ++S) {
    double e = 0;
    for (int u = 0; u < k; ++u) {
      if (!(S >> u & 1)) continue;
      bool maximal = true;
      for (int w = 0; w < k && maximal; ++w)
        if ((S >> w & 1) && less[u][w]) maximal = false;
      if (maximal) e += m->ext[S & ~(1u << u)];
    }
    m->ext[S] = e;
  }
  greedy->assign(P->dev.order, P->dev.order + k);
  stm_plan_free(P);
  return STM_OK;
}

}  // namespace

extern "C" stm_status stm_graph_stats_host(int64_t n, const int64_t* row_ptr, const int32_t* labels,
                                           stm_graph_stats* out) {
  if (!out) return stm_fail(STM_EINVAL, "out is NULL");
  if (n < 0 || (n > 0 && !row_ptr)) return stm_fail(STM_EINVAL, "bad n / row_ptr");
  memset(out, 0, sizeof *out);
  out->n = n;
  out->nnz = n > 0 ? row_ptr[n] - row_ptr[0] : 0;
  if (n == 0) return STM_OK;
  const double cap = std::sqrt((double)out->nnz);
  double acc[STM_STATS_MOMENTS] = {};
  for (int64_t v = 0; v < n; ++v) {
    const int64_t d = row_ptr[v + 1] - row_ptr[v];
    if (d < 0) return stm_fail(STM_EINVAL, "row_ptr decreases at %lld", (long long)v);
    const double w = std::min((double)d, cap);
    double p = 1;
    for (int j = 0; j < STM_STATS_MOMENTS; ++j) { acc[j] += p; p *= w; }
  }
  for (int j = 0; j < STM_STATS_MOMENTS; ++j) out->moment[j] = acc[j] / (double)n;
  if (labels) {
    std::map<int32_t, int64_t> freq;
    for (int64_t v = 0; v < n; ++v) {
      if (labels[v] < 0) return stm_fail(STM_EINVAL, "negative vertex label at %lld", (long long)v);
      ++freq[labels[v]];
    }
    if (freq.size() > STM_STATS_LABELS)
      return stm_fail(STM_EUNSUPPORTED, "%zu distinct labels > %d", freq.size(), (int)STM_STATS_LABELS);
    for (auto& kv : freq) {
      out->label_value[out->n_labels] = kv.first;
      out->label_freq[out->n_labels] = (double)kv.second / (double)n;
      ++out->n_labels;
    }
  }
  return STM_OK;
}

extern "C" stm_status stm_order_cost(int k, int n_edges, const int32_t* edges, const int32_t* labels,
                                     int n_restr, const int32_t* restr, uint32_t flags,
                                     const stm_graph_stats* stats, const int32_t* order, double* cost,
                                     double* est_count) {
  if (!order) return stm_fail(STM_EINVAL, "order is NULL");
  Model m;
  std::vector<int> greedy;
  stm_status st = build_model(k, n_edges, edges, labels, n_restr, restr, flags, stats, &m, &greedy);
  if (st != STM_OK) return st;
  double c, e;
  if (!eval(m, order, &c, &e))
    return stm_fail(STM_EINVAL, "order is not a connected permutation (PAPER.md:52)");
  if (cost) *cost = c;
  if (est_count) *est_count = e;
  return STM_OK;
}

extern "C" stm_status stm_order_optimize(int k, int n_edges, const int32_t* edges, const int32_t* labels,
                                         int n_restr, const int32_t* restr, uint32_t flags,
                                         const stm_graph_stats* stats, int32_t* order_out, double* cost,
                                         double* est_count) {
  if (!order_out) return stm_fail(STM_EINVAL, "order_out is NULL");
  Model m;
  std::vector<int> greedy;
  stm_status st = build_model(k, n_edges, edges, labels, n_restr, restr, flags, stats, &m, &greedy);
  if (st != STM_OK) return st;
  std::vector<int> best = greedy;
  double greedy_c, greedy_e;
  eval(m, greedy.data(), &greedy_c, &greedy_e);
  double best_c = greedy_c, best_e = greedy_e;
  std::vector<int> p(k);
  for (int i = 0; i < k; ++i) p[i] = i;
  do {
    double c, e;
    if (!eval(m, p.data(), &c, &e)) continue;
    if (c < best_c * (1 - 1e-9)) { best = p; best_c = c; best_e = e; }
  } while (std::next_permutation(p.begin(), p.end()));
  // Trees: every order has exactly one operand per level, so the model can only rank
  // where the restriction bounds land, and it ranked that wrong on every tree motif
  // measured (C1, k = 5/6 vertex-induced: 1.2x-8.3x slower, profiles/r01_census_permotif.log).
  const bool tree = m.n_edges == k - 1;
  if (tree || best_c > greedy_c * (1 - kMinGain)) { best = greedy; best_c = greedy_c; best_e = greedy_e; }
  for (int i = 0; i < k; ++i) order_out[i] = best[i];
  if (cost) *cost = best_c;
  if (est_count) *est_count = best_e;
  return STM_OK;
}
