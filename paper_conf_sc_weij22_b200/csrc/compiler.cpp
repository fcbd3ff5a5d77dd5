// compiler.cpp -- host-side pattern compiler (stm_pattern_compile & friends).
//
// Emits, for the persistent kernel, everything that depends on the pattern only:
//   * the matching order pi (pi[l+1] adjacent to some of pi[0..l];
//     the paper adopts Dryadic's order, PAPER.md:151 -- we use a greedy order,
//     DESIGN.md reading R6),
//   * symmetry-breaking restrictions (north_star; not in the paper): the label-
//     preserving automorphism group by brute force and the Grochow-Kellis
//     stabiliser chain, plus their transitive closure as per-level value bounds,
//   * the loop-invariant code-motion plan (Sec. VII): every
//     candidate set is an operation chain over raw neighbour lists; chains are
//     merged on common prefixes (a trie over the per-level signature), and each
//     prefix is computed at the shallowest level where its operands are known,
//   * merged multi-label sets: a shared set keeps the union of
//     its consumers' labels; bounds are applied only where every consumer shares
//     them,
//   * vertex-induced set differences or their removal for
//     edge-induced matching.
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <map>
#include <new>
#include <string>
#include <vector>

#include "internal.h"

namespace {

struct Chain {
  int f = -1;                        // first pattern-neighbour position (start operand N(v_f))
  std::vector<std::pair<int, int>> ops;  // (opcode, position j)
  std::vector<int> level;            // level of each op
};

bool next_perm(std::vector<int>& p) { return std::next_permutation(p.begin(), p.end()); }

}  // namespace

static std::string fmt_mask(unsigned m) {
  std::string s = "{";
  bool first = true;
  for (int j = 0; j < 8; ++j)
    if (m & (1u << j)) {
      if (!first) s += ",";
      s += "v" + std::to_string(j);
      first = false;
    }
  return s + "}";
}

static void build_describe(stm_plan* P) {
  const StmPlan& D = P->dev;
  std::string s;
  char buf[256];
  snprintf(buf, sizeof buf, "k=%d mode=%s%s code_motion=%s count_mode=%s aut=%lld\n", D.k,
           D.vertex_induced ? "vertex" : "edge", D.directed ? " directed" : "",
           (P->flags & STM_NO_CODE_MOTION) ? "off" : "on",
           D.count_mode == STM_COUNT_FUSED ? "fused" : "frame", (long long)P->aut);
  s += buf;
  s += "order=[";
  for (int l = 0; l < D.k; ++l) s += (l ? "," : "") + std::to_string(D.order[l]);
  s += "]\nrestrictions=[";
  for (size_t i = 0; i < P->restr.size(); ++i)
    s += (i ? "," : "") + std::string("(") + std::to_string(P->restr[i].first) + "," +
         std::to_string(P->restr[i].second) + ")";
  s += "]\n";
  auto lab = [&](unsigned m) -> std::string {
    if (m == STM_LAB_ANY) return "any";
    std::string r = "{";
    bool first = true;
    for (int i = 0; i < D.n_label_slots; ++i)
      if (m & (1u << i)) {
        if (!first) r += ",";
        r += std::to_string(D.label_value[i]);
        first = false;
      }
    return r + "}";
  };
  auto rawn = [&](int code) -> std::string {  // position code j + 8 d (directed: d = 0 out-row, 1 in-row)
    const std::string v = "(v" + std::to_string(code & 7) + ")";
    return D.directed ? ((code >> 3) ? "N-" : "N+") + v : "N" + v;
  };
  auto src = [&](const StmSrc& x) -> std::string {
    return x.kind == STM_SRC_RAW ? rawn(x.idx) : "S" + std::to_string(x.idx);
  };
  for (int i = 0; i < D.n_nodes; ++i) {
    const StmNode& n = D.nodes[i];
    std::string a = n.a_kind == STM_SRC_RAW ? rawn(n.a) : "S" + std::to_string(n.a);
    snprintf(buf, sizeof buf, "S%d: level %d stage %d = %s %s %s lab=%s lo=%s hi=%s\n", i, n.level,
             n.stage, a.c_str(), n.op == STM_OP_AND ? "&" : "-", rawn(n.b).c_str(), lab(n.lab).c_str(),
             fmt_mask(n.lo).c_str(), fmt_mask(n.hi).c_str());
    s += buf;
  }
  snprintf(buf, sizeof buf, "root: lab=%s\n", lab(D.filt[0].lab).c_str());
  s += buf;
  for (int l = 1; l < D.k - 1; ++l) {
    const StmFilter& f = D.filt[l];
    snprintf(buf, sizeof buf, "cand %d: %s lab=%s lo=%s hi=%s excl=%s\n", l, src(D.cand[l]).c_str(),
             lab(f.lab).c_str(), fmt_mask(f.lo).c_str(), fmt_mask(f.hi).c_str(), fmt_mask(f.excl).c_str());
    s += buf;
  }
  const StmFilter& f = D.filt[D.k - 1];
  std::string op = D.cnt_op == STM_OP_NONE ? "" : (D.cnt_op == STM_OP_AND ? " & " : " - ") + rawn(D.cnt_b);
  if (D.cnt_op == STM_OP_NONE) op = "";
  snprintf(buf, sizeof buf, "count %d: %s%s lab=%s lo=%s hi=%s excl=%s\n", D.k - 1, src(D.cnt_a).c_str(),
           op.c_str(), lab(f.lab).c_str(), fmt_mask(f.lo).c_str(), fmt_mask(f.hi).c_str(),
           fmt_mask(f.excl).c_str());
  s += buf;
  s += "need=[";
  for (int l = 1; l < D.k; ++l) s += (l > 1 ? "," : "") + std::to_string(D.need[l]);
  s += "] pretest=[";
  for (int l = 1; l < D.k; ++l) s += (l > 1 ? "," : "") + std::to_string(D.pretest[l]);
  s += "]\n";
  snprintf(buf, sizeof buf, "scratch_words_per_warp_per_cap=%d\n", D.n_nodes);
  s += buf;
  P->describe = s;
}

extern "C" stm_status stm_pattern_compile(int k, int n_edges, const int32_t* edges,
                                          const int32_t* labels, const int32_t* order, int n_restr,
                                          const int32_t* restr, uint32_t flags, stm_plan** out) {
  if (!out) return stm_fail(STM_EINVAL, "out is NULL");
  if (k < 2) return stm_fail(STM_EINVAL, "pattern size k=%d < 2 is not a matching query", k);
  if (k > STM_KMAX) return stm_fail(STM_EUNSUPPORTED, "pattern size k=%d > %d", k, STM_KMAX);
  if (n_edges < 1 || !edges) return stm_fail(STM_EINVAL, "pattern has no edges");
  if (flags & ~(0x1Fu | STM_DIRECTED)) return stm_fail(STM_EINVAL, "unknown flag bits 0x%x", flags);
  const bool vi = flags & STM_VERTEX_INDUCED;
  const bool directed = flags & STM_DIRECTED;  // edges are arcs a -> b (NEXT-4)
  const bool cm = !(flags & STM_NO_CODE_MOTION);
  const bool lazy = cm && (flags & STM_LAZY_UNBOUNDED);

  int adj[STM_KMAX][STM_KMAX] = {};   // underlying undirected pattern graph
  int dadj[STM_KMAX][STM_KMAX] = {};  // arcs (directed patterns; = adj for undirected ones)
  std::vector<std::pair<int, int>> E;
  for (int i = 0; i < n_edges; ++i) {
    int a = edges[2 * i], b = edges[2 * i + 1];
    if (a < 0 || b < 0 || a >= k || b >= k) return stm_fail(STM_EINVAL, "edge %d out of range", i);
    if (a == b) return stm_fail(STM_EINVAL, "self-loop in pattern at vertex %d", a);
    if (directed) {
      if (!dadj[a][b]) E.push_back({a, b});
      dadj[a][b] = 1;
    } else {
      if (!adj[a][b]) E.push_back({std::min(a, b), std::max(a, b)});
      dadj[a][b] = dadj[b][a] = 1;
    }
    adj[a][b] = adj[b][a] = 1;
  }
  {  // connectivity
    int seen[STM_KMAX] = {1}, stack[STM_KMAX], sp = 0, cnt = 1;
    stack[sp++] = 0;
    while (sp) {
      int u = stack[--sp];
      for (int v = 0; v < k; ++v)
        if (adj[u][v] && !seen[v]) { seen[v] = 1; ++cnt; stack[sp++] = v; }
    }
    if (cnt != k) return stm_fail(STM_EINVAL, "pattern is disconnected");
  }
  std::vector<int> lab(k, -2);  // -2: unlabeled pattern
  if (labels) {
    for (int u = 0; u < k; ++u) {
      if (labels[u] < -1) return stm_fail(STM_EINVAL, "pattern label %d < -1", labels[u]);
      lab[u] = labels[u];
    }
  }

  // ---- label-preserving automorphisms (brute force over k! permutations)
  std::vector<std::vector<int>> group;
  {
    std::vector<int> p(k);
    for (int i = 0; i < k; ++i) p[i] = i;
    do {
      bool ok = true;
      for (int u = 0; u < k && ok; ++u) ok = lab[p[u]] == lab[u];
      for (auto& e : E) {  // (arcs map to arcs for directed patterns)
        if (!ok) break;
        ok = dadj[p[e.first]][p[e.second]];
      }
      if (ok) group.push_back(p);
    } while (next_perm(p));
  }
  const int64_t aut = (int64_t)group.size();

  // ---- restrictions
  std::vector<std::pair<int, int>> R;
  if (flags & STM_AUTO_RESTRICT) {
    // Grochow-Kellis: fix the smallest vertex with a non-trivial orbit, order it
    // below the rest of its orbit, continue in its stabiliser.
    std::vector<std::vector<int>> G = group;
    while (G.size() > 1) {
      int u = -1;
      std::vector<int> orbit;
      for (int x = 0; x < k && u < 0; ++x) {
        std::vector<int> o;
        for (auto& p : G) o.push_back(p[x]);
        std::sort(o.begin(), o.end());
        o.erase(std::unique(o.begin(), o.end()), o.end());
        if (o.size() > 1) { u = x; orbit = o; }
      }
      for (int w : orbit)
        if (w != u) R.push_back({u, w});
      std::vector<std::vector<int>> H;
      for (auto& p : G)
        if (p[u] == u) H.push_back(p);
      G.swap(H);
    }
  } else {
    if (n_restr < 0 || (n_restr > 0 && !restr)) return stm_fail(STM_EINVAL, "bad restriction array");
    for (int i = 0; i < n_restr; ++i) {
      int a = restr[2 * i], b = restr[2 * i + 1];
      if (a < 0 || b < 0 || a >= k || b >= k) return stm_fail(STM_EINVAL, "restriction %d out of range", i);
      if (a == b) return stm_fail(STM_EINVAL, "restriction %d has a == b", i);
      R.push_back({a, b});
    }
  }
  // transitive closure over pattern vertices; a cycle means no embedding can exist
  int less[STM_KMAX][STM_KMAX] = {};
  for (auto& r : R) less[r.first][r.second] = 1;
  for (int m = 0; m < k; ++m)
    for (int i = 0; i < k; ++i)
      for (int j = 0; j < k; ++j)
        if (less[i][m] && less[m][j]) less[i][j] = 1;
  for (int i = 0; i < k; ++i)
    if (less[i][i]) return stm_fail(STM_EINVAL, "restriction set is cyclic");

  // ---- matching order
  std::vector<int> pi;
  int deg[STM_KMAX] = {};
  for (int u = 0; u < k; ++u)
    for (int v = 0; v < k; ++v) deg[u] += adj[u][v];
  if (order && !(flags & STM_AUTO_ORDER)) {
    std::vector<int> seen(k, 0);
    for (int l = 0; l < k; ++l) {
      int u = order[l];
      if (u < 0 || u >= k || seen[u]) return stm_fail(STM_EINVAL, "order is not a permutation");
      if (l > 0) {
        bool con = false;
        for (int j = 0; j < l; ++j) con |= adj[u][order[j]] != 0;
        if (!con)
          return stm_fail(STM_EINVAL, "order[%d]=%d is not adjacent to an earlier vertex (PAPER.md:52)", l, u);
      }
      seen[u] = 1;
      pi.push_back(u);
    }
  } else {
    // greedy: max degree first (lowest id), then most already-ordered neighbours,
    // ties by higher degree, then lower id (reading R6)
    std::vector<int> in(k, 0);
    int first = 0;
    for (int u = 1; u < k; ++u)
      if (deg[u] > deg[first]) first = u;
    pi.push_back(first);
    in[first] = 1;
    while ((int)pi.size() < k) {
      int best = -1, bc = -1;
      for (int u = 0; u < k; ++u) {
        if (in[u]) continue;
        int c = 0;
        for (int v : pi) c += adj[u][v];
        if (c == 0) continue;
        if (c > bc || (c == bc && deg[u] > deg[best])) { best = u; bc = c; }
      }
      pi.push_back(best);
      in[best] = 1;
    }
  }

  stm_plan* P = new (std::nothrow) stm_plan();
  if (!P) return stm_fail(STM_ENOMEM, "out of host memory");
  P->k = k;
  P->edges = E;
  P->labels = labels ? std::vector<int>(labels, labels + k) : std::vector<int>();
  P->restr = R;
  P->aut = aut;
  P->flags = flags;
  P->order_free = (flags & STM_AUTO_RESTRICT) || R.empty();
  StmPlan& D = P->dev;
  memset(&D, 0, sizeof D);
  D.k = k;
  D.vertex_induced = vi;
  D.directed = directed ? 1 : 0;
  for (int l = 0; l < k; ++l) D.order[l] = pi[l];

  // label slots
  std::vector<int> slots;
  for (int u = 0; u < k; ++u)
    if (lab[u] >= 0 && std::find(slots.begin(), slots.end(), lab[u]) == slots.end()) slots.push_back(lab[u]);
  D.n_label_slots = (int)slots.size();
  for (size_t i = 0; i < slots.size(); ++i) D.label_value[i] = slots[i];
  auto labmask = [&](int l) -> unsigned {
    int x = lab[pi[l]];
    if (x < 0) return STM_LAB_ANY;
    return 1u << (std::find(slots.begin(), slots.end(), x) - slots.begin());
  };

  // per-position signatures, bounds, exclusions.  A raw operand is named by a position
  // code j + 8 d: N(v_j) for undirected plans (d = 0); for directed ones d = 0 is the out-
  // row N+(v_j) (pattern arc pi[j] -> pi[l]) and d = 1 the in-row N-(v_j) (arc pi[l] -> pi[j]).
  int sig[STM_KMAX][2 * STM_KMAX] = {};  // per code: +1 member, -1 difference (vertex-induced), 0 none
  unsigned lo_pos[STM_KMAX] = {}, hi_pos[STM_KMAX] = {}, excl[STM_KMAX] = {};
  for (int l = 0; l < k; ++l)
    for (int j = 0; j < l; ++j) {
      if (directed) {
        sig[l][j] = dadj[pi[j]][pi[l]] ? 1 : (vi ? -1 : 0);
        sig[l][j + 8] = dadj[pi[l]][pi[j]] ? 1 : (vi ? -1 : 0);
      } else {
        sig[l][j] = adj[pi[l]][pi[j]] ? 1 : (vi ? -1 : 0);
      }
      if (less[pi[j]][pi[l]]) lo_pos[l] |= 1u << j;
      if (less[pi[l]][pi[j]]) hi_pos[l] |= 1u << j;
      if (!adj[pi[l]][pi[j]]) excl[l] |= 1u << j;
    }

  // Drop dominated bounds: w > v_j is implied by w > v_j' when f(pi[j]) < f(pi[j'])
  // already holds (transitive closure), so only the maximal lower and minimal upper
  // bound positions are kept (one compare each for cliques instead of up to k-1).
  auto reduce_lo = [&](unsigned m) {
    unsigned r = m;
    for (int j = 0; j < k; ++j)
      for (int j2 = 0; j2 < k; ++j2)
        if ((m >> j & 1) && (m >> j2 & 1) && j != j2 && less[pi[j]][pi[j2]]) r &= ~(1u << j);
    return r;
  };
  auto reduce_hi = [&](unsigned m) {
    unsigned r = m;
    for (int j = 0; j < k; ++j)
      for (int j2 = 0; j2 < k; ++j2)
        if ((m >> j & 1) && (m >> j2 & 1) && j != j2 && less[pi[j2]][pi[j]]) r &= ~(1u << j);
    return r;
  };

  // ---- operation chains and the code-motion trie
  struct TNode {
    int level, a_kind, a, b, op;
    std::vector<int> consumers;
  };
  std::vector<TNode> tn;
  std::map<std::vector<int>, int> key2node;
  std::vector<StmSrc> cand_src(k);
  for (int l = 1; l < k; ++l) {
    Chain c;
    // codes in scan order: position j, then its out- / in-row (directed)
    std::vector<int> codes;
    for (int j = 0; j < l; ++j) {
      codes.push_back(j);
      if (directed) codes.push_back(j + 8);
    }
    size_t fi = 0;
    while (fi < codes.size() && sig[l][codes[fi]] != 1) ++fi;
    c.f = codes[fi];  // (the order is connected: some earlier position is adjacent)
    for (size_t t = 0; t < fi; ++t)
      if (sig[l][codes[t]] == -1) { c.ops.push_back({STM_OP_DIFF, codes[t]}); c.level.push_back((c.f & 7) + 1); }
    for (size_t t = fi + 1; t < codes.size(); ++t)
      if (sig[l][codes[t]] != 0) {
        c.ops.push_back({sig[l][codes[t]] == 1 ? STM_OP_AND : STM_OP_DIFF, codes[t]});
        c.level.push_back((codes[t] & 7) + 1);
      }
    if (!cm)
      for (auto& x : c.level) x = l;
    std::vector<int> key = {c.f};
    if (!cm) key.push_back(100 + l);  // no sharing across targets without code motion
    int prev_kind = STM_SRC_RAW, prev = c.f;
    int lazy_level = 0;  // lazy mode: once a chain op is unbounded for this consumer, it and the
                         // rest of the chain are computed at the consumer's level
    for (size_t t = 0; t < c.ops.size(); ++t) {
      key.push_back(c.ops[t].first * 16 + c.ops[t].second);  // (codes < 16)
      int level = c.level[t];
      if (lazy) {
        const unsigned known = (1u << c.level[t]) - 1;
        const unsigned lo = reduce_lo(lo_pos[l] & known), hi = reduce_hi(hi_pos[l] & known);
        if (!lo && !hi && !lazy_level) lazy_level = l;
        if (lazy_level) level = lazy_level;
        if (prev_kind == STM_SRC_NODE) level = std::max(level, tn[prev].level);
        key.push_back(1000 + (int)(lo | hi << 8));  // no sharing across bound classes
      }
      auto it = key2node.find(key);
      int id;
      if (it == key2node.end()) {
        id = (int)tn.size();
        tn.push_back({level, prev_kind, prev, c.ops[t].second, c.ops[t].first, {}});
        key2node[key] = id;
      } else {
        id = it->second;
      }
      tn[id].consumers.push_back(l);
      prev_kind = STM_SRC_NODE;
      prev = id;
    }
    cand_src[l].kind = (int8_t)prev_kind;
    cand_src[l].idx = (int16_t)prev;
  }

  // ---- the final level is counted, never materialised (PAPER.md:75 Output at the
  // last level; counting is north_star's reading)
  int drop = -1;
  StmSrc last = cand_src[k - 1];
  if (last.kind == STM_SRC_NODE && tn[last.idx].level == k - 1) {
    const TNode& x = tn[last.idx];
    drop = last.idx;
    D.cnt_a.kind = (int8_t)x.a_kind;
    D.cnt_a.idx = (int16_t)x.a;
    D.cnt_b = (int8_t)x.b;
    D.cnt_op = (int8_t)x.op;
    bool a_same_level = x.a_kind == STM_SRC_NODE && tn[x.a].level == k - 1;
    D.count_mode = (k >= 3 && !a_same_level) ? STM_COUNT_FUSED : STM_COUNT_FRAME;
  } else {
    D.cnt_a = last;
    D.cnt_b = -1;
    D.cnt_op = STM_OP_NONE;
    D.count_mode = (k >= 3) ? STM_COUNT_FUSED : STM_COUNT_FRAME;
  }

  // ---- order nodes by (level, stage), drop the fused final node, set filters
  std::vector<int> stage(tn.size(), 0);
  for (size_t i = 0; i < tn.size(); ++i)  // creation order is topological
    if (tn[i].a_kind == STM_SRC_NODE && tn[tn[i].a].level == tn[i].level) stage[i] = stage[tn[i].a] + 1;
  std::vector<int> ids;
  for (size_t i = 0; i < tn.size(); ++i)
    if ((int)i != drop) ids.push_back((int)i);
  std::stable_sort(ids.begin(), ids.end(), [&](int x, int y) {
    return tn[x].level != tn[y].level ? tn[x].level < tn[y].level : stage[x] < stage[y];
  });
  if ((int)ids.size() > STM_MAX_NODES) {
    delete P;
    return stm_fail(STM_EUNSUPPORTED, "plan needs %zu set nodes > %d", ids.size(), STM_MAX_NODES);
  }
  std::vector<int> remap(tn.size(), -1);
  for (size_t i = 0; i < ids.size(); ++i) remap[ids[i]] = (int)i;
  D.n_nodes = (int)ids.size();
  for (size_t i = 0; i < ids.size(); ++i) {
    const TNode& x = tn[ids[i]];
    StmNode& n = D.nodes[i];
    n.level = (int8_t)x.level;
    n.stage = (int8_t)stage[ids[i]];
    n.a_kind = (int8_t)x.a_kind;
    n.a = (int16_t)(x.a_kind == STM_SRC_NODE ? remap[x.a] : x.a);
    n.b = (int8_t)x.b;
    n.op = (int8_t)x.op;
    unsigned lm = 0, lo = 0xFF, hi = 0xFF;
    for (int t : x.consumers) {
      unsigned m = labmask(t);
      lm = (lm == STM_LAB_ANY || m == STM_LAB_ANY) ? STM_LAB_ANY : (lm | m);
      lo &= lo_pos[t];
      hi &= hi_pos[t];
    }
    unsigned known = (1u << x.level) - 1;  // v_0..v_{level-1}
    n.lab = (uint8_t)lm;
    n.lo = (uint8_t)reduce_lo(lo & known);
    n.hi = (uint8_t)reduce_hi(hi & known);
  }
  for (int l = 0; l <= k; ++l) D.level_begin[l] = 0;
  for (int l = 0; l < k; ++l) {
    int b = 0;
    while (b < D.n_nodes && D.nodes[b].level < l) ++b;
    D.level_begin[l] = (int8_t)b;
  }
  D.level_begin[k] = (int8_t)D.n_nodes;
  for (int l = 0; l < k; ++l) {
    int ns = 0;
    for (int i = D.level_begin[l]; i < D.level_begin[l + 1]; ++i) ns = std::max(ns, D.nodes[i].stage + 1);
    D.n_stages[l] = (int8_t)ns;
  }
  for (int l = 1; l < k; ++l)
    if (cand_src[l].kind == STM_SRC_NODE && cand_src[l].idx != drop)
      cand_src[l].idx = (int16_t)remap[cand_src[l].idx];
  for (int l = 1; l < k; ++l) D.cand[l] = cand_src[l];
  if (D.cnt_a.kind == STM_SRC_NODE) D.cnt_a.idx = (int16_t)remap[D.cnt_a.idx];
  for (int l = 0; l < k; ++l) {
    D.filt[l].lab = (uint8_t)labmask(l);
    D.filt[l].lo = (uint8_t)reduce_lo(lo_pos[l]);
    D.filt[l].hi = (uint8_t)reduce_hi(hi_pos[l]);
    D.filt[l].excl = (uint8_t)excl[l];
  }

  // ---- candidate-set pruning (plan.h need / pretest).  v_m (m > l) is necessarily an
  // element of level l's candidate set C_l = S_l ∩ filter_l when (i) m's candidate
  // source is a subset of S_l (S_l itself, a node whose operand chain passes through
  // S_l, or a chain starting at the same raw list) and (ii) the pattern forces v_m
  // through filter_l: every bound of level l holds for pi[m] by the restriction closure
  // and the label matches.  Injectivity makes v_l and those v_m distinct elements of C_l.
  {
    auto chain_has = [&](StmSrc t, StmSrc s) {  // t ⊆ s through t's operand chain
      for (;;) {
        if (t.kind == s.kind && t.idx == s.idx) return true;
        if (t.kind == STM_SRC_RAW) return false;
        const StmNode& nd = D.nodes[t.idx];
        t.kind = nd.a_kind;
        t.idx = nd.a;
      }
    };
    auto src_of = [&](int m) -> StmSrc {  // a set containing every candidate of level m
      return m == k - 1 ? D.cnt_a : D.cand[m];
    };
    for (int l = 1; l < k; ++l) {
      int need = 1;
      const StmSrc s = src_of(l);
      const unsigned lm = labmask(l);
      for (int m = l + 1; m < k; ++m) {
        if (!chain_has(src_of(m), s)) continue;
        if (lm != STM_LAB_ANY && labmask(m) != lm) continue;
        bool forced = true;
        for (int j = 0; j < l && forced; ++j) {
          if ((lo_pos[l] >> j & 1) && !less[pi[j]][pi[m]]) forced = false;
          if ((hi_pos[l] >> j & 1) && !less[pi[m]][pi[j]]) forced = false;
        }
        if (forced) ++need;
      }
      D.need[l] = (int8_t)need;
      // pre-test: unbounded stage-0 node of level l feeding a bounded consumer
      D.pretest[l] = 0;
      if (l >= 2 && l < k - 1 && D.cand[l].kind == STM_SRC_NODE) {
        const StmNode& nd = D.nodes[D.cand[l].idx];
        if (nd.level == l && nd.stage == 0 && (D.filt[l].lo | D.filt[l].hi) &&
            ((D.filt[l].lo & ~nd.lo) | (D.filt[l].hi & ~nd.hi)))
          D.pretest[l] = 1;
      }
    }
  }
  build_describe(P);
  *out = P;
  return STM_OK;
}

extern "C" stm_status stm_plan_describe(const stm_plan* p, char* buf, size_t len) {
  if (!p || !buf) return stm_fail(STM_EINVAL, "NULL argument");
  if (p->describe.size() + 1 > len)
    return stm_fail(STM_EINVAL, "buffer too small: need %zu bytes", p->describe.size() + 1);
  memcpy(buf, p->describe.c_str(), p->describe.size() + 1);
  return STM_OK;
}

extern "C" stm_status stm_plan_raw(const stm_plan* p, void* buf, size_t len, size_t* size) {
  if (!p) return stm_fail(STM_EINVAL, "NULL plan");
  if (size) *size = sizeof(StmPlan);
  if (buf) {
    if (len < sizeof(StmPlan)) return stm_fail(STM_EINVAL, "buffer of %zu bytes < %zu", len, sizeof(StmPlan));
    memcpy(buf, &p->dev, sizeof(StmPlan));
  }
  return STM_OK;
}

extern "C" stm_status stm_plan_info(const stm_plan* p, int* k, int* n_sets, int64_t* aut) {
  if (!p) return stm_fail(STM_EINVAL, "NULL plan");
  if (k) *k = p->k;
  if (n_sets) *n_sets = p->dev.n_nodes;
  if (aut) *aut = p->aut;
  return STM_OK;
}

extern "C" stm_status stm_plan_first_vertex(const stm_plan* p, int* u0) {
  if (!p || !u0) return stm_fail(STM_EINVAL, "NULL argument");
  *u0 = p->dev.order[0];
  return STM_OK;
}

extern "C" stm_status stm_plan_free(stm_plan* p) {
  delete p;
  return STM_OK;
}
