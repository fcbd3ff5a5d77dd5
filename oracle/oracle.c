/*
 * oracle/oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously correct CPU counter of pattern embeddings.  Only
 * tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  It shares no code, header, table or helper with
 * the CUDA path (paper_conf_sc_weij22_b200/), and the product never calls it.
 *
 * What it computes (Sec. II-A problem definition):
 *
 *   count = | { f : V_Q -> V injective :
 *                for every pattern edge {a,b}:           {f(a), f(b)} in E
 *                [vertex-induced] every pattern non-edge: {f(a), f(b)} not in E
 *                [labeled]  L_G(f(u)) == L_Q(u) for every u
 *                for every restriction (a,b):            f(a) < f(b) } |   mod 2^64
 *
 * How (Algorithm 1, the Fig. 1 nested loop): a plain
 * recursive backtracking in the oracle's OWN matching order (BFS over Q from a
 * root pattern vertex), which satisfies the paper's rule that pi[l+1] is adjacent
 * to one of pi[0..l].  Candidates for pi[l] are the neighbours of
 * the image of one already-matched pattern neighbour p (the one whose image has
 * the smallest degree: the same candidate set, less work).  Every other
 * condition of the definition is then checked literally for the candidate:
 * injectivity, adjacency (binary search) to every other matched pattern
 * neighbour, non-adjacency to every matched pattern non-neighbour
 * (vertex-induced only; "removing the set difference operations"
 * gives edge-induced), the label, and every restriction whose two endpoints are
 * now matched.  No set operation, plan, code motion, unrolling or stealing.
 *
 * Level 0 is split into chunks of roots taken by pthreads from an atomic
 * counter; each thread keeps a private uint64 partial count.
 *
 * Input requirements: undirected simple graph, rows sorted ascending (checked
 * by the Python wrapper), pattern connected with 1 <= k <= 16.
 *
 * Directed graphs ("supports both directed and undirected graphs";
 * SURVEY.md 8(f) NEXT-4), oracle_count_directed: G is a simple digraph given by its
 * sorted out-neighbour rows (and, for candidate generation only, the transposed in-
 * neighbour rows); Q's edges are ordered pairs (a, b) = arc a -> b.  The definition is
 * the same with arcs:
 *
 *   for every pattern arc a -> b:                f(a) -> f(b) is an arc of G
 *   [vertex-induced] every pattern non-arc a -> b: f(a) -> f(b) is not an arc of G
 *
 * checked literally per candidate (arc x -> y = y in out(x), binary search); the
 * matching order is the BFS over Q's underlying undirected graph.
 */
#include <pthread.h>
#include <stdatomic.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OMAX 16

typedef struct {
  /* data graph */
  int64_t n;
  const int64_t *row_ptr;
  const int32_t *col_idx;
  const int32_t *labels; /* NULL = unlabeled */
  /* pattern, already arranged in matching order: position l is pattern vertex order[l] */
  int k;
  int order[OMAX];
  int adj[OMAX][OMAX];     /* pattern adjacency by pattern vertex id */
  int plabel[OMAX];        /* by pattern vertex id */
  int use_labels;
  int vertex_induced;
  int n_restr;
  const int32_t *restr;    /* pairs (a,b): f(a) < f(b), pattern vertex ids */
  /* roots */
  const int64_t *roots;    /* NULL = all of [0, n) */
  int64_t n_roots;
  atomic_llong next;
  int64_t chunk;
  uint64_t *per_root;      /* NULL or [n_roots] (indexed like roots) */
  /* listing (PAPER.md:75 Output(C, iter)): every embedding f, as f[0..k-1] in pattern-vertex
     order, is appended at an atomically taken index; only indices < list_cap are written */
  int32_t *list;
  uint64_t list_cap;
  atomic_ullong list_n;
  /* directed graphs: dadj[a][b] = 1 iff pattern arc a -> b; adj is then its underlying
     undirected graph (BFS order only); in_* = transposed rows (candidates only) */
  int directed;
  int dadj[OMAX][OMAX];
  const int64_t *in_row_ptr;
  const int32_t *in_col_idx;
} ojob;

typedef struct {
  ojob *J;
  int64_t f[OMAX];         /* f[u] = image of pattern vertex u, -1 if unmatched */
  uint64_t count;
} ostate;

static int adjacent(const ojob *J, int64_t x, int64_t y) {
  int64_t lo = J->row_ptr[x], hi = J->row_ptr[x + 1];
  while (lo < hi) {
    int64_t mid = lo + ((hi - lo) >> 1);
    int64_t c = J->col_idx[mid];
    if (c == y) return 1;
    if (c < y) lo = mid + 1; else hi = mid;
  }
  return 0;
}

/* does the candidate w for pattern vertex u satisfy the definition w.r.t. all
   already-matched pattern vertices? */
static int consistent(const ostate *S, int l, int u, int64_t w) {
  const ojob *J = S->J;
  if (J->use_labels && J->labels[w] != J->plabel[u]) return 0;
  for (int j = 0; j < l; ++j) {
    int q = J->order[j];
    int64_t fq = S->f[q];
    if (fq == w) return 0; /* injective */
    if (J->adj[u][q]) {
      if (!adjacent(J, fq, w)) return 0; /* pattern edge must be a data edge */
    } else if (J->vertex_induced) {
      if (adjacent(J, fq, w)) return 0; /* pattern non-edge must be a data non-edge */
    }
  }
  for (int r = 0; r < J->n_restr; ++r) {
    int a = J->restr[2 * r], b = J->restr[2 * r + 1];
    int64_t fa = (a == u) ? w : S->f[a];
    int64_t fb = (b == u) ? w : S->f[b];
    if ((a == u || b == u) && fa >= 0 && fb >= 0 && !(fa < fb)) return 0;
  }
  return 1;
}

/* directed: the definition with arcs, checked literally (arc x -> y: y in out(x)) */
static int consistent_directed(const ostate *S, int l, int u, int64_t w) {
  const ojob *J = S->J;
  if (J->use_labels && J->labels[w] != J->plabel[u]) return 0;
  for (int j = 0; j < l; ++j) {
    int q = J->order[j];
    int64_t fq = S->f[q];
    if (fq == w) return 0; /* injective */
    if (J->dadj[q][u]) {
      if (!adjacent(J, fq, w)) return 0; /* pattern arc q -> u must be a data arc */
    } else if (J->vertex_induced) {
      if (adjacent(J, fq, w)) return 0;
    }
    if (J->dadj[u][q]) {
      if (!adjacent(J, w, fq)) return 0; /* pattern arc u -> q must be a data arc */
    } else if (J->vertex_induced) {
      if (adjacent(J, w, fq)) return 0;
    }
  }
  for (int r = 0; r < J->n_restr; ++r) {
    int a = J->restr[2 * r], b = J->restr[2 * r + 1];
    int64_t fa = (a == u) ? w : S->f[a];
    int64_t fb = (b == u) ? w : S->f[b];
    if ((a == u || b == u) && fa >= 0 && fb >= 0 && !(fa < fb)) return 0;
  }
  return 1;
}

static void rec_directed(ostate *S, int l) {
  const ojob *J = S->J;
  if (l == J->k) {
    S->count += 1;
    return;
  }
  int u = J->order[l];
  /* candidates: the out-row of f(q) for a pattern arc q -> u, or the in-row of f(q) for
     u -> q, whichever matched pattern neighbour gives the shortest row */
  const int32_t *best = NULL;
  int64_t bestlen = -1;
  for (int j = 0; j < l; ++j) {
    int q = J->order[j];
    int64_t fq = S->f[q];
    if (J->dadj[q][u]) {
      int64_t d = J->row_ptr[fq + 1] - J->row_ptr[fq];
      if (bestlen < 0 || d < bestlen) { best = J->col_idx + J->row_ptr[fq]; bestlen = d; }
    }
    if (J->dadj[u][q]) {
      int64_t d = J->in_row_ptr[fq + 1] - J->in_row_ptr[fq];
      if (bestlen < 0 || d < bestlen) { best = J->in_col_idx + J->in_row_ptr[fq]; bestlen = d; }
    }
  }
  for (int64_t e = 0; e < bestlen; ++e) {
    int64_t w = best[e];
    if (!consistent_directed(S, l, u, w)) continue;
    S->f[u] = w;
    rec_directed(S, l + 1);
    S->f[u] = -1;
  }
}

static void rec(ostate *S, int l) {
  const ojob *J = S->J;
  if (l == J->k) {
    S->count += 1;
    if (J->list) {
      uint64_t i = atomic_fetch_add((atomic_ullong *)&J->list_n, 1);
      if (i < J->list_cap)
        for (int u = 0; u < J->k; ++u) J->list[i * (uint64_t)J->k + u] = (int32_t)S->f[u];
    }
    return;
  }
  int u = J->order[l];
  /* matched pattern neighbour whose image has the smallest degree */
  int64_t best = -1, bestdeg = 0;
  for (int j = 0; j < l; ++j) {
    int q = J->order[j];
    if (!J->adj[u][q]) continue;
    int64_t fq = S->f[q];
    int64_t d = J->row_ptr[fq + 1] - J->row_ptr[fq];
    if (best < 0 || d < bestdeg) { best = fq; bestdeg = d; }
  }
  for (int64_t e = J->row_ptr[best]; e < J->row_ptr[best + 1]; ++e) {
    int64_t w = J->col_idx[e];
    if (!consistent(S, l, u, w)) continue;
    S->f[u] = w;
    rec(S, l + 1);
    S->f[u] = -1;
  }
}

static void *worker(void *arg) {
  ostate *S = (ostate *)arg;
  ojob *J = S->J;
  for (;;) {
    int64_t b = atomic_fetch_add(&J->next, J->chunk);
    if (b >= J->n_roots) break;
    int64_t e = b + J->chunk < J->n_roots ? b + J->chunk : J->n_roots;
    for (int64_t i = b; i < e; ++i) {
      int64_t v = J->roots ? J->roots[i] : i;
      uint64_t before = S->count;
      int u0 = J->order[0];
      for (int x = 0; x < OMAX; ++x) S->f[x] = -1;
      if (J->directed) {
        if (consistent_directed(S, 0, u0, v)) {
          S->f[u0] = v;
          rec_directed(S, 1);
          S->f[u0] = -1;
        }
      } else if (consistent(S, 0, u0, v)) {
        S->f[u0] = v;
        rec(S, 1);
        S->f[u0] = -1;
      }
      if (J->per_root) J->per_root[i] = S->count - before;
    }
  }
  return NULL;
}

/*
 * Oracle's own matching order: BFS over Q starting at root_u (or, if root_u < 0,
 * at the lowest-ID vertex of maximum degree); neighbours visited in increasing
 * ID.  Returns 0 if Q is disconnected (not a valid query).
 */
static int bfs_order(int k, int adj[OMAX][OMAX], int root_u, int *order) {
  if (root_u < 0) {
    int bestd = -1;
    for (int u = 0; u < k; ++u) {
      int d = 0;
      for (int v = 0; v < k; ++v) d += adj[u][v];
      if (d > bestd) { bestd = d; root_u = u; }
    }
  }
  int seen[OMAX] = {0};
  int head = 0, tail = 0;
  order[tail++] = root_u;
  seen[root_u] = 1;
  while (head < tail) {
    int u = order[head++];
    for (int v = 0; v < k; ++v)
      if (adj[u][v] && !seen[v]) { seen[v] = 1; order[tail++] = v; }
  }
  return tail == k;
}

/*
 * Returns 0 on success, -1 on invalid input.  `edges` holds n_edges pairs of
 * pattern vertex ids; `plabels` may be NULL (unlabeled); `restr` holds n_restr
 * pairs (a, b) meaning f(a) < f(b).  `roots`/`n_roots` restrict level 0 to the
 * given data vertices (NULL = all); `per_root` (optional) receives the count
 * attributed to each root, i.e. to f(root_u).
 */
static int run(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, const int32_t *labels,
               int k, int n_edges, const int32_t *edges, const int32_t *plabels,
               int vertex_induced, int n_restr, const int32_t *restr, int root_u,
               const int64_t *roots, int64_t n_roots, int nthreads, uint64_t *per_root,
               int32_t *list, uint64_t list_cap, uint64_t *list_n, uint64_t *out_count,
               const int64_t *in_row_ptr, const int32_t *in_col_idx) {
  if (k < 1 || k > OMAX) return -1;
  ojob *J = (ojob *)calloc(1, sizeof(ojob));
  J->n = n; J->row_ptr = row_ptr; J->col_idx = col_idx; J->labels = labels;
  J->k = k;
  J->directed = in_row_ptr != NULL;
  J->in_row_ptr = in_row_ptr;
  J->in_col_idx = in_col_idx;
  if (J->directed && list) { free(J); return -1; }
  for (int i = 0; i < n_edges; ++i) {
    int a = edges[2 * i], b = edges[2 * i + 1];
    if (a < 0 || b < 0 || a >= k || b >= k || a == b) { free(J); return -1; }
    J->adj[a][b] = J->adj[b][a] = 1;
    J->dadj[a][b] = 1;
  }
  if (root_u >= k) { free(J); return -1; }
  if (!bfs_order(k, J->adj, root_u, J->order)) { free(J); return -1; }
  J->use_labels = plabels != NULL;
  if (J->use_labels && !labels) { free(J); return -1; }
  for (int u = 0; u < k; ++u) J->plabel[u] = plabels ? plabels[u] : 0;
  J->vertex_induced = vertex_induced;
  J->n_restr = n_restr;
  J->restr = restr;
  for (int r = 0; r < n_restr; ++r)
    if (restr[2 * r] < 0 || restr[2 * r] >= k || restr[2 * r + 1] < 0 || restr[2 * r + 1] >= k) {
      free(J);
      return -1;
    }
  J->roots = roots;
  J->n_roots = roots ? n_roots : n;
  atomic_init(&J->next, 0);
  J->chunk = 64;
  J->per_root = per_root;
  J->list = list;
  J->list_cap = list_cap;
  atomic_init(&J->list_n, 0);
  if (nthreads < 1) nthreads = 1;
  if (nthreads > 256) nthreads = 256;
  pthread_t th[256];
  ostate *S = (ostate *)calloc((size_t)nthreads, sizeof(ostate));
  for (int t = 0; t < nthreads; ++t) {
    S[t].J = J;
    pthread_create(&th[t], NULL, worker, &S[t]);
  }
  uint64_t total = 0;
  for (int t = 0; t < nthreads; ++t) {
    pthread_join(th[t], NULL);
    total += S[t].count;
  }
  free(S);
  if (list_n) *list_n = atomic_load(&J->list_n);
  free(J);
  *out_count = total;
  return 0;
}

/* count (see run) */
int oracle_count(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, const int32_t *labels,
                 int k, int n_edges, const int32_t *edges, const int32_t *plabels,
                 int vertex_induced, int n_restr, const int32_t *restr, int root_u,
                 const int64_t *roots, int64_t n_roots, int nthreads, uint64_t *per_root,
                 uint64_t *out_count) {
  return run(n, row_ptr, col_idx, labels, k, n_edges, edges, plabels, vertex_induced, n_restr, restr, root_u,
             roots, n_roots, nthreads, per_root, NULL, 0, NULL, out_count, NULL, NULL);
}

/* directed graphs: `edges` are arcs (a -> b); in_row_ptr / in_col_idx = the transposed rows */
int oracle_count_directed(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, const int64_t *in_row_ptr,
                          const int32_t *in_col_idx, const int32_t *labels, int k, int n_edges,
                          const int32_t *edges, const int32_t *plabels, int vertex_induced, int n_restr,
                          const int32_t *restr, int root_u, const int64_t *roots, int64_t n_roots,
                          int nthreads, uint64_t *per_root, uint64_t *out_count) {
  if (!in_row_ptr || !in_col_idx) return -1;
  return run(n, row_ptr, col_idx, labels, k, n_edges, edges, plabels, vertex_induced, n_restr, restr, root_u,
             roots, n_roots, nthreads, per_root, NULL, 0, NULL, out_count, in_row_ptr, in_col_idx);
}

/* count and list: list[i*k + u] = f(u) for the first min(count, list_cap) embeddings found
   (in no particular order); *list_n = count as well (the number of listing slots taken) */
int oracle_list(int64_t n, const int64_t *row_ptr, const int32_t *col_idx, const int32_t *labels,
                int k, int n_edges, const int32_t *edges, const int32_t *plabels,
                int vertex_induced, int n_restr, const int32_t *restr, int root_u,
                const int64_t *roots, int64_t n_roots, int nthreads,
                int32_t *list, uint64_t list_cap, uint64_t *list_n, uint64_t *out_count) {
  return run(n, row_ptr, col_idx, labels, k, n_edges, edges, plabels, vertex_induced, n_restr, restr, root_u,
             roots, n_roots, nthreads, NULL, list, list_cap, list_n, out_count, NULL, NULL);
}
