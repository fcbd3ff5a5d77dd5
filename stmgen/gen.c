/*
 * stmgen/gen.c -- seeded synthetic graph generators + CSR canonicaliser.
 *
 * INPUT GENERATION ONLY.  This file holds none of the matching method's
 * arithmetic (no set operations, no backtracking, no counting); it is the one
 * module that both the oracle tests and the CUDA path consume (DESIGN.md,
 * "Input recipe").  Everything is driven by a counter-based generator
 * (splitmix64 of (seed, stream, index)), so the same seed yields the same graph
 * on any machine and with any thread count.
 *
 * Generators (shapes follow SURVEY.md 8(d); the paper's SNAP graphs
 * and Table I at PAPER.md:170-209, are not available):
 *   - Erdos-Renyi G(n, m): m distinct uniform edges.
 *   - R-MAT (a, b, c, d) with 2^scale vertices and `ndraws` edge draws.
 *   - Chung-Lu power law: weights w_i = C (i+1+i0)^(-1/(gamma-1)), w_0 = wmax,
 *     i0 solved so sum(w) = 2m; endpoints drawn proportional to w.
 * All graphs are then: vertex IDs randomly permuted, self-loops dropped,
 * symmetrised, deduplicated, optionally isolated vertices compacted away, and
 * stored as CSR (row_ptr int64[n+1], col_idx int32[2m], each row sorted).
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
  int64_t n;
  int64_t nnz;
  int64_t *row_ptr;
  int32_t *col_idx;
} stmgen_graph;

static inline uint64_t sm64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ULL;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ULL;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBULL;
  return x ^ (x >> 31);
}
static inline uint64_t rnd(uint64_t seed, uint64_t stream, uint64_t i) {
  return sm64(sm64(seed * 0xD1B54A32D192ED03ULL + stream) ^ (i * 0x9E3779B97F4A7C15ULL));
}
static inline double unif(uint64_t seed, uint64_t stream, uint64_t i) {
  return (double)(rnd(seed, stream, i) >> 11) * (1.0 / 9007199254740992.0);
}

/* ---------------- radix sort of u64 keys ---------------- */
static void radix_sort_u64(uint64_t *a, int64_t n, int bits) {
  if (n <= 1) return;
  uint64_t *tmp = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)n);
  uint64_t *src = a, *dst = tmp;
  for (int shift = 0; shift < bits; shift += 11) {
    int64_t cnt[2048];
    memset(cnt, 0, sizeof(cnt));
    for (int64_t i = 0; i < n; ++i) cnt[(src[i] >> shift) & 2047]++;
    if (cnt[(src[0] >> shift) & 2047] == n) continue; /* digit constant: pass is a no-op */
    int64_t s = 0;
    for (int b = 0; b < 2048; ++b) { int64_t c = cnt[b]; cnt[b] = s; s += c; }
    for (int64_t i = 0; i < n; ++i) dst[cnt[(src[i] >> shift) & 2047]++] = src[i];
    uint64_t *t = src; src = dst; dst = t;
  }
  if (src != a) memcpy(a, src, sizeof(uint64_t) * (size_t)n);
  free(tmp);
}

/* random permutation of [0, n) (Fisher-Yates on the counter generator) */
static int64_t *random_perm(int64_t n, uint64_t seed) {
  int64_t *p = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
  for (int64_t i = 0; i < n; ++i) p[i] = i;
  for (int64_t i = n - 1; i > 0; --i) {
    int64_t j = (int64_t)(rnd(seed, 99, (uint64_t)i) % (uint64_t)(i + 1));
    int64_t t = p[i]; p[i] = p[j]; p[j] = t;
  }
  return p;
}

/*
 * Canonicalise an edge list (u[i], v[i]) over [0, n): optional random ID
 * permutation (perm_seed != 0), drop self-loops, symmetrise, dedupe, optional
 * compaction of isolated vertices, emit CSR.  Consumes `keys` (may realloc).
 */
static stmgen_graph *build_csr(int64_t n, uint64_t *keys, int64_t nk, int compact) {
  radix_sort_u64(keys, nk, 64);
  int64_t m = 0;
  for (int64_t i = 0; i < nk; ++i)
    if (m == 0 || keys[i] != keys[m - 1]) keys[m++] = keys[i];
  int64_t *deg = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
  for (int64_t i = 0; i < m; ++i) {
    deg[keys[i] >> 32]++;
    deg[keys[i] & 0xffffffffULL]++;
  }
  int64_t *newid = NULL;
  int64_t n2 = n;
  if (compact) {
    newid = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    n2 = 0;
    for (int64_t i = 0; i < n; ++i) newid[i] = deg[i] ? n2++ : -1;
    int64_t *deg2 = (int64_t *)calloc((size_t)n2 + 1, sizeof(int64_t));
    for (int64_t i = 0; i < n; ++i)
      if (newid[i] >= 0) deg2[newid[i]] = deg[i];
    free(deg);
    deg = deg2;
  }
  stmgen_graph *g = (stmgen_graph *)calloc(1, sizeof(stmgen_graph));
  g->n = n2;
  g->nnz = 2 * m;
  g->row_ptr = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n2 + 1));
  g->col_idx = (int32_t *)malloc(sizeof(int32_t) * (size_t)(2 * m > 0 ? 2 * m : 1));
  g->row_ptr[0] = 0;
  for (int64_t i = 0; i < n2; ++i) g->row_ptr[i + 1] = g->row_ptr[i] + deg[i];
  int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n2 + 1));
  memcpy(fill, g->row_ptr, sizeof(int64_t) * (size_t)(n2 + 1));
  /* keys sorted by (min, max): every row receives its neighbours in
     increasing order (all smaller neighbours first, then larger ones). */
  for (int64_t i = 0; i < m; ++i) {
    int64_t a = (int64_t)(keys[i] >> 32), b = (int64_t)(keys[i] & 0xffffffffULL);
    if (newid) { a = newid[a]; b = newid[b]; }
    g->col_idx[fill[a]++] = (int32_t)b;
    g->col_idx[fill[b]++] = (int32_t)a;
  }
  free(fill);
  free(deg);
  free(newid);
  return g;
}

static inline uint64_t edge_key(int64_t a, int64_t b) {
  return a < b ? ((uint64_t)a << 32) | (uint64_t)b : ((uint64_t)b << 32) | (uint64_t)a;
}

/* ---------------- public API ---------------- */

void stmgen_sizes(const stmgen_graph *g, int64_t *n, int64_t *nnz) {
  *n = g->n;
  *nnz = g->nnz;
}
void stmgen_copy(const stmgen_graph *g, int64_t *row_ptr, int32_t *col_idx) {
  memcpy(row_ptr, g->row_ptr, sizeof(int64_t) * (size_t)(g->n + 1));
  memcpy(col_idx, g->col_idx, sizeof(int32_t) * (size_t)g->nnz);
}
void stmgen_free(stmgen_graph *g) {
  if (!g) return;
  free(g->row_ptr);
  free(g->col_idx);
  free(g);
}

/* Canonicalise a caller-given edge list (used for grids, K_n, unions, ...). */
stmgen_graph *stmgen_from_edges(int64_t n, int64_t m, const int64_t *u, const int64_t *v,
                                uint64_t perm_seed, int compact) {
  int64_t *perm = perm_seed ? random_perm(n, perm_seed) : NULL;
  uint64_t *keys = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(m > 0 ? m : 1));
  int64_t nk = 0;
  for (int64_t i = 0; i < m; ++i) {
    int64_t a = u[i], b = v[i];
    if (a < 0 || b < 0 || a >= n || b >= n || a == b) continue;
    if (perm) { a = perm[a]; b = perm[b]; }
    keys[nk++] = edge_key(a, b);
  }
  stmgen_graph *g = build_csr(n, keys, nk, compact);
  free(keys);
  free(perm);
  return g;
}

/* Erdos-Renyi G(n, m): accept distinct pairs in draw order until m edges. */
stmgen_graph *stmgen_er(int64_t n, int64_t m, uint64_t seed) {
  int64_t maxm = n * (n - 1) / 2;
  if (m > maxm) m = maxm;
  int64_t cap = 1;
  while (cap < 4 * m + 16) cap <<= 1;
  uint64_t *table = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)cap);
  memset(table, 0xff, sizeof(uint64_t) * (size_t)cap);
  uint64_t *keys = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(m > 0 ? m : 1));
  int64_t got = 0;
  for (uint64_t i = 0; got < m; ++i) {
    int64_t a = (int64_t)(rnd(seed, 1, 2 * i) % (uint64_t)n);
    int64_t b = (int64_t)(rnd(seed, 1, 2 * i + 1) % (uint64_t)n);
    if (a == b) continue;
    uint64_t k = edge_key(a, b);
    uint64_t h = sm64(k) & (uint64_t)(cap - 1);
    int dup = 0;
    while (table[h] != ~0ULL) {
      if (table[h] == k) { dup = 1; break; }
      h = (h + 1) & (uint64_t)(cap - 1);
    }
    if (dup) continue;
    table[h] = k;
    keys[got++] = k;
  }
  free(table);
  stmgen_graph *g = build_csr(n, keys, got, 0);
  free(keys);
  return g;
}

typedef struct {
  int scale;
  int64_t lo, hi;
  double a, b, c;
  uint64_t seed;
  const int64_t *perm;
  uint64_t *keys;
} rmat_job;

static void *rmat_worker(void *arg) {
  rmat_job *J = (rmat_job *)arg;
  double ab = J->a + J->b, abc = J->a + J->b + J->c;
  for (int64_t i = J->lo; i < J->hi; ++i) {
    int64_t s = 0, d = 0;
    for (int lvl = 0; lvl < J->scale; ++lvl) {
      double r = unif(J->seed, 2, (uint64_t)i * 64 + (uint64_t)lvl);
      int sb = r >= ab;
      int db = (r >= J->a && r < ab) || r >= abc;
      s = (s << 1) | sb;
      d = (d << 1) | db;
    }
    if (s == d) { J->keys[i] = ~0ULL; continue; }
    J->keys[i] = edge_key(J->perm[s], J->perm[d]);
  }
  return NULL;
}

/* R-MAT: 2^scale vertices, ndraws edge draws, quadrant probabilities a,b,c,(1-a-b-c). */
stmgen_graph *stmgen_rmat(int scale, int64_t ndraws, double a, double b, double c, uint64_t seed,
                          int compact, int nthreads) {
  int64_t n = (int64_t)1 << scale;
  int64_t *perm = random_perm(n, seed ^ 0x5151ULL);
  uint64_t *keys = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(ndraws > 0 ? ndraws : 1));
  if (nthreads < 1) nthreads = 1;
  if (nthreads > 64) nthreads = 64;
  pthread_t th[64];
  rmat_job jobs[64];
  for (int t = 0; t < nthreads; ++t) {
    jobs[t].scale = scale;
    jobs[t].lo = ndraws * t / nthreads;
    jobs[t].hi = ndraws * (t + 1) / nthreads;
    jobs[t].a = a; jobs[t].b = b; jobs[t].c = c;
    jobs[t].seed = seed;
    jobs[t].perm = perm;
    jobs[t].keys = keys;
    pthread_create(&th[t], NULL, rmat_worker, &jobs[t]);
  }
  for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
  int64_t nk = 0;
  for (int64_t i = 0; i < ndraws; ++i)
    if (keys[i] != ~0ULL) keys[nk++] = keys[i];
  stmgen_graph *g = build_csr(n, keys, nk, compact);
  free(keys);
  free(perm);
  return g;
}

/* Chung-Lu power law with w_0 = wmax and sum(w) = 2m; draws ceil(draw_factor*m) edges. */
stmgen_graph *stmgen_chung_lu(int64_t n, int64_t m, double gamma, double wmax, double draw_factor,
                              uint64_t seed, int compact) {
  double beta = 1.0 / (gamma - 1.0);
  double lo = 0.0, hi = 1e12;
  for (int it = 0; it < 200; ++it) {
    double i0 = 0.5 * (lo + hi), s = 0.0;
    for (int64_t i = 0; i < n; ++i) s += wmax * pow((1.0 + i0) / ((double)i + 1.0 + i0), beta);
    if (s < 2.0 * (double)m) lo = i0; else hi = i0;
  }
  double i0 = 0.5 * (lo + hi);
  double *cdf = (double *)malloc(sizeof(double) * (size_t)n);
  double s = 0.0;
  for (int64_t i = 0; i < n; ++i) {
    s += wmax * pow((1.0 + i0) / ((double)i + 1.0 + i0), beta);
    cdf[i] = s;
  }
  int64_t nd = (int64_t)ceil(draw_factor * (double)m);
  int64_t *perm = random_perm(n, seed ^ 0x7373ULL);
  uint64_t *keys = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(nd > 0 ? nd : 1));
  int64_t nk = 0;
  for (int64_t e = 0; e < nd; ++e) {
    int64_t ends[2];
    for (int side = 0; side < 2; ++side) {
      double r = unif(seed, 3, 2 * (uint64_t)e + (uint64_t)side) * s;
      int64_t L = 0, H = n - 1;
      while (L < H) {
        int64_t M = (L + H) >> 1;
        if (cdf[M] > r) H = M; else L = M + 1;
      }
      ends[side] = L;
    }
    if (ends[0] == ends[1]) continue;
    keys[nk++] = edge_key(perm[ends[0]], perm[ends[1]]);
  }
  free(cdf);
  free(perm);
  stmgen_graph *g = build_csr(n, keys, nk, compact);
  free(keys);
  return g;
}

/* i.i.d. uniform vertex labels in [0, nlabels). */
void stmgen_labels(int64_t n, int32_t nlabels, uint64_t seed, int32_t *out) {
  for (int64_t i = 0; i < n; ++i)
    out[i] = (int32_t)(rnd(seed, 4, (uint64_t)i) % (uint64_t)nlabels);
}
