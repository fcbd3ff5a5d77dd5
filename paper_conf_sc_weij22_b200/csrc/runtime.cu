// runtime.cu -- C ABI of libstm.so: graph residency, scratch sizing, launch,
// read-back.  Product code (never calls the oracle).
#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <tuple>
#include <mutex>
#include <new>
#include <thread>
#include <vector>

#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_segmented_sort.cuh>
#include <cuda_runtime.h>

#include "internal.h"
#include "kernel.h"

// Hub bitmap defaults (stm_tuning 0 = auto): measured on B200, DESIGN.md "Hub bitmaps".
#define STM_BITMAP_AUTO_MIN_DEGREE 64
#define STM_BITMAP_AUTO_BUDGET_MB 512   // (C5 K6-e: 2048 MB -> 512 MB same time, DRAM 54 -> 28 GB per launch)
#define STM_L2_PERSIST_AUTO_MB 0   // measured neutral at 24-48 MiB, worse at 96 MiB on C5: off
#define STM_CHUNK_COST_AUTO 512    // work-balanced root chunks (stm_tuning.chunk_cost)
#define STM_ROOT_SPLIT_AUTO 512    // root splitting piece size (stm_tuning.root_split; measured 32..512 on C2-C5)

static thread_local char g_err[1024] = "";
static thread_local stm_launch_info g_info = {};
static thread_local uint64_t g_prof[STM_PROF_SIZE] = {};

stm_status stm_fail(stm_status s, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof g_err, fmt, ap);
  va_end(ap);
  return s;
}

extern "C" const char* stm_last_error(void) { return g_err; }

#define CU(call)                                                                         \
  do {                                                                                   \
    cudaError_t e_ = (call);                                                             \
    if (e_ != cudaSuccess) return stm_fail(STM_ECUDA, "%s: %s", #call, cudaGetErrorString(e_)); \
  } while (0)

namespace {
struct Scratch {
  int* arena = nullptr;
  size_t arena_bytes = 0;
  void* state = nullptr;  // StmWork + cursor + StmPoolSlot[pool capacity]
  size_t state_bytes = 0;
};

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};
}  // namespace

struct stm_graph {
  int device = 0;
  int64_t n = 0, nnz = 0, max_degree = 0;
  // Directed graphs (stm_graph_load_directed; NEXT-4): the CSR holds 2n rows, vertex v's
  // out-row at row v and its in-row at row n + v (kernel StmKParams::n_dir).  No degree-
  // ranked copy, hub bitmaps or root splitting for them (speed-only features).
  bool directed = false;
  int64_t n_rows = 0;
  int64_t* d_row_ptr = nullptr;
  int32_t* d_col_idx = nullptr;
  uint8_t* d_labels = nullptr;
  bool owns_csr = true;
  std::vector<int32_t> label_values;  // dense id -> label value
  int num_sms = 0;
  int l2_bytes = 0;
  int64_t max_window = 0, persist_max = 0;  // cudaDevAttrMaxAccessPolicyWindowSize / MaxPersistingL2CacheSize
  int64_t persist_set = 0;                  // persisting L2 set-aside this library last requested
  // Degree-ranked copy: vertex i of
  // the copy is the i-th vertex in (degree, id) order.  Plans whose restrictions
  // are order-free (STM_AUTO_RESTRICT or none) count on it; the count is the same
  // (any total order breaks symmetry), the work far smaller on skewed graphs.
  bool ranked = false;
  int64_t* d_rrow_ptr = nullptr;
  int32_t* d_rcol_idx = nullptr;
  uint8_t* d_rlabels = nullptr;
  int32_t* d_rank2orig = nullptr;  // [n]: ranked id -> caller's id (per-root output)
  // out_start[v] = index in N(v) of the first neighbour > v, per numbering (NULL if
  // it could not be built; then the kernel narrows by binary search alone)
  int32_t* d_out_start = nullptr;
  int32_t* d_rout_start = nullptr;
  // Hub adjacency bitmaps per (numbering, min degree, budget), built lazily by the
  // first launch that asks for them and kept until the
  // graph is freed: a launch on another stream may still read a set another call no
  // longer wants, so no set is ever freed or rebuilt while the graph is alive.
  struct HubBitmaps {
    int32_t* slot = nullptr;   // [n]: bitmap slot of v, -1 = none
    uint32_t* bits = nullptr;  // [n_hubs][words]
    int64_t words = 0, n_hubs = 0;
    int4* vrec = nullptr;      // [n] packed (row start, degree, out_start, hub slot) for this set
  };
  std::map<std::tuple<int, int, int64_t>, HubBitmaps> hubs;  // (ranked, min_deg, budget) -> set
  std::mutex mu;
  // root entries per (numbering, piece size) (kernel.h StmKParams::entries), built lazily
  struct RootEntries {
    int2* d = nullptr;
    int64_t n = 0;
  };
  std::map<std::pair<int, int>, RootEntries> entries;
  // work-balanced chunk bounds per (numbering, piece size or -1 = vertex ids, chunk cost)
  struct ChunkBounds {
    int32_t* d = nullptr;
    int64_t n = 0;  // chunks (d has n + 1 entries)
  };
  std::map<std::tuple<int, int, int>, ChunkBounds> chunks;
  // degree / label statistics of the graph (NEXT-2 cost model), computed at load
  bool has_stats = false;
  stm_graph_stats stats;
};

// ---------------------------------------------------------------------------- load
// max degree and monotonicity of a device row_ptr (out[0] = max degree, out[1] = bad flag)
__global__ void degree_scan(const int64_t* rp, int64_t n, long long* out) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    long long d = rp[v + 1] - rp[v];
    if (d < 0) out[1] = 1;
    else atomicMax(&out[0], d);
  }
}

// Full CSR validation on the device (stm_graph_load): one thread per adjacency entry checks
// the id range, no self-loop, strict increase within the row and (symmetric graphs) that
// the reverse entry exists (binary search in the neighbour's row).  bad[r] = the smallest
// offending vertex for reason r (1 range, 2 self-loop, 3 order, 4 symmetry); INT64_MAX = none.
__global__ void validate_entries(const int64_t* rp, const int32_t* ci, int64_t n, int symmetric,
                                 unsigned long long* bad) {
  const int64_t nnz = rp[n];
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x) {
    // the row of entry e: binary search in row_ptr
    int64_t lo = 0, hi = n;
    while (hi - lo > 1) {
      const int64_t mid = (lo + hi) >> 1;
      if (rp[mid] <= e) lo = mid; else hi = mid;
    }
    const int64_t v = lo;
    const int64_t w = ci[e];
    int why = 0;
    if (w < 0 || w >= n) why = 1;
    else if (w == v) why = 2;
    else if (e > rp[v] && ci[e - 1] >= w) why = 3;
    else if (symmetric) {
      int64_t a = rp[w], b = rp[w + 1];
      while (a < b) {
        const int64_t mid = (a + b) >> 1;
        if (ci[mid] < v) a = mid + 1; else b = mid;
      }
      if (a == rp[w + 1] || ci[a] != v) why = 4;
    }
    if (why) atomicMin(&bad[why], (unsigned long long)v);
  }
}

static stm_status validate_on_device(const int64_t* d_rp, const int32_t* d_ci, int64_t n, int64_t nnz,
                                     bool symmetric) {
  if (nnz == 0) return STM_OK;
  unsigned long long* d = nullptr;
  CU(cudaMalloc(&d, 5 * sizeof(unsigned long long)));
  unsigned long long h[5];
  for (auto& x : h) x = ~0ull;
  cudaError_t e = cudaMemcpy(d, h, sizeof h, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) {
    validate_entries<<<(unsigned)std::min<int64_t>((nnz + 255) / 256, 8192), 256>>>(d_rp, d_ci, n, symmetric ? 1 : 0, d);
    e = cudaGetLastError();
  }
  if (e == cudaSuccess) e = cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
  cudaFree(d);
  if (e != cudaSuccess) return stm_fail(STM_ECUDA, "CSR validation: %s", cudaGetErrorString(e));
  static const char* why[] = {"", "neighbour id out of range", "self-loop", "row not strictly increasing",
                              "graph not symmetric"};
  for (int r = 1; r < 5; ++r)
    if (h[r] != ~0ull) return stm_fail(STM_EINVAL, "%s at vertex %lld", why[r], (long long)h[r]);
  return STM_OK;
}

// ---------------------------------------------------------------- degree-ranked copy
__global__ void rank_keys(const int64_t* rp, int64_t n, unsigned long long* keys) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    keys[v] = ((unsigned long long)(rp[v + 1] - rp[v]) << 32) | (unsigned long long)v;
}
__global__ void rank_scatter(const unsigned long long* sorted, int64_t n, int32_t* rank2orig, int32_t* orig2rank,
                             int64_t* newdeg, const uint8_t* lab, uint8_t* rlab) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = (int32_t)(sorted[i] & 0xffffffffull);
    rank2orig[i] = v;
    orig2rank[v] = (int32_t)i;
    newdeg[i] = (int64_t)(sorted[i] >> 32);
    if (lab) rlab[i] = lab[v];
  }
}
// one warp per ranked row: the caller's row of rank2orig[i], renumbered (unsorted)
__global__ void rank_fill(const int64_t* rp, const int32_t* ci, const int32_t* rank2orig, const int32_t* orig2rank,
                          const int64_t* rrp, int32_t* out, int64_t n) {
  const int lane = threadIdx.x & 31;
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; i < n;
       i += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const int32_t v = rank2orig[i];
    const int64_t b = rp[v], d = rp[v + 1] - b, o = rrp[i];
    for (int64_t j = lane; j < d; j += 32) out[o + j] = orig2rank[ci[b + j]];
  }
}

// Builds g's degree-ranked copy on the device (load time, not the query).  Only
// speed depends on it: when it cannot be built (sizes beyond CUB's int range, no
// memory) `ranked` stays false and every plan counts on the caller's numbering.
static void build_ranked(stm_graph* g) {
  const int64_t n = g->n, nnz = g->nnz;
  if (n < 2 || nnz < 1 || nnz > INT32_MAX) return;
  unsigned long long *keys = nullptr, *skeys = nullptr;
  int32_t* orig2rank = nullptr;
  int32_t* tmpcol = nullptr;
  void* temp = nullptr;
  size_t t1 = 0, t2 = 0, t3 = 0;
  cudaError_t e = cudaSuccess;
  auto ok = [&](cudaError_t x) { if (e == cudaSuccess) e = x; return e == cudaSuccess; };
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, 8 * 1024);
  ok(cudaMalloc(&keys, sizeof(unsigned long long) * n));
  ok(cudaMalloc(&skeys, sizeof(unsigned long long) * n));
  ok(cudaMalloc(&orig2rank, sizeof(int32_t) * n));
  ok(cudaMalloc(&g->d_rank2orig, sizeof(int32_t) * n));
  ok(cudaMalloc(&g->d_rrow_ptr, sizeof(int64_t) * (n + 1)));
  ok(cudaMalloc(&g->d_rcol_idx, sizeof(int32_t) * nnz));
  ok(cudaMalloc(&tmpcol, sizeof(int32_t) * nnz));
  if (g->d_labels) ok(cudaMalloc(&g->d_rlabels, n));
  if (e == cudaSuccess) {
    int end_bit = 33;
    while (end_bit < 64 && (g->max_degree >> (end_bit - 32)) != 0) ++end_bit;
    ok(cub::DeviceRadixSort::SortKeys(nullptr, t1, keys, skeys, (int)n, 0, end_bit));
    ok(cub::DeviceScan::ExclusiveSum(nullptr, t2, g->d_rrow_ptr, g->d_rrow_ptr, (int)(n + 1)));
    ok(cub::DeviceSegmentedSort::SortKeys(nullptr, t3, tmpcol, g->d_rcol_idx, (int)nnz, (int)n, g->d_rrow_ptr,
                                          g->d_rrow_ptr + 1));
    ok(cudaMalloc(&temp, std::max<size_t>(std::max(t1, std::max(t2, t3)), 16)));
    if (e == cudaSuccess) {
      rank_keys<<<grid, 256>>>(g->d_row_ptr, n, keys);
      ok(cub::DeviceRadixSort::SortKeys(temp, t1, keys, skeys, (int)n, 0, end_bit));
      ok(cudaMemset(g->d_rrow_ptr + n, 0, sizeof(int64_t)));
      rank_scatter<<<grid, 256>>>(skeys, n, g->d_rank2orig, orig2rank, g->d_rrow_ptr, g->d_labels, g->d_rlabels);
      ok(cub::DeviceScan::ExclusiveSum(temp, t2, g->d_rrow_ptr, g->d_rrow_ptr, (int)(n + 1)));
      rank_fill<<<grid, 256>>>(g->d_row_ptr, g->d_col_idx, g->d_rank2orig, orig2rank, g->d_rrow_ptr, tmpcol, n);
      ok(cub::DeviceSegmentedSort::SortKeys(temp, t3, tmpcol, g->d_rcol_idx, (int)nnz, (int)n, g->d_rrow_ptr,
                                            g->d_rrow_ptr + 1));
      ok(cudaGetLastError());
      ok(cudaDeviceSynchronize());
    }
  }
  cudaFree(keys);
  cudaFree(skeys);
  cudaFree(orig2rank);
  cudaFree(tmpcol);
  cudaFree(temp);
  if (e == cudaSuccess) {
    g->ranked = true;
    return;
  }
  cudaGetLastError();  // clear the non-sticky error (e.g. out of memory)
  cudaFree(g->d_rank2orig);
  cudaFree(g->d_rrow_ptr);
  cudaFree(g->d_rcol_idx);
  cudaFree(g->d_rlabels);
  g->d_rank2orig = nullptr;
  g->d_rrow_ptr = nullptr;
  g->d_rcol_idx = nullptr;
  g->d_rlabels = nullptr;
}

static void query_persist(stm_graph* g) {
  int a = 0, b = 0;
  if (cudaDeviceGetAttribute(&a, cudaDevAttrMaxAccessPolicyWindowSize, g->device) != cudaSuccess) a = 0;
  if (cudaDeviceGetAttribute(&b, cudaDevAttrMaxPersistingL2CacheSize, g->device) != cudaSuccess) b = 0;
  cudaGetLastError();
  g->max_window = a;
  g->persist_max = b;
}

// ---------------------------------------------------------------- out_start
// per row: index of the first entry > the row's vertex (row r is vertex r, or r - nv for
// the in-rows of a directed graph)
__global__ void out_start_fill(const int64_t* rp, const int32_t* ci, int64_t n, int64_t nv, int32_t* out) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t x = v < nv ? v : v - nv;
    int64_t lo = rp[v], hi = rp[v + 1];
    const int64_t b = lo;
    while (lo < hi) {
      const int64_t mid = (lo + hi) >> 1;
      if (ci[mid] <= x) lo = mid + 1; else hi = mid;
    }
    out[v] = (int32_t)(lo - b);
  }
}

static int32_t* build_out_start(const int64_t* rp, const int32_t* ci, int64_t n, int64_t nv) {
  int32_t* d = nullptr;
  if (n < 1 || cudaMalloc(&d, sizeof(int32_t) * n) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  out_start_fill<<<(unsigned)std::min<int64_t>((n + 255) / 256, 8192), 256>>>(rp, ci, n, nv, d);
  if (cudaGetLastError() != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess) {
    cudaGetLastError();
    cudaFree(d);
    return nullptr;
  }
  return d;
}

// ---------------------------------------------------------------- hub bitmaps
__global__ void count_deg_ge(const int64_t* rp, int64_t n, int64_t min_deg, unsigned long long* out) {
  unsigned long long c = 0;
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    c += (rp[v + 1] - rp[v]) >= min_deg;
  if (c) atomicAdd(out, c);
}
// hub i is the vertex of ranked id n - H + i (the H highest in (degree, id) order)
__global__ void hub_slots(int64_t n, int64_t H, const int32_t* rank2orig, int32_t* slot) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < H; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = n - H + i;
    slot[rank2orig ? rank2orig[r] : r] = (int32_t)i;
  }
}
// one block per hub: set the bits of its neighbour list
__global__ void hub_fill(int64_t n, int64_t H, const int32_t* rank2orig, const int64_t* rp, const int32_t* ci,
                         int64_t words, uint32_t* bits) {
  for (int64_t i = blockIdx.x; i < H; i += gridDim.x) {
    const int64_t r = n - H + i;
    const int32_t v = rank2orig ? rank2orig[r] : (int32_t)r;
    uint32_t* b = bits + (size_t)i * (size_t)words;
    for (int64_t e = rp[v] + threadIdx.x; e < rp[v + 1]; e += blockDim.x) {
      const int32_t x = ci[e];
      atomicOr(&b[x >> 5], 1u << (x & 31));
    }
  }
}

// ---------------------------------------------------------------- root entries
__global__ void entry_counts(const int64_t* rp, int64_t n, int T, int64_t* cnt) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t d = rp[v + 1] - rp[v];
    cnt[v] = d > T ? (d + T - 1) / T : 1;
  }
}
__global__ void entry_fill(const int64_t* off, int64_t n, int2* out) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    for (int64_t c = 0; c < off[v + 1] - off[v]; ++c) out[off[v] + c] = make_int2((int)v, (int)c);
}

// Entries (v, piece) in vertex order for the numbering `ranked`; caller holds g->mu.
// NULL (no splitting) on any failure -- speed only.
static const stm_graph::RootEntries* ensure_entries(stm_graph* g, bool ranked, int T) {
  const auto key = std::make_pair(ranked ? 1 : 0, T);
  auto it = g->entries.find(key);
  if (it != g->entries.end()) return it->second.d ? &it->second : nullptr;
  stm_graph::RootEntries& E = g->entries[key];
  const int64_t n = g->n;
  if (n < 1 || T < 1) return nullptr;
  const int64_t* rp = ranked ? g->d_rrow_ptr : g->d_row_ptr;
  int64_t* off = nullptr;
  void* temp = nullptr;
  size_t tb = 0;
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, 4096);
  cudaError_t e = cudaMalloc(&off, sizeof(int64_t) * (n + 1));
  if (e == cudaSuccess) {
    entry_counts<<<grid, 256>>>(rp, n, T, off);
    e = cudaMemset(off + n, 0, sizeof(int64_t));
  }
  if (e == cudaSuccess) e = cub::DeviceScan::ExclusiveSum(nullptr, tb, off, off, (int)(n + 1));
  if (e == cudaSuccess) e = cudaMalloc(&temp, std::max<size_t>(tb, 16));
  if (e == cudaSuccess) e = cub::DeviceScan::ExclusiveSum(temp, tb, off, off, (int)(n + 1));
  int64_t total = 0;
  if (e == cudaSuccess) e = cudaMemcpy(&total, off + n, sizeof total, cudaMemcpyDeviceToHost);
  if (e == cudaSuccess && total < INT32_MAX) {
    e = cudaMalloc(&E.d, sizeof(int2) * (size_t)total);
    if (e == cudaSuccess) {
      entry_fill<<<grid, 256>>>(off, n, E.d);
      e = cudaGetLastError();
      if (e == cudaSuccess) e = cudaDeviceSynchronize();
    }
  }
  cudaFree(off);
  cudaFree(temp);
  if (e != cudaSuccess || total >= INT32_MAX || !E.d) {
    cudaGetLastError();
    cudaFree(E.d);
    E.d = nullptr;
    return nullptr;
  }
  E.n = total;
  return &E;
}

// estimated cost of root-space position e: 1 + its level-1 candidate-list length (the
// piece of its root's neighbour list when entries are used)
__global__ void chunk_cost_fill(const int64_t* rp, const int2* ent, int64_t ne, int T, int64_t* cost) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < ne; e += (int64_t)gridDim.x * blockDim.x) {
    const int v = ent ? ent[e].x : (int)e;
    const int64_t d = rp[v + 1] - rp[v];
    const int64_t len = ent ? min((int64_t)T, d - (int64_t)ent[e].y * T) : d;
    cost[e] = 1 + max(len, (int64_t)0);
  }
}
// position e starts a chunk iff its exclusive cost prefix lies in another multiple of C than e-1's
__global__ void chunk_flag_fill(const int64_t* pre, int64_t ne, int64_t C, int32_t* flag) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < ne; e += (int64_t)gridDim.x * blockDim.x)
    flag[e] = (e == 0 || pre[e] / C != pre[e - 1] / C) ? 1 : 0;
}
__global__ void chunk_scatter(const int32_t* flag, const int32_t* pos, int64_t ne, int32_t* out) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < ne; e += (int64_t)gridDim.x * blockDim.x)
    if (flag[e]) out[pos[e]] = (int32_t)e;
}

// Chunk bounds over the root space [0, ne) (entries E or vertex ids): consecutive positions
// grouped until their cost reaches C.  Caller holds g->mu.  NULL on any failure (speed only:
// the launch then uses fixed chunks).
static const stm_graph::ChunkBounds* ensure_chunks(stm_graph* g, bool ranked, const stm_graph::RootEntries* E,
                                                   int T, int C) {
  const auto key = std::make_tuple(ranked ? 1 : 0, E ? T : -1, C);
  auto it = g->chunks.find(key);
  if (it != g->chunks.end()) return it->second.d ? &it->second : nullptr;
  stm_graph::ChunkBounds& B = g->chunks[key];
  const int64_t ne = E ? E->n : g->n;
  if (ne < 1 || ne >= INT32_MAX || C < 1) return nullptr;
  const int64_t* rp = ranked ? g->d_rrow_ptr : g->d_row_ptr;
  int64_t* cost = nullptr;
  int32_t *flag = nullptr, *pos = nullptr;
  void* temp = nullptr;
  size_t tb = 0, tb2 = 0;
  const unsigned grid = (unsigned)std::min<int64_t>((ne + 255) / 256, 4096);
  cudaError_t e = cudaMalloc(&cost, sizeof(int64_t) * ne);
  if (e == cudaSuccess) e = cudaMalloc(&flag, sizeof(int32_t) * ne);
  if (e == cudaSuccess) e = cudaMalloc(&pos, sizeof(int32_t) * ne);
  if (e == cudaSuccess) e = cub::DeviceScan::ExclusiveSum(nullptr, tb, cost, cost, (int)ne);
  if (e == cudaSuccess) e = cub::DeviceScan::ExclusiveSum(nullptr, tb2, flag, pos, (int)ne);
  if (e == cudaSuccess) e = cudaMalloc(&temp, std::max<size_t>(std::max(tb, tb2), 16));
  if (e == cudaSuccess) {
    chunk_cost_fill<<<grid, 256>>>(rp, E ? E->d : nullptr, ne, T, cost);
    e = cub::DeviceScan::ExclusiveSum(temp, tb, cost, cost, (int)ne);
  }
  if (e == cudaSuccess) {
    chunk_flag_fill<<<grid, 256>>>(cost, ne, (int64_t)C, flag);
    e = cub::DeviceScan::ExclusiveSum(temp, tb2, flag, pos, (int)ne);
  }
  int32_t last[2] = {0, 0};
  if (e == cudaSuccess) e = cudaMemcpy(&last[0], pos + ne - 1, sizeof(int32_t), cudaMemcpyDeviceToHost);
  if (e == cudaSuccess) e = cudaMemcpy(&last[1], flag + ne - 1, sizeof(int32_t), cudaMemcpyDeviceToHost);
  const int64_t nc = (int64_t)last[0] + last[1];
  if (e == cudaSuccess) e = cudaMalloc(&B.d, sizeof(int32_t) * (nc + 1));
  if (e == cudaSuccess) {
    chunk_scatter<<<grid, 256>>>(flag, pos, ne, B.d);
    const int32_t end = (int32_t)ne;
    e = cudaMemcpy(B.d + nc, &end, sizeof end, cudaMemcpyHostToDevice);
  }
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  cudaFree(cost);
  cudaFree(flag);
  cudaFree(pos);
  cudaFree(temp);
  if (e != cudaSuccess) {
    cudaGetLastError();
    cudaFree(B.d);
    B.d = nullptr;
    return nullptr;
  }
  B.n = nc;
  return &B;
}

static void free_hub(stm_graph::HubBitmaps& h) {
  cudaFree(h.slot);
  cudaFree(h.bits);
  cudaFree(h.vrec);
  h = stm_graph::HubBitmaps();
}

// packed per-vertex records of one numbering and hub set (kernel.cu vrec())
__global__ void vrec_fill(const int64_t* rp, int64_t n, const int32_t* out_start, const int32_t* slot, int4* out) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = rp[v];
    out[v] = make_int4((int)(uint32_t)b, (int)(rp[v + 1] - b), out_start ? out_start[v] : -1, slot ? slot[v] : -1);
  }
}

// The launch-side view of a graph for one numbering (`ranked`) and hub set: hub
// bitmaps of every vertex with degree >= min_deg (at most budget bytes, highest
// degrees first; min_deg < 0: none) and the packed vertex records that point into
// them.  Caller holds g->mu.  Built once per key and kept until the graph is freed.
// Returns NULL only if the records cannot be built (the bitmaps are speed only: on
// failure the set simply has none).
static const stm_graph::HubBitmaps* ensure_hub(stm_graph* g, bool ranked, int min_deg, int64_t budget) {
  if (min_deg < 0 || !g->ranked) { min_deg = -1; budget = 0; }
  const auto key = std::make_tuple(ranked ? 1 : 0, min_deg, budget);
  auto it = g->hubs.find(key);
  if (it != g->hubs.end()) return it->second.vrec ? &it->second : nullptr;
  stm_graph::HubBitmaps& h = g->hubs[key];
  const int64_t n = g->n;
  const int64_t* rp = ranked ? g->d_rrow_ptr : g->d_row_ptr;
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, 4096);
  cudaError_t e = cudaSuccess;
  if (min_deg >= 0 && n > 0) {
    const int64_t words = (n + 31) / 32;
    const int64_t hmax = budget / (words * 4);
    unsigned long long* d = nullptr;
    unsigned long long H = 0;
    e = cudaMalloc(&d, sizeof H);
    if (e == cudaSuccess) e = cudaMemset(d, 0, sizeof H);
    if (e == cudaSuccess) count_deg_ge<<<grid, 256>>>(g->d_rrow_ptr, n, std::max(min_deg, 1), d);
    if (e == cudaSuccess) e = cudaMemcpy(&H, d, sizeof H, cudaMemcpyDeviceToHost);
    cudaFree(d);
    H = std::min<unsigned long long>(H, (unsigned long long)std::max<int64_t>(hmax, 0));
    if (e == cudaSuccess && H > 0) {
      e = cudaMalloc(&h.slot, sizeof(int32_t) * n);
      if (e == cudaSuccess) e = cudaMalloc(&h.bits, sizeof(uint32_t) * (size_t)words * H);
      if (e == cudaSuccess) e = cudaMemset(h.slot, 0xFF, sizeof(int32_t) * n);
      if (e == cudaSuccess) e = cudaMemset(h.bits, 0, sizeof(uint32_t) * (size_t)words * H);
      if (e == cudaSuccess) {
        const int32_t* r2o = ranked ? nullptr : g->d_rank2orig;
        hub_slots<<<(unsigned)std::min<unsigned long long>((H + 255) / 256, 4096), 256>>>(n, (int64_t)H, r2o, h.slot);
        hub_fill<<<(unsigned)std::min<unsigned long long>(H, 65535), 256>>>(
            n, (int64_t)H, r2o, rp, ranked ? g->d_rcol_idx : g->d_col_idx, words, h.bits);
        e = cudaGetLastError();
        if (e == cudaSuccess) e = cudaDeviceSynchronize();
      }
      if (e == cudaSuccess) {
        h.words = words;
        h.n_hubs = (int64_t)H;
      }
    }
    if (e != cudaSuccess) {  // no bitmaps (speed only)
      cudaGetLastError();
      cudaFree(h.slot);
      cudaFree(h.bits);
      h.slot = nullptr;
      h.bits = nullptr;
      h.n_hubs = h.words = 0;
    }
  }
  // one record per CSR row (directed graphs: out-rows then in-rows; no bitmaps there)
  const int64_t nr = g->n_rows;
  e = cudaMalloc(&h.vrec, sizeof(int4) * (size_t)std::max<int64_t>(nr, 1));
  if (e == cudaSuccess && nr > 0) {
    vrec_fill<<<(unsigned)std::min<int64_t>((nr + 255) / 256, 4096), 256>>>(
        rp, nr, ranked ? g->d_rout_start : g->d_out_start, g->directed ? nullptr : h.slot, h.vrec);
    e = cudaGetLastError();
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
  }
  if (e != cudaSuccess) {
    cudaGetLastError();
    cudaFree(h.vrec);
    h.vrec = nullptr;
    return nullptr;
  }
  return &h;
}

static stm_status validate_csr(int64_t n, const int64_t* rp, const int32_t* ci, bool symmetric) {
  if (rp[0] != 0) return stm_fail(STM_EINVAL, "row_ptr[0] != 0");
  for (int64_t v = 0; v < n; ++v)
    if (rp[v + 1] < rp[v]) return stm_fail(STM_EINVAL, "row_ptr decreases at %lld", (long long)v);
  unsigned nt = std::max(1u, std::min(32u, std::thread::hardware_concurrency()));
  std::vector<int> bad(nt, 0);
  std::vector<int64_t> badv(nt, -1);
  std::vector<std::thread> th;
  for (unsigned t = 0; t < nt; ++t)
    th.emplace_back([&, t] {
      int64_t lo = n * t / nt, hi = n * (t + 1) / nt;
      for (int64_t v = lo; v < hi && !bad[t]; ++v) {
        for (int64_t e = rp[v]; e < rp[v + 1]; ++e) {
          int64_t w = ci[e];
          if (w < 0 || w >= n) { bad[t] = 1; badv[t] = v; break; }
          if (w == v) { bad[t] = 2; badv[t] = v; break; }
          if (e > rp[v] && ci[e - 1] >= w) { bad[t] = 3; badv[t] = v; break; }
          if (!symmetric) continue;
          // symmetry: v must be in N(w)
          const int32_t* b = ci + rp[w];
          const int32_t* x = std::lower_bound(b, ci + rp[w + 1], (int32_t)v);
          if (x == ci + rp[w + 1] || *x != v) { bad[t] = 4; badv[t] = v; break; }
        }
      }
    });
  for (auto& x : th) x.join();
  static const char* why[] = {"", "neighbour id out of range", "self-loop", "row not strictly increasing",
                              "graph not symmetric"};
  for (unsigned t = 0; t < nt; ++t)
    if (bad[t]) return stm_fail(STM_EINVAL, "%s at vertex %lld", why[bad[t]], (long long)badv[t]);
  return STM_OK;
}

static stm_status dense_labels(int64_t n, const int32_t* labels, std::vector<uint8_t>& dense,
                               std::vector<int32_t>& values) {
  values.assign(labels, labels + n);
  std::sort(values.begin(), values.end());
  values.erase(std::unique(values.begin(), values.end()), values.end());
  if (!values.empty() && values[0] < 0) return stm_fail(STM_EINVAL, "negative vertex label %d", values[0]);
  if (values.size() > 255)
    return stm_fail(STM_EUNSUPPORTED, "%zu distinct vertex labels > 255", values.size());
  dense.resize(n);
  for (int64_t v = 0; v < n; ++v)
    dense[v] = (uint8_t)(std::lower_bound(values.begin(), values.end(), labels[v]) - values.begin());
  return STM_OK;
}

// Upload a validated CSR of n_rows rows over n vertices (n_rows = 2n for a directed graph:
// out-rows then in-rows) and build the per-graph structures.
static stm_status upload_graph(int64_t n, int64_t n_rows, const int64_t* row_ptr, const int32_t* col_idx,
                               const int32_t* labels, int device, bool directed, stm_graph** out,
                               bool validate_symmetric = false) {
  const int64_t nnz = row_ptr[n_rows];
  std::vector<uint8_t> dense;
  std::vector<int32_t> values;
  if (labels) {
    stm_status s = dense_labels(n, labels, dense, values);
    if (s != STM_OK) return s;
  }
  int64_t maxd = 0;
  for (int64_t v = 0; v < n_rows; ++v) maxd = std::max(maxd, row_ptr[v + 1] - row_ptr[v]);
  int ndev = 0;
  CU(cudaGetDeviceCount(&ndev));
  if (device < 0 || device >= ndev) return stm_fail(STM_EINVAL, "device %d of %d", device, ndev);
  DeviceGuard dg(device);
  stm_graph* g = new (std::nothrow) stm_graph();
  if (!g) return stm_fail(STM_ENOMEM, "host allocation");
  g->device = device;
  g->n = n;
  g->n_rows = n_rows;
  g->directed = directed;
  g->nnz = nnz;
  g->max_degree = maxd;
  g->label_values = values;
  cudaError_t e = cudaMalloc(&g->d_row_ptr, sizeof(int64_t) * (n_rows + 1));
  if (e == cudaSuccess) e = cudaMalloc(&g->d_col_idx, sizeof(int32_t) * std::max<int64_t>(nnz, 1));
  if (e == cudaSuccess && labels) e = cudaMalloc(&g->d_labels, std::max<int64_t>(n, 1));
  if (e == cudaSuccess) e = cudaMemcpy(g->d_row_ptr, row_ptr, sizeof(int64_t) * (n_rows + 1), cudaMemcpyHostToDevice);
  if (e == cudaSuccess && nnz) e = cudaMemcpy(g->d_col_idx, col_idx, sizeof(int32_t) * nnz, cudaMemcpyHostToDevice);
  if (e == cudaSuccess && labels && n) e = cudaMemcpy(g->d_labels, dense.data(), n, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&g->num_sms, cudaDevAttrMultiProcessorCount, device);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&g->l2_bytes, cudaDevAttrL2CacheSize, device);
  query_persist(g);
  if (e != cudaSuccess) {
    stm_graph_free(g);
    return stm_fail(e == cudaErrorMemoryAllocation ? STM_ENOMEM : STM_ECUDA, "graph upload: %s",
                    cudaGetErrorString(e));
  }
  if (validate_symmetric) {  // the entry checks of stm_graph_load, on the uploaded copy
    const stm_status vs = validate_on_device(g->d_row_ptr, g->d_col_idx, n, nnz, true);
    if (vs != STM_OK) {
      stm_graph_free(g);
      return vs;
    }
  }
  if (!directed) {
    g->has_stats = stm_graph_stats_host(n, row_ptr, labels, &g->stats) == STM_OK;
    build_ranked(g);
  }
  g->d_out_start = build_out_start(g->d_row_ptr, g->d_col_idx, g->n_rows, g->n);
  if (g->ranked) g->d_rout_start = build_out_start(g->d_rrow_ptr, g->d_rcol_idx, g->n, g->n);
  *out = g;
  return STM_OK;
}

extern "C" stm_status stm_graph_load(int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                                     const int32_t* labels, int device, stm_graph** out) {
  if (!out) return stm_fail(STM_EINVAL, "out is NULL");
  if (n < 0 || n > INT32_MAX - 1) return stm_fail(STM_EINVAL, "n=%lld out of range", (long long)n);
  if (!row_ptr) return stm_fail(STM_EINVAL, "row_ptr is NULL");
  int64_t nnz = row_ptr[n];
  if (nnz > 0 && !col_idx) return stm_fail(STM_EINVAL, "col_idx is NULL");
  if (nnz > (int64_t)UINT32_MAX)  // packed vertex records hold 32-bit row starts (kernel.cu vrec)
    return stm_fail(STM_EUNSUPPORTED, "%lld adjacency entries >= 2^32", (long long)nnz);
  // row_ptr checks on the host (O(n)); the O(m log d) entry checks (range, self-loops, order,
  // symmetry) on the device after the upload -- the same checks and messages as validate_csr
  if (row_ptr[0] != 0) return stm_fail(STM_EINVAL, "row_ptr[0] != 0");
  for (int64_t v = 0; v < n; ++v)
    if (row_ptr[v + 1] < row_ptr[v]) return stm_fail(STM_EINVAL, "row_ptr decreases at %lld", (long long)v);
  return upload_graph(n, n, row_ptr, col_idx, labels, device, false, out, true);
}

extern "C" stm_status stm_graph_load_directed(int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                                              const int32_t* labels, int device, stm_graph** out) {
  if (!out) return stm_fail(STM_EINVAL, "out is NULL");
  if (n < 0 || n > INT32_MAX - 1) return stm_fail(STM_EINVAL, "n=%lld out of range", (long long)n);
  if (!row_ptr) return stm_fail(STM_EINVAL, "row_ptr is NULL");
  const int64_t m = row_ptr[n];
  if (m > 0 && !col_idx) return stm_fail(STM_EINVAL, "col_idx is NULL");
  if (2 * m > (int64_t)UINT32_MAX) return stm_fail(STM_EUNSUPPORTED, "%lld arcs: 2m >= 2^32", (long long)m);
  stm_status s = validate_csr(n, row_ptr, col_idx, false);
  if (s != STM_OK) return s;
  // rows 0..n-1: the out-rows as given; rows n..2n-1: the in-rows (transpose, sorted)
  std::vector<int64_t> rp(2 * n + 1, 0);
  std::vector<int32_t> ci(2 * m);
  for (int64_t v = 0; v <= n; ++v) rp[v] = row_ptr[v];
  std::vector<int64_t> indeg(n + 1, 0);
  for (int64_t e = 0; e < m; ++e) ++indeg[col_idx[e]];
  for (int64_t v = 0; v < n; ++v) rp[n + v + 1] = rp[n + v] + indeg[v];
  std::copy(col_idx, col_idx + m, ci.begin());
  std::vector<int64_t> fill(rp.begin() + n, rp.begin() + 2 * n);
  for (int64_t v = 0; v < n; ++v)  // sources in increasing order: each in-row comes out sorted
    for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) ci[fill[col_idx[e]]++] = (int32_t)v;
  return upload_graph(n, 2 * n, rp.data(), ci.data(), labels, device, true, out);
}

extern "C" stm_status stm_graph_load_device(int64_t n, int64_t nnz, const int64_t* d_row_ptr,
                                            const int32_t* d_col_idx, const int32_t* d_labels, int device,
                                            stm_graph** out) {
  if (!out || !d_row_ptr || (nnz > 0 && !d_col_idx)) return stm_fail(STM_EINVAL, "NULL argument");
  if (n < 0 || n > INT32_MAX - 1 || nnz < 0) return stm_fail(STM_EINVAL, "bad sizes");
  if (nnz > (int64_t)UINT32_MAX)  // packed vertex records hold 32-bit row starts (kernel.cu vrec)
    return stm_fail(STM_EUNSUPPORTED, "%lld adjacency entries >= 2^32", (long long)nnz);
  {
    int ndev = 0;
    CU(cudaGetDeviceCount(&ndev));
    if (device < 0 || device >= ndev) return stm_fail(STM_EINVAL, "device %d of %d", device, ndev);
  }
  DeviceGuard dg(device);
  // cheap checks on the device: row_ptr[0] == 0, row_ptr[n] == nnz, monotone; max degree
  int64_t maxd = 0;
  {
    long long* d = nullptr;
    CU(cudaMalloc(&d, 3 * sizeof(long long)));
    long long init[3] = {0, 0, 0};
    CU(cudaMemcpy(d, init, sizeof init, cudaMemcpyHostToDevice));
    if (n > 0) degree_scan<<<(unsigned)std::min<int64_t>((n + 255) / 256, 65535), 256>>>(d_row_ptr, n, d);
    long long h[3];
    cudaError_t e = cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
    int64_t ends[2] = {0, 0};
    if (e == cudaSuccess) e = cudaMemcpy(&ends[0], d_row_ptr, sizeof(int64_t), cudaMemcpyDeviceToHost);
    if (e == cudaSuccess) e = cudaMemcpy(&ends[1], d_row_ptr + n, sizeof(int64_t), cudaMemcpyDeviceToHost);
    cudaFree(d);
    if (e != cudaSuccess) return stm_fail(STM_ECUDA, "%s", cudaGetErrorString(e));
    if (ends[0] != 0 || ends[1] != nnz) return stm_fail(STM_EINVAL, "row_ptr does not match nnz");
    if (h[1]) return stm_fail(STM_EINVAL, "row_ptr decreases");
    maxd = h[0];
  }
  stm_graph* g = new (std::nothrow) stm_graph();
  if (!g) return stm_fail(STM_ENOMEM, "host allocation");
  g->device = device;
  g->n = n;
  g->n_rows = n;
  g->nnz = nnz;
  g->max_degree = maxd;
  g->owns_csr = false;
  g->d_row_ptr = const_cast<int64_t*>(d_row_ptr);
  g->d_col_idx = const_cast<int32_t*>(d_col_idx);
  std::vector<int32_t> lab;
  if (d_labels) {
    lab.resize(n);
    cudaError_t e = cudaMemcpy(lab.data(), d_labels, sizeof(int32_t) * n, cudaMemcpyDeviceToHost);
    std::vector<uint8_t> dense;
    stm_status s = e == cudaSuccess ? dense_labels(n, lab.data(), dense, g->label_values)
                                    : stm_fail(STM_ECUDA, "%s", cudaGetErrorString(e));
    if (s == STM_OK) {
      e = cudaMalloc(&g->d_labels, std::max<int64_t>(n, 1));
      if (e == cudaSuccess && n) e = cudaMemcpy(g->d_labels, dense.data(), n, cudaMemcpyHostToDevice);
      if (e != cudaSuccess) s = stm_fail(STM_ECUDA, "%s", cudaGetErrorString(e));
    }
    if (s != STM_OK) {
      stm_graph_free(g);
      return s;
    }
  }
  cudaDeviceGetAttribute(&g->num_sms, cudaDevAttrMultiProcessorCount, device);
  cudaDeviceGetAttribute(&g->l2_bytes, cudaDevAttrL2CacheSize, device);
  query_persist(g);
  {
    std::vector<int64_t> rp(n + 1);
    if (cudaMemcpy(rp.data(), d_row_ptr, sizeof(int64_t) * (n + 1), cudaMemcpyDeviceToHost) == cudaSuccess)
      g->has_stats = stm_graph_stats_host(n, rp.data(), d_labels ? lab.data() : nullptr, &g->stats) == STM_OK;
    cudaGetLastError();
  }
  build_ranked(g);
  g->d_out_start = build_out_start(g->d_row_ptr, g->d_col_idx, g->n_rows, g->n);
  if (g->ranked) g->d_rout_start = build_out_start(g->d_rrow_ptr, g->d_rcol_idx, g->n, g->n);
  *out = g;
  return STM_OK;
}

extern "C" stm_status stm_graph_info(const stm_graph* g, int64_t* n, int64_t* nnz, int64_t* maxd) {
  if (!g) return stm_fail(STM_EINVAL, "NULL graph");
  if (n) *n = g->n;
  if (nnz) *nnz = g->nnz;
  if (maxd) *maxd = g->max_degree;
  return STM_OK;
}

extern "C" stm_status stm_graph_get_stats(const stm_graph* g, stm_graph_stats* out) {
  if (!g || !out) return stm_fail(STM_EINVAL, "NULL argument");
  if (!g->has_stats) return stm_fail(STM_EUNSUPPORTED, "graph statistics unavailable");
  *out = g->stats;
  return STM_OK;
}

extern "C" stm_status stm_graph_free(stm_graph* g) {
  if (!g) return STM_OK;
  DeviceGuard dg(g->device);
  if (g->owns_csr) {
    cudaFree(g->d_row_ptr);
    cudaFree(g->d_col_idx);
  }
  cudaFree(g->d_labels);
  cudaFree(g->d_rank2orig);
  cudaFree(g->d_rrow_ptr);
  cudaFree(g->d_rcol_idx);
  cudaFree(g->d_rlabels);
  cudaFree(g->d_out_start);
  cudaFree(g->d_rout_start);
  for (auto& kv : g->hubs) free_hub(kv.second);
  for (auto& kv : g->entries) cudaFree(kv.second.d);
  for (auto& kv : g->chunks) cudaFree(kv.second.d);
  delete g;
  return STM_OK;
}

extern "C" void stm_tuning_default(stm_tuning* t) {
  if (!t) return;
  memset(t, 0, sizeof *t);
  t->local_steal = 1;
  t->global_steal = 1;
  t->stop_level = 2;
  t->detect_level = 8;  // donors look at the pool's demand at every frame (measured)
  t->unroll = 0;      // auto: 32 with the 40-register kernel, 16 with the 64-register one (measured)
  t->occupancy = 0;   // auto: 40-register kernel when the CSR does not fit in half the L2
  t->root_order = 0;  // auto
  t->l2_persist_mb = 0;  // auto
  t->drive_ratio = 0;    // off (measured)
  t->root_chunk = 0;  // auto: 1 with the 64-register kernel, 2 with the 40-register one (measured)
  t->block_warps = 32;  // (measured: C2 K4 -11 %, C3 K5 -5 %, C5 K5 -6 %, K6-e -4 % vs 16)
  t->blocks_per_sm = 0;
  t->bitmap_min_degree = 0;  // auto
  t->bitmap_budget_mb = 0;   // auto
}

// ---------------------------------------------------------------------------- match
struct MultiArgs {     // merged census launch (STM_MULTI kernel build)
  const StmMVert* d_verts = nullptr;
  const StmMNode* d_nodes = nullptr;
  unsigned long long* d_counts = nullptr;
};

struct ListArgs {      // stm_match_list: root range and device output
  int64_t root_lo = 0, root_hi = -1;
  int32_t* d_out = nullptr;
  uint64_t cap = 0;
  uint64_t n_found = 0;  // out
};

static stm_status launch(const stm_graph* gc, const stm_plan* p, const stm_tuning* tin,
                         const stm_shard* shard, void* stream, stm_async_result* d_result,
                         unsigned long long* d_per_root, uint64_t* h_count, ListArgs* la = nullptr,
                         const MultiArgs* ma = nullptr) {
  if (!gc || !p) return stm_fail(STM_EINVAL, "NULL graph or plan");
  stm_graph* g = const_cast<stm_graph*>(gc);
  stm_tuning t;
  if (tin) t = *tin; else stm_tuning_default(&t);
  if (t.unroll < 0 || t.unroll > STM_UMAX) return stm_fail(STM_EINVAL, "unroll %d not in 0..%d", t.unroll, STM_UMAX);
  if (t.occupancy < 0 || t.occupancy > 2) return stm_fail(STM_EINVAL, "occupancy %d not in 0..2", t.occupancy);
  if (t.root_order < 0 || t.root_order > 3) return stm_fail(STM_EINVAL, "root_order %d not in 0..3", t.root_order);
  if (t.root_chunk < 0) return stm_fail(STM_EINVAL, "root_chunk %d < 0", t.root_chunk);
  if (t.block_warps == 0) t.block_warps = 32;
  if (t.block_warps < 1 || t.block_warps > 32) return stm_fail(STM_EINVAL, "block_warps %d", t.block_warps);
  if (t.stop_level < 1) t.stop_level = 1;
  if (t.watchdog_ms < 0) return stm_fail(STM_EINVAL, "watchdog_ms %d < 0", t.watchdog_ms);
  if (t.backoff_max < 0 || t.backoff_max > 12) return stm_fail(STM_EINVAL, "backoff_max %d not in 0..12", t.backoff_max);
  if (t.carveout_pct < -1 || t.carveout_pct > 100) return stm_fail(STM_EINVAL, "carveout_pct %d", t.carveout_pct);
  if (t.root_split < -1) return stm_fail(STM_EINVAL, "root_split %d", t.root_split);
  if (t.chunk_cost < -1) return stm_fail(STM_EINVAL, "chunk_cost %d", t.chunk_cost);
  if (t.jit < -1 || t.jit > 1) return stm_fail(STM_EINVAL, "jit %d not in -1..1", t.jit);
  if (d_result && ((uintptr_t)d_result & 7)) return stm_fail(STM_EINVAL, "d_result not 8-byte aligned");
  const StmPlan& P = p->dev;
  if ((P.directed != 0) != g->directed)
    return stm_fail(STM_EINVAL, g->directed ? "directed graph needs a STM_DIRECTED plan"
                                             : "STM_DIRECTED plan on an undirected graph");
  if (!p->labels.empty() && !g->d_labels) {
    bool any = false;
    for (int x : p->labels) any |= x >= 0;
    if (any) return stm_fail(STM_EINVAL, "labeled pattern on an unlabeled graph");
  }
  if (shard) {
    if (shard->world < 1 || shard->world > 8 || shard->rank < 0 || shard->rank >= shard->world ||
        shard->chunk < 0 || !shard->d_cursors[shard->rank])
      return stm_fail(STM_EINVAL, "bad shard");
  }
  DeviceGuard dg(g->device);

  StmKParams kp;
  memset(&kp, 0, sizeof kp);
  kp.plan = P;
  // order-free restrictions count on the degree-ranked copy (same count, less work)
  const bool use_rank = g->ranked && p->order_free && t.vertex_order == 0;
  kp.col_idx = use_rank ? g->d_rcol_idx : g->d_col_idx;
  kp.labels = use_rank ? g->d_rlabels : g->d_labels;
  kp.root_map = use_rank ? g->d_rank2orig : nullptr;
  kp.split = t.narrow_split == 0 ? 1 : 0;
  kp.n = g->n;
  kp.n_dir = g->directed ? (int32_t)g->n : 0;
  if (la) {
    kp.root_lo = la->root_lo;
    kp.n = la->root_hi;
    kp.list_out = la->d_out;
    kp.list_cap = la->cap;
  }
  std::unique_lock<std::mutex> glock(g->mu);  // per-numbering records / hub cache + L2 persistence state
  {
    const int min_deg = t.bitmap_min_degree == 0 ? STM_BITMAP_AUTO_MIN_DEGREE : t.bitmap_min_degree;
    const int64_t budget = (int64_t)(t.bitmap_budget_mb > 0 ? t.bitmap_budget_mb : STM_BITMAP_AUTO_BUDGET_MB) << 20;
    const stm_graph::HubBitmaps* hb = ensure_hub(g, use_rank, min_deg, budget);
    if (!hb) return stm_fail(STM_ENOMEM, "per-vertex records: %s", cudaGetErrorString(cudaGetLastError()));
    kp.vrec = hb->vrec;
    kp.bitmaps = hb->bits;
    kp.bm_words = hb->words;
    g_info.hubs = hb->n_hubs;
    // root splitting (stm_tuning.root_split): not for listing pages, which are root-id ranges
    const int T = t.root_split == 0 ? STM_ROOT_SPLIT_AUTO : t.root_split;
    const stm_graph::RootEntries* E = nullptr;
    if (!la && T > 0 && !g->directed) {
      E = ensure_entries(g, use_rank, T);
      if (E) {
        kp.entries = E->d;
        kp.root_split = T;
        kp.n = E->n;
      }
    }
    // work-balanced chunks (stm_tuning.chunk_cost): not for listing pages (root-id ranges)
    // auto: at most STM_CHUNK_COST_AUTO, and at least ~8 chunks per resident warp (48 per SM)
    const int64_t c_auto = (g->n + g->nnz) / (8ll * 48 * std::max(1, g->num_sms));
    const int C = t.chunk_cost == 0 ? (int)std::max<int64_t>(16, std::min<int64_t>(STM_CHUNK_COST_AUTO, c_auto))
                                    : t.chunk_cost;
    if (!la && C > 0) {
      const stm_graph::ChunkBounds* B = ensure_chunks(g, use_rank, E, T, C);
      if (B) {
        kp.chunk_bounds = B->d;
        kp.n_chunks = B->n;
      }
    }
  }
  // label-slot table: dense graph label -> bitmask of pattern slots with that value
  for (int d = 0; d < (int)g->label_values.size(); ++d)
    for (int s = 0; s < P.n_label_slots; ++s)
      if (g->label_values[d] == P.label_value[s]) kp.lab2slot[d] |= (uint8_t)(1u << s);
  const int64_t cap64 = std::max<int64_t>(32, (g->max_degree + 31) / 32 * 32);
  if (cap64 > INT32_MAX / 4) return stm_fail(STM_EUNSUPPORTED, "max degree too large");
  kp.cap = (int)cap64;
  kp.block_warps = t.block_warps;
  kp.local_steal = t.local_steal;
  kp.global_steal = t.global_steal;
  kp.stop_level = t.stop_level;
  kp.detect_level = t.detect_level;
  // kernel variant: DRAM-resident graphs are latency-bound -> more warps
  int variant = t.occupancy;
  if (variant == 0) {
    const int64_t csr = (int64_t)g->nnz * 4 + (g->n + 1) * 8;
    variant = csr > (int64_t)g->l2_bytes / 2 ? 2 : 1;
  }
  kp.unroll = t.unroll ? t.unroll : (variant == 2 ? 32 : 16);
  if (ma) {  // the merged build is compiled with 8 siblings per frame
    kp.unroll = std::min(kp.unroll, 8);
    kp.mv = ma->d_verts;
    kp.mn = ma->d_nodes;
    kp.mcount = ma->d_counts;
  }
  const int root_chunk = t.root_chunk ? t.root_chunk : (variant == 2 ? 2 : 1);
  // root order: ascending by default -- descending (high-degree roots first on the
  // ranked copy) measured 1.2-1.7x slower on C2/C3 and neutral on C5
  kp.root_desc = t.root_order == 2 ? 1 : t.root_order == 3 ? 2 : 0;
  // L2 persistence (B200 126 MB L2): on the degree-ranked copy the rows are in degree
  // order, so the tail of col_idx holds the longest lists -- the ones every set
  // operation probes.  Keep up to l2_persist_mb of it persisting in L2 when the CSR
  // does not fit (auto: off -- measured no gain).
  {
    const int64_t csr = (int64_t)g->nnz * 4 + (g->n + 1) * 8;
    const int mb = t.l2_persist_mb == 0 ? STM_L2_PERSIST_AUTO_MB : t.l2_persist_mb;
    if (use_rank && mb > 0 && csr > (int64_t)g->l2_bytes / 2 && g->max_window > 0) {
      int64_t w = std::min<int64_t>((int64_t)mb << 20, std::min<int64_t>(g->max_window, g->nnz * 4));
      w = std::min<int64_t>(w, g->persist_max);
      if (w > 0) {
        if (g->persist_set != w) {
          if (cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)w) == cudaSuccess) g->persist_set = w;
          else cudaGetLastError();
        }
        if (g->persist_set > 0) {
          kp.l2_window_base = (const void*)(g->d_rcol_idx + g->nnz - w / 4);
          kp.l2_window_bytes = std::min<int64_t>(w, g->persist_set);
        }
      }
    }
  }
  glock.unlock();
  // roots gathered per frame-1 batch: with work-balanced chunks a light chunk holds many roots
  kp.root_batch = (kp.chunk_bounds && t.root_chunk == 0) ? STM_RMAX : std::max(1, std::min(STM_RMAX, root_chunk));
  if (P.level_begin[1] != P.level_begin[2]) kp.root_batch = 1;  // level-1 set nodes: built per root (kernel.cu)
  kp.count_bytes = t.instrument ? 1 : 0;
  if (t.hash_slots < 0 || t.hash_slots > 4096 || (t.hash_slots && (t.hash_slots < 64 || (t.hash_slots & (t.hash_slots - 1)))))
    return stm_fail(STM_EINVAL, "hash_slots %d: 0 or a power of two in 64..4096", t.hash_slots);
  if (t.hash_slots && !stm_hash_compiled())
    return stm_fail(STM_EUNSUPPORTED, "hash_slots: this build has no hash-set path (-DSTM_WITH_HASH=1)");
  kp.ht_slots = t.hash_slots;
  kp.donate_mask = 0;  // look for idle blocks at every opportunity (measured: rate limiting starves idle blocks)
  kp.backoff_max = t.backoff_max ? t.backoff_max : 8;
  if (t.drive_ratio > 1 && !stm_drive_compiled())
    return stm_fail(STM_EUNSUPPORTED, "drive_ratio: this build has no drive-ratio path (-DSTM_DRIVE_RATIO=1)");
  kp.drive_ratio = t.drive_ratio;
  kp.watchdog_ns = (long long)t.watchdog_ms * 1000000LL;
  kp.result = (unsigned long long*)d_result;

  int bps = 0;
  if (ma && (la || t.instrument)) return stm_fail(STM_EINVAL, "merged launches do not list or instrument");
  // plan-specialised kernel (jit.cpp; stm_tuning.jit) for plain counting launches
  const void* jfn = nullptr;
  if (!ma && !la && !t.instrument && t.jit >= 0) {
    std::string jerr;
    jfn = stm_jit_kernel(P, variant, &jerr);
    if (!jfn && t.jit == 1) return stm_fail(STM_EUNSUPPORTED, "plan-specialised kernel: %s", jerr.c_str());
  }
  int oe = jfn ? stm_occupancy_fn(jfn, t.block_warps, P.k, P.n_nodes, t.hash_slots, t.carveout_pct, &bps)
               : (ma ? stm_occupancy_multi : la ? stm_occupancy_list : t.instrument ? stm_occupancy_instr : stm_occupancy)(
                     variant, t.block_warps, P.k, P.n_nodes, t.hash_slots, t.carveout_pct, &bps);
  if (oe != 0) return stm_fail(STM_ECUDA, "occupancy (variant %d, %s build, %d warps): %s", variant, la ? "list" : t.instrument ? "instr" : "count", t.block_warps, cudaGetErrorString((cudaError_t)oe));
  if (bps < 1) return stm_fail(STM_EUNSUPPORTED, "kernel does not fit on an SM with %d warps", t.block_warps);
  if (t.blocks_per_sm > 0) bps = std::min(bps, t.blocks_per_sm);
  // no more warps than root chunks (tiny graphs: the idle surplus would only add start-up,
  // work-sharing and termination traffic)
  int grid = bps * g->num_sms;
  if (kp.chunk_bounds && !shard) grid = (int)std::max<int64_t>(1, std::min<int64_t>(grid, (kp.n_chunks + t.block_warps - 1) / t.block_warps));
  const int64_t warps = (int64_t)grid * t.block_warps;
  const size_t arena_bytes = (size_t)warps * (size_t)P.n_nodes * (size_t)kp.cap * sizeof(int32_t);
  // task pool: never more tasks than blocks (StmWork::deficit), capacity 2 * grid rounded up
  int pool_shift = 6;
  while ((1 << pool_shift) < 2 * grid) ++pool_shift;
  const size_t state_bytes = sizeof(StmWork) + 64 + sizeof(StmPoolSlot) * ((size_t)1 << pool_shift);

  // per-launch scratch (set arena + scheduler state), cached per (device, stream) for the
  // process and shared by every graph counted on that stream (stream order serialises its
  // users): a new graph does not pay a multi-GB allocation on its first launch
  Scratch* S;
  {
    static std::mutex scratch_mu;
    static std::map<std::pair<int, void*>, Scratch> scratch_cache;
    std::lock_guard<std::mutex> lk(scratch_mu);
    S = &scratch_cache[std::make_pair(g->device, stream)];
    if (S->arena_bytes < arena_bytes) {
      cudaFree(S->arena);
      S->arena = nullptr;
      S->arena_bytes = 0;
      if (arena_bytes) {
        cudaError_t e = cudaMalloc(&S->arena, arena_bytes);
        if (e != cudaSuccess)
          return stm_fail(STM_ENOMEM, "set arena of %zu bytes: %s", arena_bytes, cudaGetErrorString(e));
        S->arena_bytes = arena_bytes;
      }
    }
    if (S->state_bytes < state_bytes) {
      cudaFree(S->state);
      S->state = nullptr;
      S->state_bytes = 0;
      CU(cudaMalloc(&S->state, state_bytes));
      S->state_bytes = state_bytes;
    }
  }
  StmWork* work = (StmWork*)S->state;
  unsigned long long* own_cursor = (unsigned long long*)((char*)S->state + sizeof(StmWork));
  kp.arena = S->arena;
  kp.work = work;
  kp.pool = (StmPoolSlot*)((char*)S->state + sizeof(StmWork) + 64);
  kp.pool_shift = pool_shift;
  kp.pool_mask = (1 << pool_shift) - 1;
  kp.total_warps = (int)warps;
  kp.per_root = d_per_root;
  if (shard) {
    kp.rank = shard->rank;
    kp.world = shard->world;
    kp.chunk = shard->chunk ? shard->chunk : root_chunk;
    for (int r = 0; r < shard->world; ++r) kp.cursors[r] = (unsigned long long*)shard->d_cursors[r];
  } else {
    kp.rank = 0;
    kp.world = 1;
    kp.chunk = root_chunk;
    kp.cursors[0] = own_cursor;
  }
  cudaStream_t st = (cudaStream_t)stream;
  CU(cudaMemsetAsync(S->state, 0, state_bytes, st));
  int le = jfn ? stm_launch_fn(jfn, kp, grid, stream)
               : (ma ? stm_launch_multi : la ? stm_launch_list : t.instrument ? stm_launch_instr : stm_launch)(
                     variant, kp, grid, stream);
  if (le != 0) return stm_fail(STM_ECUDA, "launch: %s", cudaGetErrorString((cudaError_t)le));
  g_info.grid = grid;
  g_info.block_threads = t.block_warps * 32;
  g_info.smem_bytes = ma ? stm_smem_bytes_multi(t.block_warps, P.k, P.n_nodes)
                         : stm_smem_bytes(t.block_warps, P.k, P.n_nodes, t.hash_slots);
  g_info.arena_bytes = (int64_t)arena_bytes;
  g_info.cap = kp.cap;
  g_info.ranked = use_rank ? 1 : 0;
  g_info.jit = jfn ? 1 : 0;
  g_info.variant = variant;
  g_info.unroll = kp.unroll;
  if (h_count) {
    StmWork hw;
    CU(cudaMemcpyAsync(&hw, work, sizeof(StmWork), cudaMemcpyDeviceToHost, st));
    CU(cudaStreamSynchronize(st));
    if (hw.overflow == 2) return stm_fail(STM_ETIMEOUT, "launch aborted after watchdog_ms = %d", t.watchdog_ms);
    if (hw.overflow) return stm_fail(STM_EOVERFLOW, "device capacity exceeded");
    g_info.local_steals = (int64_t)hw.n_local_steals;
    g_info.global_steals = (int64_t)hw.n_global_steals;
    g_info.chunks = (int64_t)hw.n_chunks;
    g_info.peer_chunks = (int64_t)hw.n_peer_chunks;
    g_info.alg_bytes = (int64_t)hw.alg_bytes;
    g_info.merge_bytes = (int64_t)hw.merge_bytes;
    g_info.jobs = (int64_t)hw.n_jobs;
    g_info.idle_cycles = (int64_t)hw.idle_cycles;
    memcpy(g_prof, hw.prof, sizeof g_prof);
    g_info.warp_cycles = (int64_t)hw.warp_cycles;
    if (la) la->n_found = hw.list_n;
    *h_count = hw.count;
  }
  return STM_OK;
}

extern "C" stm_status stm_match_count(const stm_graph* g, const stm_plan* p, void* stream, uint64_t* count) {
  if (!count) return stm_fail(STM_EINVAL, "count is NULL");
  return launch(g, p, nullptr, nullptr, stream, nullptr, nullptr, count);
}

extern "C" stm_status stm_match_count_ex(const stm_graph* g, const stm_plan* p, const stm_tuning* t,
                                         const stm_shard* shard, void* stream, uint64_t* count) {
  if (!count) return stm_fail(STM_EINVAL, "count is NULL");
  return launch(g, p, t, shard, stream, nullptr, nullptr, count);
}

extern "C" stm_status stm_match_count_async(const stm_graph* g, const stm_plan* p, const stm_tuning* t,
                                            const stm_shard* shard, void* stream, stm_async_result* d_result) {
  if (!d_result) return stm_fail(STM_EINVAL, "d_result is NULL");
  return launch(g, p, t, shard, stream, d_result, nullptr, nullptr);
}

extern "C" stm_status stm_match_count_per_root(const stm_graph* g, const stm_plan* p, const stm_tuning* t,
                                               void* stream, uint64_t* per_root, uint64_t* count) {
  if (!g || !per_root || !count) return stm_fail(STM_EINVAL, "NULL argument");
  DeviceGuard dg(g->device);
  unsigned long long* d = nullptr;
  CU(cudaMalloc(&d, sizeof(unsigned long long) * std::max<int64_t>(g->n, 1)));
  cudaError_t ze = cudaMemsetAsync(d, 0, sizeof(unsigned long long) * std::max<int64_t>(g->n, 1), (cudaStream_t)stream);
  if (ze != cudaSuccess) {
    cudaFree(d);
    return stm_fail(STM_ECUDA, "per-root buffer: %s", cudaGetErrorString(ze));
  }
  uint64_t c = 0;
  stm_status s = launch(g, p, t, nullptr, stream, nullptr, d, &c);
  if (s == STM_OK) {
    cudaError_t e = cudaMemcpy(per_root, d, sizeof(uint64_t) * g->n, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) s = stm_fail(STM_ECUDA, "%s", cudaGetErrorString(e));
  }
  cudaFree(d);
  if (s == STM_OK) *count = c;
  return s;
}

extern "C" stm_status stm_match_list(const stm_graph* g, const stm_plan* p, const stm_tuning* t,
                                     int64_t root_begin, int64_t root_end, void* stream, int32_t* out,
                                     uint64_t capacity, uint64_t* n_listed, uint64_t* count) {
  if (!g || !p || !n_listed || !count) return stm_fail(STM_EINVAL, "NULL argument");
  if (capacity > 0 && !out) return stm_fail(STM_EINVAL, "out is NULL with capacity %llu", (unsigned long long)capacity);
  if (root_begin < 0 || root_end < root_begin || root_end > g->n)
    return stm_fail(STM_EINVAL, "root range [%lld, %lld) not within [0, %lld)", (long long)root_begin,
                    (long long)root_end, (long long)g->n);
  const int k = p->k;
  if (capacity > (uint64_t)(INT64_MAX / 4 / k)) return stm_fail(STM_EINVAL, "capacity too large");
  DeviceGuard dg(g->device);
  int32_t* d = nullptr;
  const size_t bytes = sizeof(int32_t) * (size_t)k * (size_t)std::max<uint64_t>(capacity, 1);
  cudaError_t e = cudaMalloc(&d, bytes);
  if (e != cudaSuccess) return stm_fail(STM_ENOMEM, "listing buffer of %zu bytes: %s", bytes, cudaGetErrorString(e));
  ListArgs la;
  la.root_lo = root_begin;
  la.root_hi = root_end;
  la.d_out = d;
  la.cap = capacity;
  uint64_t c = 0;
  stm_status s = launch(g, p, t, nullptr, stream, nullptr, nullptr, &c, &la);
  const uint64_t nl = std::min<uint64_t>(la.n_found, capacity);
  if (s == STM_OK && nl) {
    e = cudaMemcpy(out, d, sizeof(int32_t) * (size_t)k * (size_t)nl, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) s = stm_fail(STM_ECUDA, "%s", cudaGetErrorString(e));
  }
  cudaFree(d);
  if (s == STM_OK) {
    *n_listed = nl;
    *count = c;
  }
  return s;
}

stm_status stm_launch_merged(const stm_graph* g, const stm_merged& m, const stm_tuning* t, void* stream,
                             uint64_t* counts) {
  if (!g) return stm_fail(STM_EINVAL, "NULL graph");
  DeviceGuard dg(g->device);
  stm_plan tmp;  // the launch-shape view of the merged plan (k, set regions)
  memset(&tmp.dev, 0, sizeof tmp.dev);
  tmp.dev.k = m.k;
  tmp.dev.n_nodes = m.n_regions;
  tmp.dev.filt[0].lab = STM_LAB_ANY;
  tmp.k = m.k;
  tmp.order_free = m.order_free;
  tmp.flags = STM_AUTO_RESTRICT;
  MultiArgs ma;
  void *dv = nullptr, *dn = nullptr, *dc = nullptr;
  const size_t bv = sizeof(StmMVert) * std::max<size_t>(m.verts.size(), 1);
  const size_t bn = sizeof(StmMNode) * std::max<size_t>(m.nodes.size(), 1);
  const size_t bc = sizeof(unsigned long long) * std::max(m.n_patterns, 1);
  cudaError_t e = cudaMalloc(&dv, bv);
  if (e == cudaSuccess) e = cudaMalloc(&dn, bn);
  if (e == cudaSuccess) e = cudaMalloc(&dc, bc);
  if (e == cudaSuccess) e = cudaMemcpy(dv, m.verts.data(), sizeof(StmMVert) * m.verts.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess && !m.nodes.empty())
    e = cudaMemcpy(dn, m.nodes.data(), sizeof(StmMNode) * m.nodes.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemsetAsync(dc, 0, bc, (cudaStream_t)stream);
  stm_status s = STM_OK;
  if (e != cudaSuccess) s = stm_fail(STM_ECUDA, "merged plan upload: %s", cudaGetErrorString(e));
  if (s == STM_OK) {
    ma.d_verts = (const StmMVert*)dv;
    ma.d_nodes = (const StmMNode*)dn;
    ma.d_counts = (unsigned long long*)dc;
    uint64_t total = 0;
    s = launch(g, &tmp, t, nullptr, stream, nullptr, nullptr, &total, nullptr, &ma);
    if (s == STM_OK) {
      e = cudaMemcpy(counts, dc, sizeof(uint64_t) * m.n_patterns, cudaMemcpyDeviceToHost);
      if (e != cudaSuccess) s = stm_fail(STM_ECUDA, "%s", cudaGetErrorString(e));
    }
  }
  cudaFree(dv);
  cudaFree(dn);
  cudaFree(dc);
  return s;
}

extern "C" stm_status stm_last_profile(uint64_t* out, int n) {
  if (!out || n < 0) return stm_fail(STM_EINVAL, "NULL out");
  for (int i = 0; i < n && i < STM_PROF_SIZE; ++i) out[i] = g_prof[i];
  return STM_OK;
}

extern "C" stm_status stm_last_launch(stm_launch_info* info) {
  if (!info) return stm_fail(STM_EINVAL, "NULL info");
  *info = g_info;
  return STM_OK;
}

// ---------------------------------------------------------------- IPC chunk cursors
extern "C" stm_status stm_cursors_alloc(int device, int n_slots, uint64_t** d_base, void* ipc_handle) {
  if (!d_base || !ipc_handle || n_slots < 1) return stm_fail(STM_EINVAL, "NULL argument or n_slots < 1");
  int ndev = 0;
  CU(cudaGetDeviceCount(&ndev));
  if (device < 0 || device >= ndev) return stm_fail(STM_EINVAL, "device %d of %d", device, ndev);
  static_assert(sizeof(cudaIpcMemHandle_t) <= STM_IPC_HANDLE_BYTES, "IPC handle size");
  DeviceGuard dg(device);
  void* d = nullptr;
  const size_t bytes = (size_t)n_slots * 64;
  CU(cudaMalloc(&d, bytes));
  cudaError_t e = cudaMemset(d, 0, bytes);
  cudaIpcMemHandle_t h;
  if (e == cudaSuccess) e = cudaIpcGetMemHandle(&h, d);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e != cudaSuccess) {
    cudaFree(d);
    return stm_fail(STM_ECUDA, "cursor allocation / IPC handle: %s", cudaGetErrorString(e));
  }
  memset(ipc_handle, 0, STM_IPC_HANDLE_BYTES);
  memcpy(ipc_handle, &h, sizeof h);
  *d_base = (uint64_t*)d;
  return STM_OK;
}

extern "C" stm_status stm_cursors_open(int device, const void* ipc_handle, uint64_t** d_peer_base) {
  if (!ipc_handle || !d_peer_base) return stm_fail(STM_EINVAL, "NULL argument");
  DeviceGuard dg(device);
  cudaIpcMemHandle_t h;
  memcpy(&h, ipc_handle, sizeof h);
  void* d = nullptr;
  CU(cudaIpcOpenMemHandle(&d, h, cudaIpcMemLazyEnablePeerAccess));
  *d_peer_base = (uint64_t*)d;
  return STM_OK;
}

extern "C" stm_status stm_cursors_close(int device, uint64_t* d_peer_base) {
  if (!d_peer_base) return STM_OK;
  DeviceGuard dg(device);
  CU(cudaIpcCloseMemHandle(d_peer_base));
  return STM_OK;
}

extern "C" stm_status stm_cursors_reset(int device, uint64_t* d_base, int first_slot, int n_slots,
                                        void* stream) {
  if (!d_base || first_slot < 0 || n_slots < 0) return stm_fail(STM_EINVAL, "bad cursor range");
  DeviceGuard dg(device);
  CU(cudaMemsetAsync((char*)d_base + (size_t)first_slot * 64, 0, (size_t)n_slots * 64, (cudaStream_t)stream));
  return STM_OK;
}

extern "C" stm_status stm_cursors_free(int device, uint64_t* d_base) {
  if (!d_base) return STM_OK;
  DeviceGuard dg(device);
  CU(cudaFree(d_base));
  return STM_OK;
}
