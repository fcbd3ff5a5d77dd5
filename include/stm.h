/*
 * stm.h -- C ABI of the B200-native STMatch counting hot path (libstm.so).
 *
 * The library counts the embeddings of a small query pattern Q in a large data
 * graph G on one B200 (sm_100a) with a single persistent CUDA kernel: outer-loop
 * parallel, stack-based backtracking (Sec. IV), set
 * intersection / difference of sorted neighbour lists,
 * loop unrolling (Sec. VI), loop-invariant code motion
 * (Sec. VII) and two-level work stealing (Sec. V,
 * PAPER.md:80-114).  Multi-GPU runs replicate the graph and split the
 * outermost loop; the caller sums the per-rank partial counts.
 *
 * Conventions for every function:
 *   - extern "C", never throws, returns stm_status.  On anything but STM_OK the
 *     out-parameters are left untouched and stm_last_error() returns a
 *     thread-local, human-readable message.
 *   - Host arrays passed in are BORROWED for the duration of the call only (the
 *     library copies what it keeps); the caller may free them afterwards.
 *   - Handles (stm_graph*, stm_plan*) are owned by the library and released by
 *     the matching *_free call.  Graphs and plans are immutable after creation
 *     and may be shared by concurrent calls on different CUDA streams.
 *   - Per-launch scratch (set arena, scheduler state) is library-owned, cached per
 *     (device, stream) for the life of the process and reused by every graph counted
 *     on that stream; calls on ONE stream must therefore be issued from one host
 *     thread at a time (their launches are stream-ordered).
 *   - CUDA failures map to STM_ECUDA (message carries cudaGetErrorString).
 *   - A count is never silently wrong: capacity problems are STM_EOVERFLOW.
 *
 * Result semantics (problem statement PAPER.md:44-48):
 *
 *   count = #{ f : V_Q -> V injective |
 *              every pattern edge {a,b} maps to a data edge {f(a), f(b)};
 *              [vertex-induced] every pattern non-edge maps to a data non-edge;
 *              [labeled] L_G(f(u)) == L_Q(u) for every u;
 *              f(a) < f(b) (caller's original vertex IDs) for every restriction (a,b) }
 *   modulo 2^64.  With STM_AUTO_RESTRICT the restriction set is a complete
 *   symmetry-breaking set of the label-preserving automorphism group of Q, so the
 *   count is the number of distinct subgraphs of G isomorphic to Q.
 */
#ifndef STM_H_
#define STM_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  STM_OK = 0,
  STM_EINVAL = 1,        /* invalid argument (bad CSR, bad pattern, bad order, cyclic restrictions, ...) */
  STM_ENOMEM = 2,        /* host or device allocation failed */
  STM_ECUDA = 3,         /* a CUDA runtime call failed */
  STM_EUNSUPPORTED = 4,  /* valid request outside this build's limits (k > 8, > 255 graph labels, ...) */
  STM_EOVERFLOW = 5,     /* device scratch / stack capacity exceeded: no count produced */
  STM_ETIMEOUT = 6       /* the launch ran longer than stm_tuning.watchdog_ms and was aborted: no count */
} stm_status;

typedef struct stm_graph stm_graph; /* opaque, device-resident, immutable */
typedef struct stm_plan stm_plan;   /* opaque, host-side compiled pattern, immutable */

/* Pattern compilation flags (bitwise OR). */
enum {
  STM_EDGE_INDUCED = 0,    /* non-induced monomorphisms: set differences removed */
  STM_VERTEX_INDUCED = 1,  /* pattern non-edges must be data non-edges: set differences */
  STM_NO_CODE_MOTION = 2,  /* recompute every level's candidate set from raw neighbour lists (ablation) */
  STM_AUTO_RESTRICT = 4,   /* ignore `restr`; use Grochow-Kellis symmetry-breaking restrictions */
  STM_AUTO_ORDER = 8,      /* ignore `order`; use the greedy connected order */
  STM_CENSUS_PER_MOTIF = 32, /* stm_motif_census only: one counting launch per motif instead of the merged
                                trie launch (A/B baseline of pattern merging) */
  STM_LAZY_UNBOUNDED = 16, /* code motion hoists only set chains that carry a restriction bound for their
                              consumer; a chain unbounded at its first operation is computed at the level
                              of its first consumer (no hoisting across levels whose prefixes rarely extend;
                              speed only) */
  STM_DIRECTED = 64        /* directed pattern (NEXT-4): `edges` are arcs (a, b) = a -> b, and
                              the plan counts in graphs loaded with stm_graph_load_directed: every arc of Q
                              an arc of G (vertex-induced: every non-arc a non-arc) */
};

enum { STM_K_MAX = 8 };

/*
 * stm_graph_load -- copy a CSR data graph to device `device` (G = (V, E, L);
 * neighbour lists are binary-searched, so rows must be sorted).
 *   n        number of vertices (>= 0); IDs are 0..n-1 and must fit in int32.
 *   row_ptr  host int64[n+1], row_ptr[0] == 0, non-decreasing.
 *   col_idx  host int32[row_ptr[n]]; each row strictly increasing (sorted, no
 *            duplicates), no self-loops, and the graph symmetric (undirected).
 *   labels   host int32[n] vertex labels (any non-negative values) or NULL.
 *            At most 255 distinct values (STM_EUNSUPPORTED otherwise).
 *   device   CUDA device ordinal.
 *   out      receives the handle.
 * Errors: STM_EINVAL for any CSR violation above (row_ptr checked on the host, the
 * O(m log d) entry checks on the device after the copy; no handle is returned on a
 * violation), STM_ENOMEM, STM_ECUDA, STM_EUNSUPPORTED (> 255 labels, or
 * row_ptr[n] >= 2^32 adjacency entries: the kernel's packed per-vertex records hold
 * 32-bit row starts).
 */
stm_status stm_graph_load(int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                          const int32_t* labels, int device, stm_graph** out);

/*
 * stm_graph_load_device -- as stm_graph_load but BORROWS device arrays already
 * resident on `device` (e.g. torch tensors).  The caller keeps them alive and
 * unmodified until stm_graph_free.  Only cheap checks are done (sizes); the
 * arrays must satisfy the same CSR contract.  Labels (if given) are remapped into
 * a library-owned device copy.
 */
stm_status stm_graph_load_device(int64_t n, int64_t nnz, const int64_t* d_row_ptr,
                                 const int32_t* d_col_idx, const int32_t* d_labels, int device,
                                 stm_graph** out);

/* stm_graph_info -- n, number of directed adjacency entries (2m), max degree. Any out may be NULL. */
stm_status stm_graph_info(const stm_graph* g, int64_t* n, int64_t* nnz, int64_t* max_degree);

/*
 * stm_graph_load_directed -- a directed simple graph (NEXT-4; "supports both directed
 * and undirected graphs").  row_ptr / col_idx are the out-neighbour rows (arc v -> col_idx[e] for
 * e in [row_ptr[v], row_ptr[v+1])), sorted strictly ascending, no self-loops, ids in [0, n); the
 * in-rows are built here.  Both are device-resident (2 * m entries).  Counted with STM_DIRECTED
 * plans only (STM_EINVAL otherwise).  No degree-ranked copy, hub bitmaps or root splitting (speed
 * only).  Ownership, labels and errors as stm_graph_load.
 */
stm_status stm_graph_load_directed(int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                                   const int32_t* labels, int device, stm_graph** out);

stm_status stm_graph_free(stm_graph* g);

/*
 * stm_pattern_compile -- host-only pattern compiler (PAPER.md:52 matching order;
 * PAPER.md:132-140 code motion with merged multi-label sets; restrictions are
 * north_star's symmetry breaking, not in the paper).
 *   k        pattern size, 2 <= k <= STM_K_MAX (k == 1 is STM_EINVAL).
 *   n_edges, edges  pattern edges as 2*n_edges vertex ids in [0,k); duplicates
 *            are merged; self-loops are STM_EINVAL; Q must be connected.
 *   labels   int32[k] pattern vertex labels, or NULL (unlabeled).  Value -1 is a
 *            wildcard (matches any label); other values must be >= 0.
 *   order    int32[k] matching order (a permutation of 0..k-1 in which every
 *            vertex after the first is adjacent to an earlier one),
 *            or NULL for the greedy order.  Ignored with STM_AUTO_ORDER.
 *   n_restr, restr  2*n_restr pattern vertex pairs (a, b) meaning f(a) < f(b).
 *            a == b or a cyclic set is STM_EINVAL.  Ignored with STM_AUTO_RESTRICT.
 *   flags    STM_* flags above.
 *   out      receives the plan handle.
 */
stm_status stm_pattern_compile(int k, int n_edges, const int32_t* edges, const int32_t* labels,
                               const int32_t* order, int n_restr, const int32_t* restr,
                               uint32_t flags, stm_plan** out);

/*
 * stm_plan_describe -- human-readable plan (order, restrictions, |Aut_L|, set
 * nodes with their operations, candidate sources, scratch words per warp).
 * Writes at most len bytes including the terminating NUL; returns STM_EINVAL if
 * len is too small (the message then holds the required size).
 */
stm_status stm_plan_describe(const stm_plan* p, char* buf, size_t len);

/* stm_plan_info -- pattern size, number of materialised set nodes, |Aut_L(Q)|. Any out may be NULL. */
stm_status stm_plan_info(const stm_plan* p, int* k, int* n_sets, int64_t* aut_size);

/* stm_plan_raw -- the compiled device plan (the StmPlan record the kernel interprets,
 * paper_conf_sc_weij22_b200/csrc/plan.h) as bytes: *size receives its size; buf (len bytes,
 * may be NULL to query the size) receives a copy.  Used to build plan-specialised kernels
 * (tools/cplan.py) and by tests.  STM_EINVAL if buf is too small. */
stm_status stm_plan_raw(const stm_plan* p, void* buf, size_t len, size_t* size);

stm_status stm_plan_free(stm_plan* p);

/* Tuning knobs: every setting changes speed only, never the count. NULL = defaults. */
typedef struct stm_tuning {
  int32_t local_steal;    /* 0/1: intra-block work sharing through shared-memory mailboxes (Sec. V-A,
                             re-designed: busy warps split their own stacks on request).  Default 1. */
  int32_t global_steal;   /* 0/1: inter-block work sharing through a grid-wide task pool (Sec. V-B,
                             re-designed: DESIGN.md "Stealing").  Default 1. */
  int32_t stop_level;     /* frames < stop_level are donated (paper: 2); while more than
                             1/8 of the warps are idle every frame is.  Default 2. */
  int32_t detect_level;   /* donors look at the grid-wide pool's demand at frames < detect_level (paper:
                             idle blocks, 1).  Default 8 (every frame). */
  int32_t unroll;         /* sibling iterations expanded together, 1..32 (paper: 8);
                             0 = auto (32 with the 40-register kernel, else 16; measured).  Default 0. */
  int32_t root_chunk;     /* roots per cursor grab, 1..32; 0 = auto (1 with the 64-register kernel,
                             2 with the 40-register one; measured on B200).  Default 0. */
  int32_t block_warps;    /* warps per block, 1..32; 0 = default (32: larger blocks share work locally). */
  int32_t blocks_per_sm;  /* 0 = as many as fit (occupancy API). */
  int32_t instrument;     /* 1 = instrumented launch: count algorithmic bytes (stm_last_launch). Default 0. */
  int32_t hash_slots;     /* per-warp shared-memory hash set for operands shared by a combined set
                             operation: 0 = off, else a power of two in 64..4096 slots. Default 0.
                             Only in builds with -DSTM_WITH_HASH=1 (else STM_EUNSUPPORTED): measured slower. */
  int32_t vertex_order;   /* 0 = plans whose restrictions are order-free (STM_AUTO_RESTRICT, or none)
                             count on the graph's degree-ranked copy: same count (any total order of V
                             breaks the symmetry), far less work on skewed graphs; per-root output
                             then attributes each match to f(order[0]) minimal in (degree, id) order.
                             1 = always the caller's vertex ids.  Default 0. */
  int32_t bitmap_min_degree; /* hub adjacency bitmaps (B200 design choice):
                             every vertex of degree >= this gets an n-bit bitmap of its neighbour list
                             in HBM, and set-operation probes into its list test one bit instead of
                             binary-searching.  0 = auto (64), -1 = off.  Built lazily on the first
                             launch that uses them and cached on the graph.  Speed only. */
  int32_t bitmap_budget_mb;  /* at most this many MiB of bitmaps (highest degrees first); 0 = auto (512:
                             on C5 K6-e the same time as 2048 with half the DRAM traffic). */
  int32_t occupancy;      /* kernel register budget: 1 = 64 registers (32 warps/SM), 2 = 32 registers
                             (64 warps/SM, more DRAM latency hidden); 0 = auto: 2 when the CSR is larger
                             than half the L2.  Speed only.  Default 0. */
  int32_t root_order;     /* order in which root chunks are handed out: 1 = ascending vertex id,
                             2 = descending (heavy roots first on the degree-ranked copy), 3 = work-
                             balanced chunks interleaved light / heavy; 0 = auto (ascending).  Speed only. */
  int32_t l2_persist_mb;  /* L2 persisting access-policy window over the longest neighbour lists (the
                             tail of the degree-ranked col_idx) when the CSR does not fit in half the L2:
                             0 = auto (off: measured no gain on C5), -1 = off, else MiB (capped by the
                             device; sets the device's persisting L2 limit).  Speed only. */
  int32_t drive_ratio;    /* intersection driving side: the shorter operand drives (0 or 1); k > 1: when
                             all jobs of a combined operation share operand A (hot in L1), B drives while
                             |B| <= k |A| (coalesced reads of B, L1 probes into A).  Speed only.  Only in
                             builds with -DSTM_DRIVE_RATIO=1 (else STM_EUNSUPPORTED): measured slower. */
  int32_t narrow_split;      /* 0 = narrow neighbour lists to restriction bounds with the per-vertex split
                             out_start[v] (first neighbour > v, built at load); 1 = binary search only.
                             Speed only.  Default 0. */
  int32_t watchdog_ms;    /* failure detection: a launch still running after this many milliseconds of
                             device time aborts itself and the call reports STM_ETIMEOUT (never a partial
                             count; the async call reports it in stm_async_result.status).  0 = off.
                             Default 0. */
  int32_t backoff_max;    /* idle warps sleep up to 32 << backoff_max ns between failed steal attempts
                             (0..12); 0 = auto (8, measured).  Speed only. */
  int32_t carveout_pct;   /* shared-memory carveout of the unified L1/shared array in percent: 0 = auto
                             (just enough for the resident DFS stacks, rest to L1), -1 = driver default,
                             else 1..100.  Speed only. */
  int32_t root_split;     /* root splitting: a root of degree d is handed out as ceil(d / root_split)
                             independent pieces, piece c enumerating positions [c*root_split,
                             (c+1)*root_split) of its level-1 candidate list, so the heaviest roots are
                             spread over many warps from the start instead of being split by stealing.
                             0 = auto (512), -1 = off (one piece per root).  Speed only. */
  int32_t chunk_cost;     /* work-balanced root chunks: consecutive root entries are grouped into one
                             cursor chunk until their estimated cost (1 + candidate-list length each)
                             reaches chunk_cost, so the light bulk of a power-law graph is handed out
                             many roots per atomic and every heavy root (piece) alone.  0 = auto
                             (min(512, (n + nnz) / (8 * 48 * SMs)), at least 16: ~8 chunks per warp),
                             -1 = off (fixed root_chunk roots per chunk).  Counting launches only (not
                             listing pages).  Speed only. */
  int32_t jit;            /* plan-specialised kernels: the counting
                             kernel is compiled once more for the plan (NVRTC, a few seconds at the first
                             launch of each plan, cached for the process) with the plan and the frame as
                             compile-time constants.  0 = auto (on; the generic kernel if the compile
                             fails), 1 = required (STM_EUNSUPPORTED if it cannot be built), -1 = off.
                             Counting launches only (not instrumented, listing or census launches).
                             Speed only. */
} stm_tuning;

/* Fill t with the defaults. */
void stm_tuning_default(stm_tuning* t);

/*
 * Multi-GPU shard (duplicate the graph, divide the outermost loop).
 * The root space [0, n) is cut into chunks of `chunk` roots; chunk c belongs to
 * rank c % world.  Each rank owns one device-resident uint64 chunk cursor.  With
 * peer pointers set, a rank whose own cursor is exhausted takes chunks from the
 * peers' cursors (atomics over NVLink), so every chunk is processed exactly
 * once across the job.  All ranks must use the same world, chunk and plan.
 */
typedef struct stm_shard {
  int32_t rank, world;           /* 0 <= rank < world <= 8 */
  int32_t chunk;                 /* roots per chunk (>= 1); 0 = the launch's automatic root_chunk */
  int32_t reserved;
  uint64_t* d_cursors[8];        /* d_cursors[r] = device pointer to rank r's cursor (own entry
                                    required; peers NULL = no cross-GPU stealing).  The caller zeroes
                                    every cursor before the ranks start and keeps them alive. */
} stm_shard;

/*
 * stm_match_count -- count on the graph's device (one persistent kernel launch +
 * an 8-byte read-back, synchronous w.r.t. the host).
 *   cuda_stream  cudaStream_t to launch on, or NULL for the legacy default stream.
 *   count        receives the count (mod 2^64).
 */
stm_status stm_match_count(const stm_graph* g, const stm_plan* p, void* cuda_stream,
                           uint64_t* count);

/*
 * stm_match_count_ex -- as stm_match_count with tuning and an optional shard
 * (NULL = the whole root space).  With a shard the result is this rank's partial
 * count; the caller sums the partials (e.g. one NCCL all-reduce).
 */
stm_status stm_match_count_ex(const stm_graph* g, const stm_plan* p, const stm_tuning* t,
                              const stm_shard* shard, void* cuda_stream, uint64_t* count);

/*
 * Result record of an asynchronous count, written in DEVICE memory by the launch
 * itself (the last block to finish writes it; no extra copy is enqueued).
 */
typedef struct stm_async_result {
  uint64_t count;        /* the (partial, with a shard) count mod 2^64; meaningful only if status == 0 */
  uint64_t status;       /* 0 = OK, else the stm_status the synchronous call would have returned
                            (STM_EOVERFLOW, STM_ETIMEOUT): the count must not be used */
  uint64_t chunks;       /* root chunks this launch took from all cursors */
  uint64_t peer_chunks;  /* ... of which from peer ranks' cursors (cross-GPU stealing) */
} stm_async_result;

/*
 * stm_match_count_async -- enqueue the kernel on cuda_stream and return without
 * synchronising; the launch overwrites *d_result (device memory, 32 bytes, 8-byte
 * aligned) when it completes.  Used by the benchmark and the multi-GPU layer: the
 * all-reduce runs on d_result->count and the caller checks d_result->status
 * (summed statuses are non-zero iff some rank failed).  Host-side argument errors
 * are returned immediately; device-side failures only through d_result->status.
 */
stm_status stm_match_count_async(const stm_graph* g, const stm_plan* p, const stm_tuning* t,
                                 const stm_shard* shard, void* cuda_stream, stm_async_result* d_result);

/*
 * Chunk cursors shared across processes (multi-GPU layer, PAPER.md:164 + north_star's
 * cross-GPU stealing): every rank allocates its cursors on its own GPU and exports a
 * CUDA IPC handle; every peer maps it, so a kernel whose own cursor is exhausted takes
 * root chunks from a peer's cursor with atomics over NVLink (or, for ranks sharing one
 * GPU, in the same HBM).
 *   stm_cursors_alloc  n_slots zeroed uint64 cursors, 64 bytes apart (slot s at
 *                      d_base + 8*s words), on `device`; *ipc_handle receives
 *                      STM_IPC_HANDLE_BYTES bytes to send to the peers.
 *   stm_cursors_open   map a peer's handle into this process (on `device`); the peer's
 *                      cursors must stay allocated until stm_cursors_close.
 *   stm_cursors_close / stm_cursors_free  unmap / release.
 * Errors: STM_EINVAL (NULL out, n_slots < 1, bad device), STM_ECUDA (IPC unsupported).
 */
enum { STM_IPC_HANDLE_BYTES = 64 };
stm_status stm_cursors_alloc(int device, int n_slots, uint64_t** d_base, void* ipc_handle);
stm_status stm_cursors_open(int device, const void* ipc_handle, uint64_t** d_peer_base);
stm_status stm_cursors_close(int device, uint64_t* d_peer_base);
/* stm_cursors_reset -- zero n_slots cursors from slot first_slot of THIS process's own
   allocation, in stream order on cuda_stream (cudaMemsetAsync). */
stm_status stm_cursors_reset(int device, uint64_t* d_base, int first_slot, int n_slots, void* cuda_stream);
stm_status stm_cursors_free(int device, uint64_t* d_base);

/*
 * stm_match_count_per_root -- localisation build: host uint64[n] receives, for every
 * root vertex v, the number of counted embeddings with f(order[0]) == v
 * (order[0] = the plan's first pattern vertex, see stm_plan_describe).  Also
 * returns the total in *count.
 */
stm_status stm_match_count_per_root(const stm_graph* g, const stm_plan* p, const stm_tuning* t,
                                    void* cuda_stream, uint64_t* per_root, uint64_t* count);

/*
 * stm_match_list -- enumerate the embeddings (PAPER.md:75 and :99,
 * Output(C, iter) at the last level of the stack loop) instead of only counting them.
 *   root_begin, root_end  the page of the root space to enumerate: embeddings whose
 *                 level-0 vertex has counting id in [root_begin, root_end); [0, n)
 *                 enumerates everything.  Counting ids are the caller's vertex ids, or
 *                 (stm_tuning.vertex_order == 0 with order-free restrictions) positions in
 *                 (degree, id) order; pages of any partition of [0, n) enumerate every
 *                 embedding exactly once.
 *   out          HOST int32[capacity][k]: row i = (f(0), ..., f(k-1)) in pattern-vertex
 *                 order, caller's vertex ids, rows in no particular order.  May be NULL
 *                 when capacity == 0 (count only).
 *   n_listed     receives min(count, capacity): rows written.
 *   count        receives the number of embeddings of the page (mod 2^64).  When count >
 *                 capacity the rows are an arbitrary subset: split the page and repeat.
 * The device buffer (capacity * k * 4 bytes) is allocated and freed by the call.  Errors:
 * STM_EINVAL (bad range, NULL out with capacity > 0), STM_ENOMEM, STM_ECUDA.
 */
stm_status stm_match_list(const stm_graph* g, const stm_plan* p, const stm_tuning* t,
                          int64_t root_begin, int64_t root_end, void* cuda_stream, int32_t* out,
                          uint64_t capacity, uint64_t* n_listed, uint64_t* count);

/* stm_plan_first_vertex -- the pattern vertex matched at level 0 (order[0]). */
stm_status stm_plan_first_vertex(const stm_plan* p, int* u0);

/* Launch record of this thread's last successful stm_match_count* call. */
typedef struct stm_launch_info {
  int32_t grid;            /* persistent blocks launched (blocks/SM x SMs) */
  int32_t block_threads;
  int32_t smem_bytes;      /* dynamic shared memory per block (DFS stacks) */
  int32_t cap;             /* words per set-node region (>= max degree) */
  int64_t arena_bytes;     /* device set arena (all warps) */
  int64_t local_steals;    /* intra-block steals (Sec. V-A); synchronous calls only */
  int64_t global_steals;   /* inter-block steals (Sec. V-B); synchronous calls only */
  int64_t chunks;          /* root chunks taken from cursors; synchronous calls only */
  int64_t alg_bytes;       /* algorithmic bytes W; instrumented calls only (tuning.instrument == 1) */
  int64_t merge_bytes;     /* merge-equivalent bytes W_merge; instrumented calls only */
  int64_t jobs;            /* set operations executed; instrumented calls only */
  int32_t ranked;          /* 1 = counted on the degree-ranked copy (stm_tuning.vertex_order) */
  int32_t jit;             /* 1 = the plan-specialised kernel ran (stm_tuning.jit), 0 = the generic one */
  int64_t idle_cycles;     /* sum over warps of SM cycles spent acquiring work (root cursor, stealing,
                              waiting idle); instrumented calls only */
  int64_t warp_cycles;     /* sum over warps of their lifetime in SM cycles; instrumented calls only.
                              idle_cycles / warp_cycles = idle/stealing fraction of warps */
  int64_t hubs;            /* vertices with a hub adjacency bitmap in the counted numbering */
  int32_t variant;         /* kernel variant launched (stm_tuning.occupancy: 1 or 2) */
  int32_t unroll;          /* unroll factor used */
  int64_t peer_chunks;     /* root chunks taken from peer ranks' cursors (shard launches); synchronous calls only */
} stm_launch_info;

stm_status stm_last_launch(stm_launch_info* info);

/*
 * stm_last_profile -- per-phase cycle buckets of this thread's last synchronous call,
 * filled only by libraries built with -DSTM_PROFILE=1 (A/B builds; zeros otherwise).
 * out receives min(n, 114) uint64: for phase i in 0..11 (root gather, root sibling
 * set-up, candidate gather, set-node build, frame count, fused count, donate,
 * work acquisition, next-sibling set-up, descend set-up, combined-operation set-up,
 * combined-operation element loop) the triple (warp cycles, calls, items), then
 * the summed and the maximal warp lifetime, the summed and the maximal time (from
 * the warp's start) at which the root cursors were first seen exhausted; then for
 * kind in (candidate pre-test, set build, count) and level 0..7 the triple (warp
 * cycles, combined operations, driven elements); then the longest time one warp held a
 * single task (root chunk or stolen work, cycles) and a reserved word.
 */
stm_status stm_last_profile(uint64_t* out, int n);

/* ---------------------------------------------------------------------------------------
 * Cost-based matching order.  PAPER.md:151: STMatch adopts
 * Dryadic's matching order; PAPER.md:52 requires only that every pi[l] after the first
 * be adjacent to an earlier one.  The order changes the work, never the count.  These
 * calls are host-only (no CUDA) and choose the `order` argument of stm_pattern_compile
 * from degree / label statistics of the data graph (cost model: DESIGN.md reading R15).
 * ------------------------------------------------------------------------------------- */
enum { STM_STATS_MOMENTS = 9, STM_STATS_LABELS = 256 };

typedef struct stm_graph_stats {
  int64_t n;                                /* vertices */
  int64_t nnz;                              /* directed adjacency entries (2m) */
  double moment[STM_STATS_MOMENTS];         /* moment[j] = (1/n) sum_v w(v)^j, w(v) = min(d(v), sqrt(nnz)) */
  int32_t n_labels;                         /* distinct vertex labels (0 = unlabeled graph) */
  int32_t reserved;
  int32_t label_value[STM_STATS_LABELS];    /* ascending label values */
  double label_freq[STM_STATS_LABELS];      /* fraction of vertices carrying label_value[i] */
} stm_graph_stats;

/*
 * stm_graph_stats_host -- degree moments and label frequencies of a host CSR (the same
 * row_ptr / labels arrays stm_graph_load takes; col_idx is not needed).  O(n).
 * Caller owns `out`.  Errors: STM_EINVAL (NULL out, n < 0, decreasing row_ptr,
 * negative label), STM_EUNSUPPORTED (> 256 distinct labels).
 */
stm_status stm_graph_stats_host(int64_t n, const int64_t* row_ptr, const int32_t* labels,
                                stm_graph_stats* out);

/*
 * stm_graph_get_stats -- the statistics of a loaded graph (computed by stm_graph_load /
 * stm_graph_load_device exactly as stm_graph_stats_host does), so callers get the
 * cost-based order without keeping host arrays: stm_motif_census uses them by default.
 * Errors: STM_EINVAL (NULL), STM_EUNSUPPORTED (graph with > 256 distinct labels).
 */
stm_status stm_graph_get_stats(const stm_graph* g, stm_graph_stats* out);

/*
 * stm_order_cost -- model cost of matching `order` (int32[k], a connected permutation)
 * for the pattern (k, edges, labels, restrictions, flags exactly as stm_pattern_compile
 * takes them; STM_AUTO_RESTRICT uses the compiler's Grochow-Kellis set) on a graph with
 * statistics `stats`.  *cost = expected merge work (n + sum over levels of estimated
 * prefixes x summed operand list lengths); *est_count = estimated number of counted
 * embeddings (Chung-Lu expectation of homomorphisms, label and restriction factors).
 * Either output may be NULL.  Errors: those of stm_pattern_compile; STM_EINVAL for a
 * NULL stats / order or an order that is not a connected permutation.
 */
stm_status stm_order_cost(int k, int n_edges, const int32_t* edges, const int32_t* labels, int n_restr,
                          const int32_t* restr, uint32_t flags, const stm_graph_stats* stats,
                          const int32_t* order, double* cost, double* est_count);

/*
 * stm_order_optimize -- the connected order of minimal model cost (exhaustive over the
 * <= 8! permutations); the compiler's greedy order is kept unless that minimum is at
 * least 10% below the greedy order's cost (near-ties are not ranked by the model),
 * and always for trees (|E| = k - 1; measured).  Writes int32[k] to order_out (caller-owned); cost / est_count as in
 * stm_order_cost (may be NULL).  Errors as stm_order_cost.
 */
stm_status stm_order_optimize(int k, int n_edges, const int32_t* edges, const int32_t* labels, int n_restr,
                              const int32_t* restr, uint32_t flags, const stm_graph_stats* stats,
                              int32_t* order_out, double* cost, double* est_count);

/* ---------------------------------------------------------------------------------------
 * Motif census (many patterns per graph).
 * ------------------------------------------------------------------------------------- */

/*
 * stm_motif_catalog -- the connected graphs on k vertices up to isomorphism, 2 <= k <= 6
 * (1, 2, 6, 21, 112 motifs for k = 2..6), host only.  Motif i has n_edges[i] edges
 * written as vertex pairs (a < b) to edges[i * k*(k-1) + 2e + {0,1}]; motifs are sorted
 * by edge count, then by canonical edge mask.  At most `capacity` motifs are written;
 * *n_motifs receives the full number (call with capacity 0 to size the arrays).
 * Errors: STM_EUNSUPPORTED (k outside 2..6), STM_EINVAL (NULL n_motifs, NULL arrays
 * with capacity > 0).
 */
stm_status stm_motif_catalog(int k, int capacity, int32_t* n_edges, int32_t* edges, int* n_motifs);

/*
 * stm_motif_census -- count every motif of stm_motif_catalog(k) in g, in catalog order,
 * as distinct subgraphs (Grochow-Kellis restrictions).  flags: 0 (edge-induced) or
 * STM_VERTEX_INDUCED (induced motif frequencies; they sum to the number of connected
 * induced k-vertex subsets), optionally | STM_NO_CODE_MOTION / STM_LAZY_UNBOUNDED.
 * stats: graph statistics (stm_graph_stats_host) to give each motif its cost-based
 * order (stm_order_optimize), or NULL for the graph's own statistics (stm_graph_get_stats);
 * flags | STM_AUTO_ORDER keeps the compiler's greedy order.  Counts are the same either way.
 * Pattern merging: the motif plans are merged into one trie of matching
 * levels -- motifs whose levels 0..d have the same candidate sources, filters and set-node
 * definitions share one DFS frame and every set built on the way -- and the whole census
 * is ONE persistent launch of the merged-plan kernel (a group whose merged plan exceeds
 * the kernel's per-level limits is split into halves, one launch each;
 * stm_motif_census_launches reports how many).  flags | STM_CENSUS_PER_MOTIF instead runs
 * one counting launch per motif (the A/B baseline).  Synchronous on `cuda_stream`; t may be
 * NULL (defaults).  counts: caller-owned uint64[capacity], capacity >= the catalog size.
 * Errors: as stm_motif_catalog and stm_match_count_ex; STM_EINVAL for other flag bits or a
 * short capacity.
 */
stm_status stm_motif_census(const stm_graph* g, int k, uint32_t flags, const stm_graph_stats* stats,
                            const stm_tuning* t, void* cuda_stream, int capacity, uint64_t* counts,
                            int* n_motifs);

/* stm_motif_census_launches -- counting launches of this thread's last stm_motif_census. */
stm_status stm_motif_census_launches(int* launches);

/*
 * stm_motif_merge_stats -- shape of the merged trie of the size-k census (greedy orders,
 * flags & STM_VERTEX_INDUCED): trie vertices per depth (int[k]), pool set nodes and
 * per-warp set regions.  STM_EUNSUPPORTED when one merged launch cannot hold the census.
 */
stm_status stm_motif_merge_stats(int k, uint32_t flags, int* verts_per_depth, int* n_nodes, int* n_regions);

/* stm_last_error -- thread-local message for the last non-OK status of this thread. */
const char* stm_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* STM_H_ */
