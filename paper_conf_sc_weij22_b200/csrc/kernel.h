// kernel.h -- launch interface between the runtime (runtime.cu) and the persistent
// matching kernel (kernel.cu).  Product code only.
#pragma once
#ifndef STM_NVRTC  // (JIT compiles get the fixed-width types from stm_nvrtc_prelude.h)
#include <stdint.h>

#include <cuda_runtime.h>  // int4
#endif

#include "plan.h"

// ---------------------------------------------------------------------------------
// Merged multi-pattern plan (motif census; "pattern merging",
// PAPER.md:25): the per-pattern plans are merged into a trie of matching levels.  A
// trie vertex at depth d stands for every pattern whose levels 0..d are identical
// (candidate source, filter, need, and the definitions of the set nodes they read);
// its children are the distinct continuations.  The set nodes needed below a vertex
// are built once per prefix when v_d is chosen (the union over its subtree, shared
// by every pattern under it), and the leaves (depth k-1) carry each pattern's final
// counting operation.  Built by motif.cpp, read by the STM_MULTI build of kernel.cu.
struct StmMNode {     // a set node of the merged plan (StmNode fields + storage region)
  StmNode nd;         // nd.a = pool index when nd.a_kind == STM_SRC_NODE
  int16_t region;     // arena region / NOFF row of the node
  int16_t pad;
};
struct StmMVert {
  int16_t depth;
  int16_t child_begin, n_children;   // children are vertices [child_begin, child_begin + n_children)
  int16_t build_begin, n_build;      // pool nodes [build_begin, +n_build) of level depth+1, by stage
  int8_t n_stages;
  int8_t need;
  StmSrc cand;                       // candidate source of level `depth` (leaves: the counted operand A)
  StmFilter filt;                    // filter of level `depth`
  int8_t cnt_b, cnt_op;              // leaves: count |A op N(v_cnt_b)|
  int16_t motif;                     // leaves: pattern index (output slot)
};

// A unit of stealable work (Sec. V).  level 0: root-ID range
// [b, e).  level l >= 1: the prefix v_0..v_{l-1} (prefix[0..l-1]) and the
// positions [b, e) of the level-l candidate list of that prefix.  The candidate
// list is a sorted set determined by the prefix alone, so the receiver rebuilds
// the sets of levels 1..l from the prefix instead of copying them (DESIGN.md,
// "Stealing": differs from PAPER.md:142, which copies the sets).
struct StmTask {
  int32_t level;
  int32_t b, e;
  int32_t prefix[STM_KMAX];
  int16_t tv[STM_KMAX];   // STM_MULTI: trie vertex of each level 0..level on the stolen path
};

// phases of the STM_PROFILE build: 0 gather_roots, 1 root set_sibling, 2 gather_batch,
// 3 build_nodes, 4 frame_count, 5 fused_count, 6 maybe_donate, 7 acquire_work,
// 8 next-sibling set_sibling, 9 descend set_sibling, 10 run_jobs set-up (operand
// narrowing), 11 run_jobs element loop (probes + compaction)
#define STM_PROF_N 12
// STM_PROFILE builds also keep, per level l (0..7) and kind (0 pre-test, 1 set build,
// 2 count), the triple (warp cycles, combined operations, driven elements)
#define STM_PROF_LVL (3 * 3 * 8 + 2)  // + (longest busy interval between sharing checks, spare)
// STM_PROFILE builds also keep a timeline: busy warp-nanoseconds per 0.5 ms bucket of the
// launch (%globaltimer since each warp's start), 64 buckets
#define STM_PROF_TL 64
#define STM_PROF_TL_NS 500000
#define STM_PROF_SIZE (3 * STM_PROF_N + 4 + STM_PROF_LVL + STM_PROF_TL)

// Device-resident scheduler state of one launch (zeroed before every launch).
struct StmWork {
  unsigned long long count;       // result accumulator (mod 2^64)
  // Termination and the grid-wide task pool (kernel.cu acquire_work): `active` counts busy
  // warps + queued pool tasks + claimed local donations; once every warp has started
  // (`started` == all warps) and `active` is 0 no work can appear any more.  `deficit` =
  // block pollers waiting for pool work - queued tasks: a donor pushes only after claiming
  // a unit of it, so the pool never holds more tasks than there are blocks.
  int32_t active, started, deficit;
  int32_t overflow;               // 1: a capacity check failed, 2: the watchdog expired (no count)
  unsigned long long pool_head, pool_tail;  // tasks popped / pushed so far (tickets)
  unsigned long long n_local_steals, n_global_steals, n_chunks;
  unsigned long long n_peer_chunks;  // chunks taken from peer ranks' cursors
  unsigned int blocks_done;          // blocks that finished (the last one writes the async result)
  unsigned int pad0;
  unsigned long long alg_bytes;    // SURVEY.md 8(d) W = sum W_op (instrumented launches only)
  unsigned long long merge_bytes;  // W_merge = sum 4(|A|+|B|)
  unsigned long long n_jobs;
  unsigned long long idle_cycles;  // sum over warps of cycles spent acquiring work (instrumented)
  unsigned long long warp_cycles;  // sum over warps of their lifetime in cycles (instrumented)
  unsigned long long list_n;       // listing build: embeddings found (slots taken) so far
  unsigned long long prof[STM_PROF_SIZE];  // STM_PROFILE builds: (cycles, calls, items) per phase, summed
                                                // lifetime, max lifetime, summed / max time cursors ran dry
};

struct StmPoolSlot {              // one slot of the grid-wide task pool (64 bytes)
  int32_t seq;                    // 2r: free for the r-th round of tickets on this slot, 2r+1: holds it
  StmTask task;
};
static_assert(sizeof(StmPoolSlot) == 64, "pool slot layout");

struct StmKParams {
  StmPlan plan;
  const int4* vrec;               // [n] packed (row start, degree, out_start, hub slot), kernel.cu vrec()
  const int32_t* col_idx;
  const uint8_t* labels;          // dense graph label ids, or NULL
  // Hub adjacency bitmaps: vrec[v].w >= 0 selects the
  // n-bit row bitmaps[slot * bm_words ...] of N(v); membership probes into such a
  // row read one word instead of a binary search.
  int32_t split;                  // 1: narrow rows with the out_start split of vrec (stm_tuning.narrow_split 0)
  const uint32_t* bitmaps;
  int64_t bm_words;
  // Root entries: when set, the root space [root_lo, n) indexes
  // entries[] = (root vertex, chunk c) and level 1 of that entry enumerates only positions
  // [c * root_split, (c + 1) * root_split) of the root's candidate list, so a heavy root is
  // handed out as several independent pieces from the start.  NULL: root space = vertex ids.
  const int2* entries;
  int32_t root_split;
  int32_t n_dir;                  // directed graphs: vertex v's in-row is record v + n_dir (= n); 0 otherwise
  // Work-balanced chunks (stm_tuning.chunk_cost): chunk c is root-space positions
  // [chunk_bounds[c], chunk_bounds[c + 1]); NULL: fixed chunks of `chunk` positions.
  const int32_t* chunk_bounds;
  int64_t n_chunks;
  int64_t n;                      // root space end: roots are [root_lo, n)
  int64_t root_lo;
  int32_t* list_out;              // listing build: [list_cap][k] rows (pattern-vertex order)
  unsigned long long list_cap;
  int32_t cap;                    // words per set-node region per warp
  int32_t block_warps;
  int32_t* arena;                 // [total_warps][n_nodes][cap]
  StmWork* work;
  StmPoolSlot* pool;              // [pool_mask + 1] task pool (global work sharing)
  int32_t pool_mask, pool_shift;  // capacity - 1, log2(capacity)
  int32_t total_warps;            // warps of the launch (termination: StmWork::started)
  unsigned long long* per_root;   // [n] or NULL (indexed by the caller's vertex id)
  const int32_t* root_map;        // counting id -> caller's id (degree-ranked copy), or NULL
  unsigned long long* cursors[8]; // chunk cursors (own rank + optional peers)
  int32_t rank, world, chunk;
  int32_t root_desc;              // 1: chunk c covers the root ids [n-(c+1)chunk, n-c*chunk) (descending);
                                  // 2: work-balanced chunks interleaved light / heavy (c even: c/2, odd: from the end)
  int32_t local_steal, global_steal, stop_level, detect_level, unroll, root_batch;
  int32_t count_bytes;            // 1 = accumulate algorithmic bytes (instrumented launch)
  int32_t ht_slots;               // per-warp shared-memory hash slots (0 = off)
  int32_t donate_mask;            // donors look for idle blocks every (mask+1)-th opportunity
  int32_t drive_ratio;            // drive B while |B| <= drive_ratio |A| when A is shared by all jobs (0/1 = shorter)
  int32_t backoff_max;            // idle warps sleep up to 32 << backoff_max ns between steal attempts
  long long watchdog_ns;          // abort (work->overflow = 2) after this much %globaltimer time; 0 = off
  unsigned long long* result;     // stm_async_result {count, status, chunks, peer_chunks} or NULL
  const void* l2_window_base;     // L2 persisting access-policy window (0 bytes = none)
  long long l2_window_bytes;
  uint8_t lab2slot[256];          // dense graph label -> pattern label-slot bitmask
  // STM_MULTI (merged census) launches: the trie and node pool, per-pattern counts
  const StmMVert* mv;
  const StmMNode* mn;
  unsigned long long* mcount;     // [n_patterns] counts (zeroed by the host)
};

#ifndef STM_NVRTC  // host-side launch interface (not part of a JIT compile)
// 1 if the shared-memory hash-set path is compiled in (-DSTM_WITH_HASH=1)
int stm_hash_compiled();
// 1 if the drive_ratio operand choice is compiled in (-DSTM_DRIVE_RATIO=1)
int stm_drive_compiled();
// size in bytes of the dynamic shared memory for one block
int stm_smem_bytes(int block_warps, int k, int n_nodes, int ht_slots);
// kernel variants (register budgets): 1 = 64 registers, 2 = 32 registers (more warps)
// launches the persistent kernel (cooperative); returns cudaError_t as int
int stm_launch(int variant, const StmKParams& kp, int grid, void* stream);
int stm_launch_instr(int variant, const StmKParams& kp, int grid, void* stream);  // instrumented build
int stm_launch_list(int variant, const StmKParams& kp, int grid, void* stream);   // listing build
int stm_launch_multi(int variant, const StmKParams& kp, int grid, void* stream);  // merged census build
// max co-resident blocks per SM for the given block size
// carveout: stm_tuning.carveout_pct (0 = auto, -1 = driver default, else percent)
int stm_occupancy(int variant, int block_warps, int k, int n_nodes, int ht_slots, int carveout, int* blocks_per_sm);
// the same for a given kernel: a plan-specialised JIT kernel (cudaKernel_t), runtime.cu jit_kernel
int stm_occupancy_fn(const void* fn, int block_warps, int k, int n_nodes, int ht_slots, int carveout,
                     int* blocks_per_sm);
int stm_launch_fn(const void* fn, const StmKParams& kp, int grid, void* stream);
int stm_occupancy_instr(int variant, int block_warps, int k, int n_nodes, int ht_slots, int carveout,
                        int* blocks_per_sm);
int stm_occupancy_list(int variant, int block_warps, int k, int n_nodes, int ht_slots, int carveout,
                       int* blocks_per_sm);
int stm_occupancy_multi(int variant, int block_warps, int k, int n_nodes, int ht_slots, int carveout,
                        int* blocks_per_sm);
int stm_smem_bytes_multi(int block_warps, int k, int n_regions);
#endif  // !STM_NVRTC
