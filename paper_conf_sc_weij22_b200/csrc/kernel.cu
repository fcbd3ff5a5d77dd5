// kernel.cu -- the single persistent sm_100a matching kernel (product hot path).
//
// One launch runs the whole backtracking ("finish the computation with
// one kernel launch").  Every warp runs the stack-based while-loop of Fig. 3
// on its own DFS stack kept in shared memory; the candidate
// sets (the paper's C arrays) live in a per-warp global arena sized from the
// graph's true maximum degree (PAPER.md:154 used a fixed MAX_DEGREE=4096; reading
// R11).  Level 0 takes chunks of root vertices from a global atomic cursor
// (Fig. 4).
//
// Set operations: a *job* is one "A op N(v)" with op in
// {intersect, difference}, or a filtered scan.  Up to 32 jobs --
// the sets of several unrolled sibling iterations (Sec. VI, Fig. 7)
// or, at the last level, the counts of many candidates -- are flattened into one
// element stream that the warp walks 32 elements at a time: an inclusive scan of
// job sizes, a per-lane job lookup, a binary search of the element in the probed
// sorted list, then ballot/popc compaction into the output set (the combined set
// operation of Fig. 8).  For an intersection the shorter operand
// drives and the longer one is probed; value bounds from symmetry-breaking
// restrictions first narrow both operands by binary search.  The last level is
// counted and never materialised.
//
// Load balance (Sec. V): intra-block stealing through shared memory (Sec. V-A,
// PAPER.md:84) and inter-block stealing through per-block global mailboxes pushed
// by busy donors (Sec. V-B, Fig. 6).  Stolen work is a task
// (prefix, position range); the thief rebuilds the prefix's sets itself.
#ifdef STM_NVRTC
// plan-specialised JIT compile (runtime.cu jit_kernel, NVRTC): device code only
#include "stm_nvrtc_prelude.h"
#else
#include <algorithm>
#include <climits>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstdint>

#include <cuda_runtime.h>
#endif

#include "kernel.h"

#define FULLMASK 0xffffffffu
// A/B build switches (tools/gpu_variants.sh); the defaults are the measured best.
#ifndef STM_JOBS_INLINE
#define STM_JOBS_INLINE 1   // 0: one out-of-line copy of run_jobs (smaller code, W in local memory)
#endif
#ifndef STM_MAXT
#define STM_MAXT 1024       // __launch_bounds__ max threads: 1024 -> 64 registers, 512 -> 128
#endif
#ifndef STM_STEP_NOINLINE
#define STM_STEP_NOINLINE 0 // 1: build_nodes / gather_batch / fused_count out of line
#endif
#if STM_JOBS_INLINE
#define JOBS_INL __forceinline__
#else
#define JOBS_INL __noinline__
#endif
#if STM_STEP_NOINLINE
#define STEP_INL __noinline__
#else
#define STEP_INL
#endif
#ifndef STM_HDR_SYNC
#define STM_HDR_SYNC 1  // __syncwarp() between the lanes' reads of a stack-header field and lane 0's rewrite
#endif
#if STM_HDR_SYNC
#define HDR_SYNC() __syncwarp()
#else
#define HDR_SYNC() ((void)0)
#endif
#ifndef STM_GATHER_SLOW_NOINLINE
#define STM_GATHER_SLOW_NOINLINE 0  // 1: the per-candidate admission path out of line (A/B)
#endif
#if STM_GATHER_SLOW_NOINLINE
#define GATHER_SLOW_INL __noinline__
#else
#define GATHER_SLOW_INL __forceinline__
#endif
#ifndef STM_OCC_MAXT
#define STM_OCC_MAXT 2048   // __launch_bounds__ of the high-occupancy variant (32 registers, 64 warps/SM)
#endif
#ifndef STM_INSTR
#define STM_INSTR 0         // 1: the instrumented build (kernel_instr.cu): algorithmic-byte / idle counters
#endif
#ifndef STM_LIST
#define STM_LIST 0          // 1: the listing build (kernel_list.cu): last level emits embeddings (NEXT-1)
#endif
#ifndef STM_MULTI
#define STM_MULTI 0         // 1: the merged-census build (kernel_multi.cu): a trie of patterns (NEXT-3)
#endif
#if STM_INSTR
#define STM_SYM(x) x##_instr
#elif STM_LIST
#define STM_SYM(x) x##_list
#elif STM_MULTI
#define STM_SYM(x) x##_multi
#else
#define STM_SYM(x) x
#endif
#ifndef STM_ELEM_NOINLINE
#define STM_ELEM_NOINLINE 1 // 1: run_jobs' element loop is one out-of-line function (i-cache)
#endif
#ifndef STM_BM_CS
#define STM_BM_CS 0         // 1: hub-bitmap probes as streaming loads (L2 evict-first): K6-e -3 % time
                            //    but +17 % DRAM traffic (fewer L2 hits on re-probed words) -- off
#endif
#if STM_BM_CS
#define STM_BM_LOAD(p) __ldcs(p)
#else
#define STM_BM_LOAD(p) __ldg(p)
#endif
#ifndef STM_BATCH_ELEMS
#define STM_BATCH_ELEMS 0   // > 0: admit siblings into a batch only while the summed set-size
#endif                      //    bounds stay within this many elements (0: the arena region)
#ifndef STM_DEEP_FRAC
#define STM_DEEP_FRAC 8     // every frame is donated while more than 1/STM_DEEP_FRAC of the warps idle
#endif
#ifndef STM_GCHK_CYCLES
#define STM_GCHK_CYCLES 4096  // busy warps look at the pool's demand at most this often (SM cycles)
#endif
#ifndef STM_ELEM_INLINE_MAX
#define STM_ELEM_INLINE_MAX 0  // element streams up to this long run the inline copy instead
#endif
#ifndef STM_CPLAN
#define STM_CPLAN 0         // 1: plan-specialised build: the plan is the compile-time record of
#endif                      //    STM_CPLAN_HEADER (tools/cplan.py) instead of kp.plan
#ifndef STM_DEBUG
#define STM_DEBUG 0         // 1: watchdog state dumps (printf)
#endif
#ifndef STM_PROFILE
#define STM_PROFILE 0       // 1: per-phase clock64() buckets (stm_last_profile); A/B builds only
#endif
#if STM_PROFILE
#define PROF_BEGIN(id) const long long prof_t##id = clock64();
#define PROF_END(id, items)                                    \
  if (w.lane == 0) {                                           \
    w.prof_cyc[id] += (unsigned long long)(clock64() - prof_t##id); \
    w.prof_cnt[id] += 1;                                       \
    w.prof_items[id] += (unsigned long long)(items);           \
  }
// per-level buckets: kind 0 pre-test, 1 set build, 2 count (level = the level computed)
#define PROF_LVL_BEGIN() const long long prof_lt = clock64();
#define PROF_LVL_END(kind, lvl)                                                                       \
  if (w.lane == 0) {                                                                                \
    unsigned long long* pl = &w.kp->work->prof[3 * STM_PROF_N + 4 + 3 * (8 * (kind) + (lvl))];        \
    atomicAdd(pl, (unsigned long long)(clock64() - prof_lt));                                       \
    atomicAdd(pl + 1, 1ull);                                                                        \
    atomicAdd(pl + 2, (unsigned long long)w.last_total);                                            \
  }
// longest busy interval between two work-sharing checks: the indivisible unit of work
// (the critical path a split can never shorten)
#define PROF_CHK()                                                                      \
  if (w.lane == 0) {                                                                    \
    const long long now_ = clock64();                                                   \
    if (w.prof_chk)                                                                     \
      atomicMax(&w.kp->work->prof[3 * STM_PROF_N + 4 + STM_PROF_LVL - 2],               \
                (unsigned long long)(now_ - w.prof_chk));                               \
    w.prof_chk = now_;                                                                  \
    prof_timeline(w);                                                                   \
  }
#else
#define PROF_BEGIN(id)
#define PROF_END(id, items)
#define PROF_LVL_BEGIN()
#define PROF_LVL_END(kind, lvl)
#define PROF_CHK()
#endif

namespace {

struct WarpHdr {
  // Local work sharing: an idle warp sets its bit in
  // BlockHdr::idle_mask and waits; a busy warp of the block that sees the bit claims
  // it (clears it with an atomic), splits its OWN stack and posts the task here.  Only
  // the owner ever reads or writes a stack, so the busy path takes no locks.
  int mail_full;              // 1 when `mail` holds a task donated to this warp
  int L;                      // current frame (0 = root level)
  int root_it, root_end;      // frame 0: remaining root-ID range of the current chunk
  int nsib[STM_KMAX], cur[STM_KMAX], it[STM_KMAX], end[STM_KMAX];
  int used[STM_MAX_NODES];    // words used in each node region by the frame being built
  int stage_c[32], stage_u[32];
  // per-warp scheduler state kept here (not in registers) so that the cold, out-of-line
  // work-acquisition functions need no reference to the warp's register state
  unsigned exhausted;         // cursors known to be exhausted (bit per rank)
  unsigned donate_tick;
  int steal_fails;
  int pad0;
  long long first_dry;        // STM_PROFILE: clock64() when the root cursors were first seen exhausted
  long long gchk;             // clock64() of the last look at the pool's demand
  long long wd0;              // %globaltimer at the warp's start (watchdog)
  int deep;                   // 1: donate from every frame (grid starving, split_stop)
  int pad1;
  // STM_MULTI: frame F iterates the virtual siblings vs = child * nr[F] + u, u < nr[F]
  // the real sibling (value of v_{F-1}) and child the child of trie vertex pv[F] whose
  // candidates are enumerated (child-major: consecutive virtual siblings share a child,
  // so the last level's counts pack up to 32 (sibling, candidate) pairs of one child)
  int pv[STM_KMAX], nr[STM_KMAX];
  int rent[STM_RMAX];         // root entries (kp.entries): entry index of frame-1 sibling u
  StmTask mail;               // the donated task (valid while mail_full == 1)
};

struct BlockHdr {
  int idle_mask;              // warps idle and waiting for a donation (bit per warp)
  int poller;                 // the idle warp that polls the grid-wide pool (-1: none)
  int done;
  int pad;
  unsigned char lab2slot[256];
};

__host__ __device__ constexpr int warp_bytes_fixed() { return (int)sizeof(WarpHdr); }
__host__ __device__ inline int warp_bytes(int k, int n_nodes, int ht_slots) {
  int b = warp_bytes_fixed() + k * STM_RMAX * 4 + 2 * n_nodes * STM_UMAX * 4 + ht_slots * 4;
  return (b + 15) & ~15;
}

// The warp's view of the launch: pointers into the grid-constant parameters and the
// warp's shared-memory stack.  It is rebuilt from threadIdx by make_w() wherever it is
// needed and never passed by reference to an out-of-line function, so that it stays in
// registers (an escaping W lives in local memory and turns every stack-header access
// into a generic load).
struct W {
  const StmKParams* kp;
  const StmPlan* P;
  volatile WarpHdr* h;
  volatile int* sib;   // [k][RMAX]
  int* noff;           // [n_nodes][UMAX]
  int* nsz;            // [n_nodes][UMAX]
  BlockHdr* bh;
  int* arena;
  int lane, wid;
  unsigned long long cnt;
  unsigned long long wbytes, wmerge, wjobs;  // per-lane instrumentation partials
  unsigned long long idle_cyc;               // cycles in acquire_work (instrumented launches)
#if STM_PROFILE
  unsigned long long prof_cyc[STM_PROF_N], prof_cnt[STM_PROF_N], prof_items[STM_PROF_N];
  int last_total;  // elements driven by the last combined operation
  long long prof_chk;  // clock64() of the last work-sharing check (0: idle since)
  long long prof_g;    // %globaltimer of the last check (0: idle since)
  int prof_b;          // timeline bucket being accumulated in prof_acc
  unsigned long long prof_acc;
#endif
};

extern __shared__ __align__(16) unsigned char stm_smem[];

#if STM_CPLAN
// The plan as a constant initialised global: every load from it at a constant offset folds
// to an immediate (frame_step<F> makes the frame a constant, the node loops unroll).
union StmPlanBytes {
  unsigned char b[sizeof(StmPlan)];
  StmPlan p;
};
#include STM_CPLAN_HEADER  // __device__ const StmPlanBytes kCPlan = {{...}};
#define STM_PLAN_OF(kp) (kCPlan.p)
#else
#define STM_PLAN_OF(kp) ((kp).plan)
#endif

__device__ __forceinline__ W make_w(const StmKParams& kp) {
  const StmPlan& P = STM_PLAN_OF(kp);
  W w;
  w.kp = &kp;
  w.P = &P;
  w.lane = threadIdx.x & 31;
  w.wid = threadIdx.x >> 5;
  const int wb = warp_bytes(P.k, P.n_nodes, kp.ht_slots);
  unsigned char* wbase = stm_smem + sizeof(BlockHdr) + (size_t)w.wid * wb;
  w.bh = (BlockHdr*)stm_smem;
  w.h = (volatile WarpHdr*)wbase;
  w.sib = (volatile int*)(wbase + sizeof(WarpHdr));
  w.noff = (int*)(wbase + sizeof(WarpHdr) + P.k * STM_RMAX * 4);
  w.nsz = w.noff + P.n_nodes * STM_UMAX;
  const long long gw = (long long)blockIdx.x * kp.block_warps + w.wid;
  w.arena = kp.arena + (size_t)gw * (size_t)P.n_nodes * (size_t)kp.cap;
  w.cnt = 0;
  w.wbytes = w.wmerge = w.wjobs = 0;
  w.idle_cyc = 0;
#if STM_PROFILE
  for (int i = 0; i < STM_PROF_N; ++i) w.prof_cyc[i] = w.prof_cnt[i] = w.prof_items[i] = 0;
  w.prof_chk = 0;
  w.prof_g = 0;
  w.prof_b = 0;
  w.prof_acc = 0;
#endif
  return w;
}

#if STM_PROFILE
// busy time since the last check, credited to the timeline bucket of now (lane 0)
__device__ __forceinline__ void prof_timeline(W& w) {
  long long g;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g));
  if (w.prof_g) {
    const int b = (int)((g - w.h->wd0) / STM_PROF_TL_NS);
    if (b != w.prof_b) {
      if (w.prof_acc && w.prof_b >= 0 && w.prof_b < STM_PROF_TL)
        atomicAdd(&w.kp->work->prof[3 * STM_PROF_N + 4 + STM_PROF_LVL + w.prof_b], w.prof_acc);
      w.prof_acc = 0;
      w.prof_b = b;
    }
    w.prof_acc += (unsigned long long)(g - w.prof_g);
  }
  w.prof_g = g;
}
__device__ __forceinline__ void prof_timeline_flush(W& w) {
  if (w.lane == 0 && w.prof_acc && w.prof_b >= 0 && w.prof_b < STM_PROF_TL)
    atomicAdd(&w.kp->work->prof[3 * STM_PROF_N + 4 + STM_PROF_LVL + w.prof_b], w.prof_acc);
  w.prof_acc = 0;
}
#endif

// donor sides of local / global work sharing (defined with the scheduler below)
__device__ __noinline__ void share_local(const StmKParams& kp);
__device__ __noinline__ void maybe_push(const StmKParams& kp);
__device__ __noinline__ bool watchdog(const StmKParams& kp, long long t0, const char* where);

// instrumented builds: add a W's per-lane algorithmic-byte partials to the launch totals
__device__ __forceinline__ void flush_instr(W& w) {
  if (STM_INSTR && w.kp->count_bytes) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      w.wbytes += __shfl_xor_sync(FULLMASK, w.wbytes, o);
      w.wmerge += __shfl_xor_sync(FULLMASK, w.wmerge, o);
      w.wjobs += __shfl_xor_sync(FULLMASK, w.wjobs, o);
    }
    if (w.lane == 0) {
      atomicAdd(&w.kp->work->alg_bytes, w.wbytes);
      atomicAdd(&w.kp->work->merge_bytes, w.wmerge);
      atomicAdd(&w.kp->work->n_jobs, w.wjobs);
    }
    w.wbytes = w.wmerge = w.wjobs = 0;
  }
}

#define SIB(w, l, u) ((w).sib[(l) * STM_RMAX + (u)])
#define NOFF(w, s, u) ((w).noff[(s) * STM_UMAX + (u)])
#define NSZ(w, s, u) ((w).nsz[(s) * STM_UMAX + (u)])

__device__ __forceinline__ int bcast(int x) { return __shfl_sync(FULLMASK, x, 0); }

// Branchless binary searches (a select per probe, ceil(log2 n) dependent loads):
// lbound = #elements < x; member = x in a.  Lanes with equal n stay converged.
__device__ __forceinline__ int lbound(const int* __restrict__ a, int n, int x) {
  if (n <= 0) return 0;
  const int* base = a;
#pragma unroll 1
  while (n > 1) {
    const int half = n >> 1;
    base = (base[half] < x) ? base + half : base;
    n -= half;
  }
  return (int)(base - a) + (*base < x);
}

__device__ __forceinline__ bool member(const int* __restrict__ a, int n, int x) {
  if (n <= 0) return false;
  const int* base = a;
#pragma unroll 1
  while (n > 1) {
    const int half = n >> 1;
    base = (base[half] <= x) ? base + half : base;
    n -= half;
  }
  return *base == x;
}

// Packed per-vertex record (StmKParams::vrec, built at the first launch per numbering and
// hub set): x = row start in col_idx, y = degree, z = out_start (index of the first
// neighbour > v, -1 = unknown), w = hub bitmap slot (-1 = none) -- one 16-byte load
// instead of row_ptr[v], row_ptr[v+1], out_start[v] and hub_slot[v] from four arrays.
__device__ __forceinline__ int4 vrec(const W& w, int v) { return __ldg(w.kp->vrec + v); }
// raw neighbour lists by position code (plan.h): dir 1 = the in-row of a directed graph
// (its records follow the n out-row records, StmKParams::n_dir)
__device__ __forceinline__ void row(const W& w, int v, const int*& p, int& len, int dir = 0) {
  const int4 r = vrec(w, v + (dir ? w.kp->n_dir : 0));
  p = w.kp->col_idx + (unsigned)r.x;
  len = r.y;
}
__device__ __forceinline__ int degree(const W& w, int v, int dir = 0) { return vrec(w, v + (dir ? w.kp->n_dir : 0)).y; }

// ----------------------------------------------------------------------------
// plan access.  Single-pattern builds read the StmPlan; the STM_MULTI build reads the
// merged trie (kernel.h StmMVert / StmMNode), where frame F's current sibling index
// is virtual (real sibling * children + child).
// ----------------------------------------------------------------------------
#if STM_MULTI
__device__ __forceinline__ const StmMVert& mvert(const W& w, int t) { return w.kp->mv[t]; }
// trie vertex whose candidates frame F enumerates for virtual sibling vs
__device__ __forceinline__ int vert_of(const W& w, int F, int vs) {
  return F == 0 ? 0 : mvert(w, w.h->pv[F]).child_begin + vs / w.h->nr[F];
}
__device__ __forceinline__ StmSrc lvl_cand(const W& w, int F, int vs) { return mvert(w, vert_of(w, F, vs)).cand; }
__device__ __forceinline__ StmFilter lvl_filt(const W& w, int F, int vs) { return mvert(w, vert_of(w, F, vs)).filt; }
__device__ __forceinline__ int lvl_need(const W& w, int F, int vs) { return mvert(w, vert_of(w, F, vs)).need; }
__device__ __forceinline__ const StmNode& pnode(const W& w, int s) { return w.kp->mn[s].nd; }
__device__ __forceinline__ int pregion(const W& w, int s) { return w.kp->mn[s].region; }
// pool nodes built after v_F is chosen from frame F's virtual sibling vs
__device__ __forceinline__ void bset(const W& w, int F, int vs, int& b, int& e, int& nst) {
  const StmMVert& t = mvert(w, vert_of(w, F, vs));
  b = t.build_begin;
  e = t.build_begin + t.n_build;
  nst = t.n_stages;
}
#else
__device__ __forceinline__ StmSrc lvl_cand(const W& w, int F, int) { return w.P->cand[F]; }
__device__ __forceinline__ StmFilter lvl_filt(const W& w, int F, int) { return w.P->filt[F]; }
__device__ __forceinline__ int lvl_need(const W& w, int F, int) { return w.P->need[F]; }
__device__ __forceinline__ const StmNode& pnode(const W& w, int s) { return w.P->nodes[s]; }
__device__ __forceinline__ int pregion(const W&, int s) { return s; }
__device__ __forceinline__ void bset(const W& w, int F, int, int& b, int& e, int& nst) {
  b = w.P->level_begin[F + 1];
  e = w.P->level_begin[F + 2];
  nst = w.P->n_stages[F + 1];
}
#endif
// real sibling index of frame F's (virtual) sibling index vs
#if STM_MULTI
__device__ __forceinline__ int rsib(const W& w, int F, int vs) { return vs % w.h->nr[F]; }
#else
__device__ __forceinline__ int rsib(const W&, int, int vs) { return vs; }
#endif

// value of v_j in the context "frame F, sibling u, candidate c of level F"
__device__ __forceinline__ int pval(const W& w, int j, int F, int u, int c) {
  if (j == F) return c;
  if (j == F - 1) return SIB(w, F, rsib(w, F, u));
  return SIB(w, j + 1, rsib(w, j + 1, w.h->cur[j + 1]));
}

__device__ __forceinline__ void node_slice(const W& w, int s, int F, int u, int un, const int*& p,
                                           int& len) {
#if STM_MULTI
  const int lvl = pnode(w, s).level;
  const int idx = lvl == F + 1 ? un : (lvl == F ? rsib(w, F, u) : rsib(w, lvl, w.h->cur[lvl]));
  const int r = pregion(w, s);
  p = w.arena + (size_t)r * w.kp->cap + NOFF(w, r, idx);
  len = NSZ(w, r, idx);
#else
  int lvl = w.P->nodes[s].level;
  int idx = lvl == F + 1 ? un : (lvl == F ? u : w.h->cur[lvl]);
  p = w.arena + (size_t)s * w.kp->cap + NOFF(w, s, idx);
  len = NSZ(w, s, idx);
#endif
}

__device__ __forceinline__ void src_slice(const W& w, StmSrc src, int F, int u, int c, int un,
                                          const int*& p, int& len) {
  if (src.kind == STM_SRC_RAW) row(w, pval(w, src.idx & 7, F, u, c), p, len, src.idx >> 3);
  else node_slice(w, src.idx, F, u, un, p, len);
}

__device__ __forceinline__ void bounds(const W& w, unsigned lo_m, unsigned hi_m, int F, int u, int c,
                                       int& lo, int& hi) {
  lo = -1;
  hi = INT_MAX;
  for (unsigned m = lo_m; m; m &= m - 1) lo = max(lo, pval(w, __ffs(m) - 1, F, u, c));
  for (unsigned m = hi_m; m; m &= m - 1) hi = min(hi, pval(w, __ffs(m) - 1, F, u, c));
}

__device__ __forceinline__ bool labok(const W& w, int x, unsigned lab) {
  if (lab == STM_LAB_ANY) return true;
  return (w.bh->lab2slot[w.kp->labels[x]] & lab) != 0;
}

// ----------------------------------------------------------------------------
// Flattened multi-job set operation (Fig. 8).  Lane j < njobs owns job j.
// ----------------------------------------------------------------------------
struct Job {
  const int* A;
  const int* B;  // NULL: filtered scan of A
  int alen, blen;
  int op;
  int lo, hi;
  unsigned lab;
  int* out;      // materialise target (NULL in count mode)
  int u, c;      // context for exclusions / per-root attribution
  int a_node;    // 0: A is a CSR row; l+1: A is an arena set node of level l (rebuilt with its frame)
  int abm, bbm;  // hub bitmap slot of A (if a CSR row) / of B, -1 = none
};

__device__ __forceinline__ void narrow(const int*& p, int& n, int lo, int hi) {
  if (n > 16) {
    if (lo >= 0) { int b = lbound(p, n, lo + 1); p += b; n -= b; }
    if (hi < INT_MAX) n = lbound(p, n, hi);
  }
}

// Narrow the CSR row p[0..n) of vertex v to the open interval (lo, hi) at job
// construction.  The split s = out_start[v] cuts the sorted row at v (p[0..s) < v <
// p[s..n)), so the bound lo = v (the common case v_{l-1} < w of a restriction chain)
// costs nothing and every other bound searches only one side of the split.
__device__ __forceinline__ void narrow_split(int v, int s, const int*& p, int& n, int lo, int hi) {
  if (lo < 0 && hi == INT_MAX) return;
  if (s < 0) { narrow(p, n, lo, hi); return; }
  const bool big = n > 16;
  int b = 0, e = n;
  if (lo >= v) { b = s; if (lo > v && big) b += lbound(p + s, n - s, lo + 1); }
  else if (lo >= 0 && big) b = lbound(p, s, lo + 1);
  if (hi <= v) { e = s; if (hi < v && big) e = lbound(p, s, hi); }
  else if (hi < INT_MAX && big && hi > v + 1) e = s + lbound(p + s, n - s, hi);
  else if (hi == v + 1) e = s;
  e = max(e, b);
  p += b;
  n = e - b;
}

// N(v) from its packed record, narrowed to (lo, hi); hub receives v's bitmap slot
__device__ __forceinline__ void row_narrow(const W& w, int v, const int*& p, int& n, int& hub, int lo, int hi,
                                           int dir = 0) {
  const int4 r = vrec(w, v + (dir ? w.kp->n_dir : 0));
  p = w.kp->col_idx + (unsigned)r.x;
  n = r.y;
  hub = r.w;
  narrow_split(v, w.kp->split ? r.z : -1, p, n, lo, hi);
}

__device__ __forceinline__ int log2c(int n) { return 32 - __clz(n); }  // ceil(log2(n+1))

struct ElemOut {
  unsigned long long jc;
  int outc;
};

// The element loop of a combined set operation (Fig. 8): 32 elements of the flattened
// job stream per pass -- per-lane job lookup, membership probe, ballot compaction into
// the output set (materialise) or a popcount (count).  Out of line so that every
// run_jobs call site shares one copy (measured: i-cache stalls).
__device__ __forceinline__ ElemOut elem_loop_inl(const int lane, const int incl, const int total, const int start,
                                          const unsigned long long Dll, const unsigned long long Pll,
                                          const unsigned long long Oll, const int plen, const int flags,
                                          const int lo, const int hi, const unsigned lab, const bool mine,
                                          const bool count_mode, const uint8_t* const glabels,
                                          const unsigned char* const l2s) {
  int outc = 0;
  unsigned long long jc = 0;
  for (int e0 = 0; e0 < total; e0 += 32) {
    const int e = e0 + lane;
    int j = 0;
#pragma unroll
    for (int step = 16; step > 0; step >>= 1) {
      int v = __shfl_sync(FULLMASK, incl, j + step - 1);
      if (v <= e) j += step;
    }
    const bool valid = e < total;
    const int* Dj = (const int*)__shfl_sync(FULLMASK, Dll, j);
    const int* Pj = (const int*)__shfl_sync(FULLMASK, Pll, j);
    const int sj = __shfl_sync(FULLMASK, start, j);
    const int pl = __shfl_sync(FULLMASK, plen, j);
    const int fj = __shfl_sync(FULLMASK, flags, j);
    const int loj = __shfl_sync(FULLMASK, lo, j);
    const int hij = __shfl_sync(FULLMASK, hi, j);
    const unsigned labj = __shfl_sync(FULLMASK, lab, j);
    bool keep = false;
    int x = 0;
    if (valid) {
      x = Dj[e - sj];
      keep = x > loj && x < hij;
      if (keep && (fj & 1)) {
        bool f;
        if (fj & 8) f = (STM_BM_LOAD((const unsigned*)Pj + (x >> 5)) >> (x & 31)) & 1u;
        else f = member(Pj, pl, x);
        keep = (fj & 4) ? !f : f;
      }
      if (keep && labj != STM_LAB_ANY) keep = (l2s[glabels[x]] & labj) != 0;
    }
    const unsigned km = __ballot_sync(FULLMASK, keep);
    // lanes of my own job inside this chunk
    int a = start - e0, b = incl - e0;
    a = a < 0 ? 0 : a;
    b = b > 32 ? 32 : b;
    unsigned rmask = 0;
    if (mine && a < b) rmask = (b == 32 ? FULLMASK : ((1u << b) - 1)) & ~((1u << a) - 1);
    if (count_mode) {
      jc += __popc(km & rmask);
    } else {
      int* Oj = (int*)__shfl_sync(FULLMASK, Oll, j);
      int base = __shfl_sync(FULLMASK, outc, j);
      int fl = sj - e0;
      fl = fl < 0 ? 0 : fl;
      unsigned before = km & ((1u << lane) - 1) & ~((1u << fl) - 1);
      if (keep) Oj[base + __popc(before)] = x;
      outc += __popc(km & rmask);
    }
  }
  return ElemOut{jc, outc};
}
__device__ __noinline__ ElemOut elem_loop(const int lane, const int incl, const int total, const int start,
                                          const unsigned long long Dll, const unsigned long long Pll,
                                          const unsigned long long Oll, const int plen, const int flags,
                                          const int lo, const int hi, const unsigned lab, const bool mine,
                                          const bool count_mode, const uint8_t* const glabels,
                                          const unsigned char* const l2s) {
  return elem_loop_inl(lane, incl, total, start, Dll, Pll, Oll, plen, flags, lo, hi, lab, mine, count_mode,
                       glabels, l2s);
}

// Returns the (warp-uniform) number of kept elements summed over all jobs when
// counting; in materialise mode *outc (lane j) receives job j's output size.  probe:
// count mode for the candidate-set pre-test (plan.h pretest) -- *outc (lane j) receives
// job j's count, with no exclusion correction, per-root attribution or listing.
__device__ JOBS_INL unsigned long long run_jobs(W& w, Job J, int njobs, bool count_mode, int F,
                                                    unsigned excl, int* outc_lane, bool probe = false) {
  const int lane = w.lane;
  PROF_BEGIN(10)
  const bool mine = lane < njobs;
  // operands narrowed to the open interval (lo, hi) of the restriction bounds
  const int* An = J.A;
  int an = mine ? J.alen : 0;
  const int* Bn = J.B;
  int bn = (mine && J.B) ? J.blen : 0;
  // CSR-row operands were narrowed at job construction (narrow_row); arena sets here
  if (mine && J.a_node) narrow(An, an, J.lo, J.hi);
  // ---- per-job driving side: for an intersection the shorter (bound-narrowed) operand
  // drives and the longer one is probed
  const int* D = An;
  const int* Pp = Bn;
  int dlen = an, plen = bn;
  int pslot = -1;  // bitmap slot of the probed operand
  if (mine) {
    pslot = J.bbm;
    if (J.op == STM_OP_AND && bn < an) {
      D = Bn; dlen = bn; Pp = An; plen = an; pslot = J.abm;
    }
    if (!J.B) { Pp = nullptr; plen = 0; pslot = -1; }
    // a probed hub row is tested in its bitmap: one word per element instead of
    // ceil(log2 |P|) dependent loads (the driving element already lies in (lo, hi))
    if (pslot >= 0) Pp = (const int*)(w.kp->bitmaps + (size_t)pslot * (size_t)w.kp->bm_words);
  }
  // A counted set with no probe operand and no label filter is a bounded view: its
  // count is the narrowed length (narrowing is exact once that exceeds 16), no element
  // is visited -- the last level of K6-e / stars / paths is O(log) per job instead of
  // O(|A|) (the exclusion correction below still applies).
  unsigned long long jc0 = 0;
  if (!STM_LIST && count_mode && !probe && mine && !J.B && J.lab == STM_LAB_ANY && an > 16) {
    jc0 = (unsigned long long)an;
    dlen = 0;
  }
  if (STM_INSTR && w.kp->count_bytes && mine) {
    // W_op = 4|A| + 4 min(|B|, |A| ceil(log2(|B|+1))) (+ 4|out| below),
    // with A the driving operand and B the probed one (before hashing); a counted
    // bounded view moves only its two bound searches
    int d, pl;
    if (J.op == STM_OP_AND) { d = min(an, bn); pl = max(an, bn); } else { d = an; pl = bn; }
    if (jc0) w.wbytes += 8ull * (unsigned long long)log2c(J.alen);
    else w.wbytes += 4ull * (unsigned long long)d + 4ull * (unsigned long long)min((long long)pl, (long long)d * log2c(pl));
    w.wmerge += 4ull * (unsigned long long)(an + bn);
    w.wjobs += 1;
  }
  PROF_END(10, njobs)
  PROF_BEGIN(11)
  int incl = dlen;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int t = __shfl_up_sync(FULLMASK, incl, o);
    if (lane >= o) incl += t;
  }
  const int total = __shfl_sync(FULLMASK, incl, 31);
  const int start = incl - dlen;
#if STM_PROFILE
  w.last_total = total;
#endif
  const int flags = (Pp != nullptr ? 1 : 0) | (J.op == STM_OP_DIFF ? 4 : 0) | (pslot >= 0 ? 8 : 0);
  const uint8_t* const glabels = w.kp->labels;
  const unsigned char* const l2s = w.bh->lab2slot;
#if STM_ELEM_NOINLINE && !STM_LIST
  // one out-of-line copy of the element loop for every call site (i-cache: the plan-
  // specialised kernels instantiate run_jobs once per frame and kind); short streams stay
  // inline (the call costs more than it saves there)
  unsigned long long jc = jc0;
  int outc = 0;
  if (total > STM_ELEM_INLINE_MAX) {
    const ElemOut eo = elem_loop(lane, incl, total, start, (unsigned long long)D, (unsigned long long)Pp,
                                 (unsigned long long)J.out, plen, flags, J.lo, J.hi, J.lab, mine, count_mode,
                                 glabels, l2s);
    jc += eo.jc;
    outc = eo.outc;
  } else {
    const ElemOut eo = elem_loop_inl(lane, incl, total, start, (unsigned long long)D, (unsigned long long)Pp,
                                     (unsigned long long)J.out, plen, flags, J.lo, J.hi, J.lab, mine, count_mode,
                                     glabels, l2s);
    jc += eo.jc;
    outc = eo.outc;
  }
#else
  int outc = 0;
  unsigned long long jc = jc0;
  const unsigned long long Dll = (unsigned long long)D, Pll = (unsigned long long)Pp,
                           Oll = (unsigned long long)J.out;
  for (int e0 = 0; e0 < total; e0 += 32) {
    const int e = e0 + lane;
    int j = 0;
#pragma unroll
    for (int step = 16; step > 0; step >>= 1) {
      int v = __shfl_sync(FULLMASK, incl, j + step - 1);
      if (v <= e) j += step;
    }
    const bool valid = e < total;
    const int* Dj = (const int*)__shfl_sync(FULLMASK, Dll, j);
    const int* Pj = (const int*)__shfl_sync(FULLMASK, Pll, j);
    const int sj = __shfl_sync(FULLMASK, start, j);
    const int pl = __shfl_sync(FULLMASK, plen, j);
    const int fj = __shfl_sync(FULLMASK, flags, j);
    const int loj = __shfl_sync(FULLMASK, J.lo, j);
    const int hij = __shfl_sync(FULLMASK, J.hi, j);
    const unsigned labj = __shfl_sync(FULLMASK, J.lab, j);
    bool keep = false;
    int x = 0;
    if (valid) {
      x = Dj[e - sj];
      keep = x > loj && x < hij;
      if (keep && (fj & 1)) {
        bool f;
        if (fj & 8) f = (STM_BM_LOAD((const unsigned*)Pj + (x >> 5)) >> (x & 31)) & 1u;
        else f = member(Pj, pl, x);
        keep = (fj & 4) ? !f : f;
      }
      if (keep && labj != STM_LAB_ANY) keep = (l2s[glabels[x]] & labj) != 0;
    }
#if STM_LIST
    // listing build: injectivity exclusions are applied per element (instead of the
    // count correction below), then every kept element is one embedding
    int uj = 0, cj = 0;
    if (count_mode && !probe) {
      uj = __shfl_sync(FULLMASK, J.u, j);
      cj = __shfl_sync(FULLMASK, J.c, j);
      if (keep && excl)
        for (int t = 0; t < STM_KMAX; ++t)
          if ((excl >> t & 1u) && x == pval(w, t, F, uj, cj)) keep = false;
    }
#endif
    const unsigned km = __ballot_sync(FULLMASK, keep);
    // lanes of my own job inside this chunk
    int a = start - e0, b = incl - e0;
    a = a < 0 ? 0 : a;
    b = b > 32 ? 32 : b;
    unsigned rmask = 0;
    if (mine && a < b) rmask = (b == 32 ? FULLMASK : ((1u << b) - 1)) & ~((1u << a) - 1);
    if (count_mode) {
      jc += __popc(km & rmask);
#if STM_LIST
      if (km && !probe) {
        // PAPER.md:75 Output(C, iter): row = f(0..k-1) in pattern-vertex order, caller's ids
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(&w.kp->work->list_n, (unsigned long long)__popc(km));
        base = __shfl_sync(FULLMASK, base, 0);
        const unsigned long long idx = base + __popc(km & ((1u << lane) - 1));
        if (keep && idx < w.kp->list_cap) {
          const StmPlan& PL = *w.P;
          int32_t* row = w.kp->list_out + idx * (unsigned long long)PL.k;
          const int32_t* rmap = w.kp->root_map;
          for (int t = 0; t < PL.k - 1; ++t) {
            const int v = pval(w, t, F, uj, cj);
            row[PL.order[t]] = rmap ? rmap[v] : v;
          }
          row[PL.order[PL.k - 1]] = rmap ? rmap[x] : x;
        }
      }
#endif
    } else {
      int* Oj = (int*)__shfl_sync(FULLMASK, Oll, j);
      int base = __shfl_sync(FULLMASK, outc, j);
      int fl = sj - e0;
      fl = fl < 0 ? 0 : fl;
      unsigned before = km & ((1u << lane) - 1) & ~((1u << fl) - 1);
      if (keep) Oj[base + __popc(before)] = x;
      outc += __popc(km & rmask);
    }
  }
#endif
  PROF_END(11, total)
  if (probe) {
    *outc_lane = (int)jc;
    return 0;
  }
  if (!count_mode) {
    if (STM_INSTR && w.kp->count_bytes && mine) w.wbytes += 4ull * (unsigned long long)outc;
    *outc_lane = outc;
    return 0;
  }
  // exclusions: earlier matched vertices of non-adjacent pattern vertices may
  // still be in the counted set; remove them explicitly.
  if (!STM_LIST && mine && excl) {
    for (int t = 0; t < STM_KMAX; ++t) {
      if (!(excl & (1u << t))) continue;
      int x = pval(w, t, F, J.u, J.c);
      if (!(x > J.lo && x < J.hi)) continue;
      if (!labok(w, x, J.lab)) continue;
      if (!member(J.A, J.alen, x)) continue;
      if (J.B) {
        bool f = member(J.B, J.blen, x);
        if ((J.op == STM_OP_DIFF) ? f : !f) continue;
      }
      jc -= 1;
    }
  }
  if (w.kp->per_root && mine && jc) {
    const int r = pval(w, 0, F, J.u, J.c);
    atomicAdd(&w.kp->per_root[w.kp->root_map ? w.kp->root_map[r] : r], jc);
  }
  unsigned long long s = jc;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(FULLMASK, s, o);
  return s;
}

#if STM_MULTI
// count job for the final level in context (F, u, c, un); lv = the leaf trie vertex
// (STM_MULTI; ignored by single-pattern builds)
__device__ __forceinline__ Job count_job(const W& w, int F, int u, int c, int un, int lv = 0) {
#if STM_MULTI
  const StmMVert& L = mvert(w, lv);
  const StmSrc ca = L.cand;
  const int cb = L.cnt_b, cop = L.cnt_op;
  const StmFilter f = L.filt;
#else
  (void)lv;
  const StmPlan& P = *w.P;
  const StmSrc ca = P.cnt_a;
  const int cb = P.cnt_b, cop = P.cnt_op;
  const StmFilter f = P.filt[P.k - 1];
#endif
  Job J;
  if (ca.kind != STM_SRC_RAW) node_slice(w, ca.idx, F, u, un, J.A, J.alen);
  J.B = nullptr;
  J.blen = 0;
  J.op = cop;
  bounds(w, f.lo, f.hi, F, u, c, J.lo, J.hi);
  J.abm = -1;
  if (ca.kind == STM_SRC_RAW) row_narrow(w, pval(w, ca.idx & 7, F, u, c), J.A, J.alen, J.abm, J.lo, J.hi, ca.idx >> 3);
  J.bbm = -1;
  if (cop != STM_OP_NONE) row_narrow(w, pval(w, cb & 7, F, u, c), J.B, J.blen, J.bbm, J.lo, J.hi, cb >> 3);
  J.lab = f.lab;
  J.out = nullptr;
  J.u = u;
  J.c = c;
  J.a_node = ca.kind == STM_SRC_NODE ? 1 : 0;
  return J;
}
#else
// count job for the final level in context (F, u, c, un)
__device__ __forceinline__ Job count_job(const W& w, int F, int u, int c, int un, int = 0) {
  const StmPlan& P = *w.P;
  Job J;
  if (P.cnt_a.kind != STM_SRC_RAW) node_slice(w, P.cnt_a.idx, F, u, un, J.A, J.alen);
  J.B = nullptr;
  J.blen = 0;
  J.op = P.cnt_op;
  const StmFilter f = P.filt[P.k - 1];
  bounds(w, f.lo, f.hi, F, u, c, J.lo, J.hi);
  J.abm = -1;
  if (P.cnt_a.kind == STM_SRC_RAW)
    row_narrow(w, pval(w, P.cnt_a.idx & 7, F, u, c), J.A, J.alen, J.abm, J.lo, J.hi, P.cnt_a.idx >> 3);
  J.bbm = -1;
  if (P.cnt_op != STM_OP_NONE)
    row_narrow(w, pval(w, P.cnt_b & 7, F, u, c), J.B, J.blen, J.bbm, J.lo, J.hi, P.cnt_b >> 3);
  J.lab = f.lab;
  J.out = nullptr;
  J.u = u;
  J.c = c;
  J.a_node = P.cnt_a.kind == STM_SRC_NODE ? 1 : 0;
  return J;
}
#endif

// ----------------------------------------------------------------------------
// small helpers
// ----------------------------------------------------------------------------
// warps of this block waiting for a donation (uniform across the warp)
__device__ __forceinline__ int waiting_warps(const W& w) {
  int m = 0;
  if (w.lane == 0) m = *(volatile int*)&w.bh->idle_mask;
  return __shfl_sync(FULLMASK, m, 0);
}
// Grid status, looked at (two L2 loads) at most every ~2 us per warp: does the pool want
// a task (block pollers waiting)?  Is the grid starving (WarpHdr::deep, split_stop)?
__device__ __forceinline__ bool pool_wanted(const W& w) {
  int want = 0;
  if (w.lane == 0) {
    const long long now = clock64();
    if (now - w.h->gchk >= STM_GCHK_CYCLES) {
      w.h->gchk = now;
      volatile StmWork* vw = w.kp->work;
      want = vw->deficit > 0;
      w.h->deep = STM_DEEP_FRAC * (w.kp->total_warps - vw->active) > w.kp->total_warps;
    }
  }
  return __shfl_sync(FULLMASK, want, 0) != 0;
}

// candidate-list length of frame F's sibling u
__device__ __forceinline__ int src_len(const W& w, int F, int u) {
  const int* p;
  int len;
  src_slice(w, lvl_cand(w, F, u), F, u, 0, 0, p, len);
  return len;
}

// Make sibling u current in frame F.  Its candidate list is sorted, so the level's
// restriction bounds (lo, hi) select a contiguous position range: find it by
// binary search instead of filtering every element (with degree-ranked ids a
// hub's row is long but only its short suffix above v0 is a candidate).
// Positions stay positions of the full list, so stolen ranges mean the same.
__device__ __forceinline__ void set_sibling(W& w, int F, int u) {
  const int* p;
  int len;
  src_slice(w, lvl_cand(w, F, u), F, u, 0, 0, p, len);
  const StmFilter f = lvl_filt(w, F, u);
  int b = 0, e = len;
  if ((f.lo | f.hi) && len > 0) {
    int lo, hi;
    bounds(w, f.lo, f.hi, F, u, 0, lo, hi);
    if (lo >= 0) b = lbound(p, len, lo + 1);
    if (hi < INT_MAX) e = max(b, lbound(p, len, hi));
  }
  if (e - b < lvl_need(w, F, u)) e = b;  // fewer candidates than any extension needs (plan.h need)
  if (F == 1 && w.kp->entries) {  // a root entry enumerates one piece of its candidate list
    // (after the need test: the other pattern vertices may come from the whole list)
    const int c = __ldg(&w.kp->entries[w.h->rent[rsib(w, 1, u)]].y);
    b = max(b, c * w.kp->root_split);
    e = max(b, min(e, (c + 1) * w.kp->root_split));
  }
  HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
  if (w.lane == 0) {
    w.h->cur[F] = u;
    w.h->it[F] = b;
    w.h->end[F] = e;
  }
  __syncwarp();
}

// does candidate c (of level F, sibling u) pass the level's filter?
__device__ __forceinline__ bool cand_ok(const W& w, int F, int u, int c, int lo, int hi) {
  const StmFilter f = lvl_filt(w, F, u);
  if (!(c > lo && c < hi)) return false;
  if (!labok(w, c, f.lab)) return false;
  if (f.excl) {
    for (int t = 0; t < F; ++t)
      if ((f.excl & (1u << t)) && pval(w, t, F, u, c) == c) return false;
  }
  return true;
}

// upper bound on the size of node s (level F+1) for candidate c
__device__ int node_ub(const W& w, int s, int F, int u, int c) {
  int m = INT_MAX;
  for (;;) {
    const StmNode nd = pnode(w, s);
    if (nd.op == STM_OP_AND) m = min(m, degree(w, pval(w, nd.b & 7, F, u, c), nd.b >> 3));
    if (nd.a_kind == STM_SRC_RAW) return min(m, degree(w, pval(w, nd.a & 7, F, u, c), nd.a >> 3));
    if (pnode(w, nd.a).level == F + 1) { s = nd.a; continue; }
    const int* p;
    int len;
    node_slice(w, nd.a, F, u, 0, p, len);
    return min(m, len);
  }
}

// The part of node_ub that does not depend on the candidate (position F) of frame
// F, sibling u: INT_MAX when every term does.
__device__ int node_ub_const(const W& w, int s, int F, int u) {
  int m = INT_MAX;
  for (;;) {
    const StmNode nd = pnode(w, s);
    if (nd.op == STM_OP_AND && (nd.b & 7) != F) m = min(m, degree(w, pval(w, nd.b & 7, F, u, 0), nd.b >> 3));
    if (nd.a_kind == STM_SRC_RAW)
      return (nd.a & 7) != F ? min(m, degree(w, pval(w, nd.a & 7, F, u, 0), nd.a >> 3)) : m;
    if (pnode(w, nd.a).level == F + 1) { s = nd.a; continue; }
    const int* p;
    int len;
    node_slice(w, nd.a, F, u, 0, p, len);
    return min(m, len);
  }
}

// Drop the siblings of frame F+1 whose lane flag `keep` is false (lane t = sibling t < m):
// the kept siblings move down in order with their slice offsets (and sizes, once built).
__device__ __forceinline__ int compact_siblings(W& w, int F, int m, bool keep) {
  const int lane = w.lane;
  const unsigned km = __ballot_sync(FULLMASK, keep && lane < m);
  const int nm = __popc(km);
  if (nm == m) return m;
  const int dst = __popc(km & ((1u << lane) - 1));
  const bool mv = (km >> lane) & 1u;
  const int c = lane < m ? SIB(w, F + 1, lane) : 0;
  __syncwarp();
  if (mv) SIB(w, F + 1, dst) = c;
  int nb, ne, nst;
  bset(w, F, w.h->cur[F], nb, ne, nst);
  for (int s = nb; s < ne; ++s) {
    const int r = pregion(w, s);
    const int o = lane < m ? NOFF(w, r, lane) : 0, z = lane < m ? NSZ(w, r, lane) : 0;
    __syncwarp();
    if (mv) { NOFF(w, r, dst) = o; NSZ(w, r, dst) = z; }
  }
  __syncwarp();
  return nm;
}

// Compute the nodes of level F+1 for the m siblings SIB(F+1, 0..m-1); offsets
// NOFF were assigned by the caller; sizes NSZ are written here.  With `prune`
// (plan.h need / pretest), siblings whose level-(F+1) candidate set cannot supply
// need[F+1] candidates are dropped first (pre-test on bound-narrowed operands) or
// after the build; returns the number of siblings kept.
#if STM_MULTI
__device__ STEP_INL int build_nodes(W& w, int F, int m, bool prune) {
  const int L1 = F + 1;
  const int u = F >= 1 ? w.h->cur[F] : 0;
  int nb, ne, nstages;
  bset(w, F, u, nb, ne, nstages);
  if (nb == ne) return m;
#if STM_MULTI
  prune = false;  // need / pretest are per pattern; the merged build serves every child
  const StmFilter cf = {STM_LAB_ANY, 0, 0, 0};
  const bool pre = false;
  const int need1 = 1;
  const StmSrc ccand = {STM_SRC_RAW, 0, 0};
#else
  const StmPlan& P = *w.P;
  const bool pre = prune && P.pretest[L1];
  const StmFilter cf = P.filt[L1];  // the candidate consumer's filter
  const int need1 = P.need[L1];
  const StmSrc ccand = P.cand[L1];
#endif
  // phase -1: candidate pre-test (probe counts); phases 0..: the level's stages.  The
  // nodes of one stage are contiguous ([sb, se): ordered by stage).
  int se = nb;
  for (int st = pre ? -1 : 0; st < nstages; ++st) {
    int sb = se;
    if (st < 0) {
      sb = ccand.idx;
      se = sb + 1;
    } else {
      sb = st == 0 ? nb : se;
      se = sb;
      while (se < ne && pnode(w, se).stage == st) ++se;
    }
    const int njobs_total = (se - sb) * m;
    for (int j0 = 0; j0 < njobs_total; j0 += 32) {
      const int jj = j0 + w.lane;
      const int nj = min(32, njobs_total - j0);
      Job J;
      J.A = nullptr; J.B = nullptr; J.alen = 0; J.blen = 0; J.op = STM_OP_AND;
      J.lo = -1; J.hi = INT_MAX; J.lab = STM_LAB_ANY; J.out = nullptr; J.u = u; J.c = 0; J.a_node = 0; J.abm = -1; J.bbm = -1;
      int r = 0, t = 0;
      if (w.lane < nj) {
        const int s = sb + jj / m;
        t = jj % m;
        r = pregion(w, s);
        const StmNode nd = pnode(w, s);
        const int c = SIB(w, L1, t);
        J.c = c;
        if (st < 0) bounds(w, cf.lo, cf.hi, F, u, c, J.lo, J.hi);  // the consumer's bounds
        else bounds(w, nd.lo, nd.hi, F, u, c, J.lo, J.hi);
        if (nd.a_kind == STM_SRC_RAW)
          row_narrow(w, pval(w, nd.a & 7, F, u, c), J.A, J.alen, J.abm, J.lo, J.hi, nd.a >> 3);
        else node_slice(w, nd.a, F, u, t, J.A, J.alen);
        J.a_node = nd.a_kind == STM_SRC_NODE ? 1 : 0;
        row_narrow(w, pval(w, nd.b & 7, F, u, c), J.B, J.blen, J.bbm, J.lo, J.hi, nd.b >> 3);
        J.op = nd.op;
        J.lab = st < 0 ? cf.lab : nd.lab;
        J.out = st < 0 ? nullptr : w.arena + (size_t)r * w.kp->cap + NOFF(w, r, t);
      }
      int outc = 0;
      PROF_LVL_BEGIN()
      run_jobs(w, J, nj, st < 0, F, 0, &outc, st < 0);
      PROF_LVL_END(st < 0 ? 0 : 1, L1)
      if (st < 0) {  // pre-test: one job per sibling (one node, m <= 32)
        m = compact_siblings(w, F, m, outc >= need1);
        if (m == 0) return 0;
      } else {
        if (w.lane < nj) NSZ(w, r, t) = outc;
        __syncwarp();
      }
    }
    if (st < 0) se = nb;  // the stages start at nb
  }
  // post-build check: a candidate node of this level smaller (within the consumer's
  // bounds) than need[F+1] cannot be extended
  if (prune && !pre && need1 > 1 && ccand.kind == STM_SRC_NODE && pnode(w, ccand.idx).level == L1) {
    bool keep = true;
    if (w.lane < m) {
      const int c = SIB(w, L1, w.lane);
      const int* p;
      int len;
      node_slice(w, ccand.idx, F, u, w.lane, p, len);
      if (len >= need1 && (cf.lo | cf.hi)) {
        int lo, hi;
        bounds(w, cf.lo, cf.hi, F, u, c, lo, hi);
        int b = 0, e = len;
        if (lo >= 0) b = lbound(p, len, lo + 1);
        if (hi < INT_MAX) e = max(b, lbound(p, len, hi));
        len = e - b;
      }
      keep = len >= need1;
    }
    m = compact_siblings(w, F, m, keep);
  }
  return m;
}
#else
__device__ STEP_INL int build_nodes(W& w, int F, int m, bool prune) {  // single-pattern plans
  const StmPlan& P = *w.P;
  const int L1 = F + 1;
  const int nb = P.level_begin[L1], ne = P.level_begin[L1 + 1];
  if (nb == ne) return m;
  const int u = F >= 1 ? w.h->cur[F] : 0;
  // (reads above are ordered before this write by a full-warp collective)
  const bool pre = prune && P.pretest[L1];
  const StmFilter cf = P.filt[L1];  // the candidate consumer's filter
  // phase -1: candidate pre-test (probe counts); phases 0..: the level's stages
  for (int st = pre ? -1 : 0; st < P.n_stages[L1]; ++st) {
    // jobs of this phase: (node, sibling) pairs
    int nodes_in[STM_MAX_NODES];
    int nn = 0;
    if (st < 0) nodes_in[nn++] = P.cand[L1].idx;
    else
      for (int s = nb; s < ne; ++s)
        if (P.nodes[s].stage == st) nodes_in[nn++] = s;
    const int njobs_total = nn * m;
    for (int j0 = 0; j0 < njobs_total; j0 += 32) {
      const int jj = j0 + w.lane;
      const int nj = min(32, njobs_total - j0);
      Job J;
      J.A = nullptr; J.B = nullptr; J.alen = 0; J.blen = 0; J.op = STM_OP_AND;
      J.lo = -1; J.hi = INT_MAX; J.lab = STM_LAB_ANY; J.out = nullptr; J.u = u; J.c = 0; J.a_node = 0; J.abm = -1; J.bbm = -1;
      int s = 0, t = 0;
      if (w.lane < nj) {
        s = nodes_in[jj / m];
        t = jj % m;
        const StmNode nd = P.nodes[s];
        const int c = SIB(w, L1, t);
        J.c = c;
        if (st < 0) bounds(w, cf.lo, cf.hi, F, u, c, J.lo, J.hi);  // the consumer's bounds
        else bounds(w, nd.lo, nd.hi, F, u, c, J.lo, J.hi);
        if (nd.a_kind == STM_SRC_RAW)
          row_narrow(w, pval(w, nd.a & 7, F, u, c), J.A, J.alen, J.abm, J.lo, J.hi, nd.a >> 3);
        else node_slice(w, nd.a, F, u, t, J.A, J.alen);
        J.a_node = nd.a_kind == STM_SRC_NODE ? P.nodes[nd.a].level + 1 : 0;
        row_narrow(w, pval(w, nd.b & 7, F, u, c), J.B, J.blen, J.bbm, J.lo, J.hi, nd.b >> 3);
        J.op = nd.op;
        J.lab = st < 0 ? cf.lab : nd.lab;
        J.out = st < 0 ? nullptr : w.arena + (size_t)s * w.kp->cap + NOFF(w, s, t);
      }
      int outc = 0;
      PROF_LVL_BEGIN()
      run_jobs(w, J, nj, st < 0, F, 0, &outc, st < 0);
      PROF_LVL_END(st < 0 ? 0 : 1, L1)
      if (st < 0) {  // pre-test: one job per sibling (nn == 1, m <= 32)
        m = compact_siblings(w, F, m, outc >= P.need[L1]);
        if (m == 0) return 0;
      } else {
        if (w.lane < nj) NSZ(w, s, t) = outc;
        __syncwarp();
      }
    }
  }
  // post-build check: a candidate node of this level smaller (within the consumer's
  // bounds) than need[F+1] cannot be extended
  if (prune && !pre && P.need[L1] > 1 && P.cand[L1].kind == STM_SRC_NODE &&
      P.nodes[P.cand[L1].idx].level == L1) {
    bool keep = true;
    if (w.lane < m) {
      const int c = SIB(w, L1, w.lane);
      const int* p;
      int len;
      node_slice(w, P.cand[L1].idx, F, u, w.lane, p, len);
      if (len >= P.need[L1] && (cf.lo | cf.hi)) {
        int lo, hi;
        bounds(w, cf.lo, cf.hi, F, u, c, lo, hi);
        int b = 0, e = len;
        if (lo >= 0) b = lbound(p, len, lo + 1);
        if (hi < INT_MAX) e = max(b, lbound(p, len, hi));
        len = e - b;
      }
      keep = len >= P.need[L1];
    }
    m = compact_siblings(w, F, m, keep);
  }
  return m;
}
#endif

// ----------------------------------------------------------------------------
// gather: next batch of candidates of frame F (current sibling) as the
// siblings of frame F+1, admitted so that every node region fits.
// Caller holds the frame lock if the frame is stealable.  Returns batch size.
// ----------------------------------------------------------------------------
// Admission with per-candidate size bounds: used when U copies of a
// node's candidate-independent bound may not fit; kept out of line (cold for most plans).
__device__ GATHER_SLOW_INL int gather_batch_slow(W& w, int F, int U, const int* src, int lo, int hi, int pos,
                                                 const int e, const int nb, const int ne, const int cap,
                                                 const int u) {
  HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
  if (w.lane == 0)
    for (int s = nb; s < ne; ++s) w.h->used[s - nb] = 0;
  __syncwarp();
  int m = 0;
  bool cut = false;
  while (m < U && pos < e && !cut) {
    const int p = pos + w.lane;
    const bool valid = p < e;
    int c = valid ? src[p] : 0;
    bool pass = valid && cand_ok(w, F, u, c, lo, hi);
    // admission: cumulative upper bounds per node must fit in `cap`
    bool fits = true;
    for (int s = nb; s < ne; ++s) {
      int ub = pass ? node_ub(w, s, F, u, c) : 0;
      int inc = ub;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        int t = __shfl_up_sync(FULLMASK, inc, o);
        if (w.lane >= o) inc += t;
      }
      // (the first candidate of a batch is always admitted: its bound fits the region, and the
      // batch budget STM_BATCH_ELEMS only limits how many more join it)
      if (pass && w.h->used[s - nb] + inc > cap && !(m == 0 && inc == ub)) fits = false;
    }
    unsigned pm = __ballot_sync(FULLMASK, pass);
    unsigned fm = __ballot_sync(FULLMASK, pass && fits);
    // accept a prefix of passing lanes: those before the first non-fitting one, at most U-m
    unsigned bad = pm & ~fm;
    unsigned lim = bad ? ((1u << (__ffs(bad) - 1)) - 1) : FULLMASK;
    unsigned acc = pm & lim;
    int room = U - m;
    if (__popc(acc) > room) {
      // keep the first `room` set bits
      unsigned a2 = 0, t = acc;
      for (int i = 0; i < room; ++i) { unsigned lsb = t & (0u - t); a2 |= lsb; t ^= lsb; }
      acc = a2;
      cut = true;
    }
    if (bad) cut = true;
    const bool me = (acc >> w.lane) & 1u;
    const int rank = __popc(acc & ((1u << w.lane) - 1));
    // second pass: offsets for accepted lanes
    for (int s = nb; s < ne; ++s) {
      int ub = me ? node_ub(w, s, F, u, c) : 0;
      int inc = ub;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        int t = __shfl_up_sync(FULLMASK, inc, o);
        if (w.lane >= o) inc += t;
      }
      int used = w.h->used[s - nb];
      if (me) NOFF(w, pregion(w, s), m + rank) = used + inc - ub;
      int tot = __shfl_sync(FULLMASK, inc, 31);
      __syncwarp();
      if (w.lane == 0) w.h->used[s - nb] = used + tot;
      __syncwarp();
    }
    if (me) SIB(w, F + 1, m + rank) = c;
    m += __popc(acc);
    if (cut) {
      // resume right after the last accepted candidate
      unsigned hiacc = acc ? (31 - __clz(acc)) : 0;
      pos = acc ? pos + (int)hiacc + 1 : pos;
    } else {
      pos = min(pos + 32, e);
    }
    __syncwarp();
  }
  HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
  if (w.lane == 0) w.h->it[F] = pos;
  __syncwarp();
  return m;
}

__device__ STEP_INL int gather_batch(W& w, int F, int U) {
  const int u = w.h->cur[F];
  const int* src;
  int len;
  src_slice(w, lvl_cand(w, F, u), F, u, 0, 0, src, len);
  int lo, hi;
  const StmFilter f = lvl_filt(w, F, u);
  bounds(w, f.lo, f.hi, F, u, 0, lo, hi);
  int pos = w.h->it[F];
  const int e = w.h->end[F];
  int nb, ne, nst;
  bset(w, F, u, nb, ne, nst);
  const int cap = w.kp->cap;
  // Fast admission: when U copies of every node's candidate-independent size bound
  // fit in its region, any batch of <= U candidates fits -- fixed slice offsets
  // t * bound, no per-candidate degree loads or prefix sums.
  // batch budget: the sets of one batch are built by one combined operation that is never
  // split by work sharing, so it is kept to about STM_BATCH_ELEMS driving elements (not the
  // whole arena region) -- heavy hub siblings then stay in the frame, stealable
  const int capb = STM_BATCH_ELEMS > 0 ? min(cap, STM_BATCH_ELEMS) : cap;
  bool fixed = true;
  for (int s = nb; s < ne && fixed; ++s) fixed = (long long)node_ub_const(w, s, F, u) * U <= (long long)capb;
  if (fixed) {
    int m = 0;
    while (m < U && pos < e) {
      const int p = pos + w.lane;
      const bool valid = p < e;
      const int c = valid ? src[p] : 0;
      const bool pass = valid && cand_ok(w, F, u, c, lo, hi);
      unsigned acc = __ballot_sync(FULLMASK, pass);
      const int room = U - m;
      bool cut = false;
      if (__popc(acc) > room) {
        unsigned a2 = 0, t = acc;  // keep the first `room` set bits
        for (int i = 0; i < room; ++i) { const unsigned lsb = t & (0u - t); a2 |= lsb; t ^= lsb; }
        acc = a2;
        cut = true;
      }
      if ((acc >> w.lane) & 1u) SIB(w, F + 1, m + __popc(acc & ((1u << w.lane) - 1))) = c;
      m += __popc(acc);
      pos = cut ? pos + (31 - __clz(acc)) + 1 : min(pos + 32, e);
    }
    for (int s = nb; s < ne; ++s) {
      const int ub0 = node_ub_const(w, s, F, u);
      if (w.lane < m) NOFF(w, pregion(w, s), w.lane) = w.lane * ub0;
    }
    HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
    if (w.lane == 0) w.h->it[F] = pos;
    __syncwarp();
    return m;
  }
  return gather_batch_slow(w, F, U, src, lo, hi, pos, e, nb, ne, capb, u);
}

// root batch: up to root_batch roots from [root_it, root_end) with the root label
__device__ int gather_roots(W& w) {
  const unsigned rlab = lvl_filt(w, 0, 0).lab;
  const int R = w.kp->root_batch;
  const int2* ent = w.kp->entries;
  int pos = w.h->root_it;
  const int e = w.h->root_end;
  int m = 0;
  while (m < R && pos < e) {
    const int p = pos + w.lane;
    const int v = (p < e && ent) ? __ldg(&ent[p].x) : p;
    const bool pass = p < e && labok(w, v, rlab);
    unsigned pm = __ballot_sync(FULLMASK, pass);
    int room = R - m;
    unsigned acc = pm;
    bool cut = false;
    if (__popc(acc) > room) {
      unsigned a2 = 0, t = acc;
      for (int i = 0; i < room; ++i) { unsigned lsb = t & (0u - t); a2 |= lsb; t ^= lsb; }
      acc = a2;
      cut = true;
    }
    if ((acc >> w.lane) & 1u) {
      const int slot = m + __popc(acc & ((1u << w.lane) - 1));
      SIB(w, 1, slot) = v;
      w.h->rent[slot] = p;
    }
    m += __popc(acc);
    pos = cut ? pos + (31 - __clz(acc)) + 1 : min(pos + 32, e);
  }
  HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
  if (w.lane == 0) w.h->root_it = pos;
  __syncwarp();
  return m;
}

// ----------------------------------------------------------------------------
// counting
// ----------------------------------------------------------------------------
// frame-count mode: frame k-1 is built; one job per sibling
__device__ void frame_count(W& w, int m) {
  const int k = w.P->k;
  const int F = k - 2;
  const int u = F >= 1 ? w.h->cur[F] : 0;
  Job J;
  J.A = nullptr; J.B = nullptr; J.alen = 0; J.blen = 0; J.op = STM_OP_NONE;
  J.lo = -1; J.hi = INT_MAX; J.lab = STM_LAB_ANY; J.out = nullptr; J.u = u; J.c = 0; J.a_node = 0; J.abm = -1; J.bbm = -1;
#if STM_MULTI
  // every leaf (pattern) below the current trie vertex counts its final operation
  const StmMVert& sv = mvert(w, vert_of(w, F, u));
  for (int lv = sv.child_begin; lv < sv.child_begin + sv.n_children; ++lv) {
    if (w.lane < m) J = count_job(w, F, u, SIB(w, k - 1, w.lane), w.lane, lv);
    const unsigned long long c = run_jobs(w, J, m, true, F, mvert(w, lv).filt.excl, nullptr);
    w.cnt += c;
    if (w.lane == 0 && c) atomicAdd(&w.kp->mcount[mvert(w, lv).motif], c);
  }
#else
  if (w.lane < m) J = count_job(w, F, u, SIB(w, k - 1, w.lane), w.lane);
  PROF_LVL_BEGIN()
  w.cnt += run_jobs(w, J, m, true, F, w.P->filt[k - 1].excl, nullptr);
  PROF_LVL_END(2, k - 1)
#endif
}

// fused mode at frame F = k-2: count over all remaining (sibling, candidate)
// pairs, 32 jobs per pass.  Returns when the frame is exhausted.
#if !STM_MULTI
__device__ STEP_INL void fused_count(W& w, int F) {
  const StmPlan& P = *w.P;
  for (unsigned pass = 1;; ++pass) {
    if ((pass & 63) == 0 && watchdog(*w.kp, w.h->wd0, "fused")) return;  // (the main loop aborts next)
    // share with waiting warps of the block between counting passes (the stack is
    // consistent here: the staged pairs were already taken out of [it, end))
    PROF_CHK()
    if (w.kp->local_steal && waiting_warps(w)) share_local(*w.kp);
    if (pool_wanted(w) && w.kp->global_steal && F < w.kp->detect_level) maybe_push(*w.kp);
    int nj = 0;
    // gather up to 32 passing candidates across siblings
    for (;;) {
      int u = w.h->cur[F];
      if (u >= w.h->nsib[F]) break;
      int pos = w.h->it[F], e = w.h->end[F];
      if (pos >= e) {
        if (u + 1 >= w.h->nsib[F]) {
          HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
          if (w.lane == 0) w.h->cur[F] = u + 1;
          __syncwarp();
          break;
        }
        set_sibling(w, F, u + 1);
        continue;
      }
      const int* src;
      int len;
      src_slice(w, P.cand[F], F, u, 0, 0, src, len);
      int lo, hi;
      bounds(w, P.filt[F].lo, P.filt[F].hi, F, u, 0, lo, hi);
      const int p = pos + w.lane;
      const bool valid = p < e;
      const int c = valid ? src[p] : 0;
      const bool pass = valid && cand_ok(w, F, u, c, lo, hi);
      unsigned pm = __ballot_sync(FULLMASK, pass);
      int room = 32 - nj;
      unsigned acc = pm;
      bool cut = false;
      if (__popc(acc) > room) {
        unsigned a2 = 0, t = acc;
        for (int i = 0; i < room; ++i) { unsigned lsb = t & (0u - t); a2 |= lsb; t ^= lsb; }
        acc = a2;
        cut = true;
      }
      if ((acc >> w.lane) & 1u) {
        int r = nj + __popc(acc & ((1u << w.lane) - 1));
        w.h->stage_c[r] = c;
        w.h->stage_u[r] = u;
      }
      nj += __popc(acc);
      int npos = cut ? pos + (31 - __clz(acc)) + 1 : min(pos + 32, e);
      HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
      if (w.lane == 0) w.h->it[F] = npos;
      __syncwarp();
      if (nj == 32) break;
    }
    if (nj == 0) return;
    Job J;
    J.A = nullptr; J.B = nullptr; J.alen = 0; J.blen = 0; J.op = STM_OP_NONE;
    J.lo = -1; J.hi = INT_MAX; J.lab = STM_LAB_ANY; J.out = nullptr; J.u = 0; J.c = 0; J.a_node = 0; J.abm = -1; J.bbm = -1;
    if (w.lane < nj) J = count_job(w, F, w.h->stage_u[w.lane], w.h->stage_c[w.lane], 0);
    PROF_LVL_BEGIN()
    w.cnt += run_jobs(w, J, nj, true, F, P.filt[P.k - 1].excl, nullptr);
    PROF_LVL_END(2, P.k - 1)
    __syncwarp();
  }
}
#endif  // !STM_MULTI

#if STM_MULTI
// Merged plans, last iterated frame F = k-2: while the current child builds no set node,
// pack up to 32 (sibling, candidate) pairs of that child (consecutive virtual siblings,
// child-major) and count every leaf below it over them.  Returns when the frame is
// exhausted or reaches a child that needs level-(k-1) sets (the frame path builds those).
__device__ STEP_INL void fused_count_multi(W& w, int F) {
  for (unsigned pass = 1;; ++pass) {
    if ((pass & 63) == 0 && watchdog(*w.kp, w.h->wd0, "fused")) return;  // (the main loop aborts next)
    if (w.kp->local_steal && waiting_warps(w)) share_local(*w.kp);
    if (pool_wanted(w) && w.kp->global_steal && F < w.kp->detect_level) maybe_push(*w.kp);
    int nj = 0, child = -1;
    for (;;) {
      const int u = w.h->cur[F];
      if (u >= w.h->nsib[F]) break;
      const int sv = vert_of(w, F, u);
      if (mvert(w, sv).n_build != 0 || (child >= 0 && sv != child)) break;
      child = sv;
      const int pos = w.h->it[F], e = w.h->end[F];
      if (pos >= e) {
        if (u + 1 >= w.h->nsib[F]) {
          HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
          if (w.lane == 0) w.h->cur[F] = u + 1;
          __syncwarp();
          break;
        }
        set_sibling(w, F, u + 1);
        continue;
      }
      const int* src;
      int len;
      src_slice(w, lvl_cand(w, F, u), F, u, 0, 0, src, len);
      const StmFilter f = lvl_filt(w, F, u);
      int lo, hi;
      bounds(w, f.lo, f.hi, F, u, 0, lo, hi);
      const int p = pos + w.lane;
      const bool valid = p < e;
      const int c = valid ? src[p] : 0;
      const bool pass = valid && cand_ok(w, F, u, c, lo, hi);
      unsigned acc = __ballot_sync(FULLMASK, pass);
      const int room = 32 - nj;
      bool cut = false;
      if (__popc(acc) > room) {
        unsigned a2 = 0, t = acc;
        for (int i = 0; i < room; ++i) { unsigned lsb = t & (0u - t); a2 |= lsb; t ^= lsb; }
        acc = a2;
        cut = true;
      }
      if ((acc >> w.lane) & 1u) {
        const int r = nj + __popc(acc & ((1u << w.lane) - 1));
        w.h->stage_c[r] = c;
        w.h->stage_u[r] = u;
      }
      nj += __popc(acc);
      const int npos = cut ? pos + (31 - __clz(acc)) + 1 : min(pos + 32, e);
      HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
      if (w.lane == 0) w.h->it[F] = npos;
      __syncwarp();
      if (nj == 32) break;
    }
    if (nj == 0) return;
    const StmMVert& sv = mvert(w, child);
    for (int lv = sv.child_begin; lv < sv.child_begin + sv.n_children; ++lv) {
      Job J;
      J.A = nullptr; J.B = nullptr; J.alen = 0; J.blen = 0; J.op = STM_OP_NONE;
      J.lo = -1; J.hi = INT_MAX; J.lab = STM_LAB_ANY; J.out = nullptr; J.u = 0; J.c = 0; J.a_node = 0; J.abm = -1; J.bbm = -1;
      if (w.lane < nj) J = count_job(w, F, w.h->stage_u[w.lane], w.h->stage_c[w.lane], 0, lv);
      const unsigned long long c = run_jobs(w, J, nj, true, F, mvert(w, lv).filt.excl, nullptr);
      w.cnt += c;
      if (w.lane == 0 && c) atomicAdd(&w.kp->mcount[mvert(w, lv).motif], c);
    }
    __syncwarp();
  }
}
#endif

// ----------------------------------------------------------------------------
// work acquisition: root chunks, local steal, global steal (Sec. V)
// ----------------------------------------------------------------------------
__device__ __noinline__ bool try_chunk(const StmKParams& kp) {
  W w = make_w(kp);
  int b = -1, e = -1, from = -1;
  if (w.lane == 0) {
    unsigned ex = w.h->exhausted;
    for (int i = 0; i < kp.world && b < 0; ++i) {
      int r = (kp.rank + i) % kp.world;
      if (!kp.cursors[r] || (ex & (1u << r))) continue;
      unsigned long long idx = atomicAdd(kp.cursors[r], 1ull);
      long long c = (long long)r + (long long)kp.world * (long long)idx;
      if (kp.chunk_bounds) {  // work-balanced chunks (positions [bounds[c], bounds[c+1]))
        if (c < kp.n_chunks) {
          if (kp.root_desc == 1) c = kp.n_chunks - 1 - c;  // the heaviest (last) chunks first
          else if (kp.root_desc == 2) c = (c & 1) ? kp.n_chunks - 1 - (c >> 1) : (c >> 1);  // interleaved
          from = r;
          b = __ldg(&kp.chunk_bounds[c]);
          e = __ldg(&kp.chunk_bounds[c + 1]);
        } else {
          ex |= 1u << r;
        }
        continue;
      }
      long long rb = kp.root_lo + c * (long long)kp.chunk;
      if (rb < kp.n) {
        from = r;
        b = (int)rb;
        e = (int)min((long long)kp.n, rb + kp.chunk);
        if (kp.root_desc == 1) {  // chunk c covers [lo + n - e, lo + n - b): the highest ids first
          const int nb = (int)(kp.root_lo + kp.n - e);
          e = (int)(kp.root_lo + kp.n - b);
          b = nb;
        }
      } else {
        ex |= 1u << r;
      }
    }
    w.h->exhausted = ex;
#if STM_PROFILE
    if (b < 0 && w.h->first_dry == 0) w.h->first_dry = clock64();
#endif
  }
  b = bcast(b);
  e = bcast(e);
  if (b < 0) return false;
  HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
  if (w.lane == 0) {
    w.h->root_it = b;
    w.h->root_end = e;
    w.h->L = 0;
  }
  __syncwarp();
  if (w.lane == 0) {
    atomicAdd(&kp.work->n_chunks, 1ull);
    if (from != kp.rank) atomicAdd(&kp.work->n_peer_chunks, 1ull);
  }
  return true;
}

// What a donation from the warp's own stack `v` gives away (the
// shallowest stealable remaining work).  Work at the donor's current frame L is not in
// progress yet, so there the donor always keeps at least one item (otherwise a single
// item could be passed around forever); at frames shallower than L the donor is busy
// below and may give it all.
// kind: 0 = half the root range of frame 0, 1 = half the remaining root siblings of
// frame 1, 2 = half the remaining candidates of the current sibling of frame F,
// 3 = the last not-yet-started sibling of frame F >= 2, whole.  F < 0: nothing.
struct SplitPick {
  int F, kind, t;
};

// Depth limit of donations: frames < stop_level normally; every frame while the grid is
// starving (more than 1/8 of the warps idle, WarpHdr::deep refreshed by grid_status).
// Deep donations make the receiver rebuild the donor's prefix sets, which costs as much
// as the donor's own builds (K6-e: the hub-pair intersections), so they are kept for the
// tail, where idle warps would otherwise wait.
__device__ __forceinline__ int split_stop(const StmKParams& kp, volatile WarpHdr* v) {
  return v->deep ? STM_KMAX : kp.stop_level;
}

__device__ __forceinline__ SplitPick pick_split(int stop, volatile WarpHdr* v) {
  const int L = v->L;
  const int r = v->root_end - v->root_it;
  const int t = (L > 0) ? (r + 1) / 2 : r / 2;
  if (t >= 1) return {0, 0, t};
  for (int F = 1; F <= L && F < stop; ++F) {
    const int cur = v->cur[F], nsib = v->nsib[F];
    if (cur >= nsib) continue;
    const int rem = v->end[F] - v->it[F];
    const int rs = nsib - cur - 1;  // siblings not started yet
    if (F == 1 && !STM_MULTI) {  // (merged plans: child-major frames have no whole-sibling split)
      const int ts = (L > 1 || rem > 0) ? (rs + 1) / 2 : rs / 2;
      if (ts >= 1) return {1, 1, ts};
    } else if (!STM_MULTI && rs >= 1) {
      return {F, 3, 1};
    }
    const bool last_sib = cur + 1 >= nsib;
    const int tr = (L > F || !last_sib) ? (rem + 1) / 2 : rem / 2;
    if (tr >= 1) return {F, 2, tr};
  }
  return {-1, 0, 0};
}

// Split the warp's own stack `v` (only its owner calls this).  Returns false if nothing.
__device__ __noinline__ bool split_stack(const StmKParams& kp, volatile WarpHdr* v, volatile int* vsib,
                                        StmTask& T) {
  const SplitPick s = pick_split(split_stop(kp, v), v);
  if (s.F < 0) return false;
  if (s.kind == 0) {
    T.level = 0;
    T.e = v->root_end;
    T.b = v->root_end - s.t;
    v->root_end = T.b;
  } else if (s.kind == 1) {  // remaining root siblings -> root range (entry range)
    const int s0 = v->nsib[1] - s.t;
    T.level = 0;
    T.b = kp.entries ? v->rent[s0] : vsib[1 * STM_RMAX + s0];
    T.e = (kp.entries ? v->rent[v->nsib[1] - 1] : vsib[1 * STM_RMAX + v->nsib[1] - 1]) + 1;
    v->nsib[1] = s0;
  } else if (s.kind == 3) {  // the last unstarted sibling u of frame F: prefix v_0..v_{F-2}, v_{F-1} = SIB(F, u)
    const int F = s.F;
    const int u = v->nsib[F] - 1;
    T.level = F;
    T.b = -1;  // its whole (bound-narrowed) candidate list: the receiver runs set_sibling
    T.e = -1;
    for (int j = 0; j < F - 1; ++j) T.prefix[j] = vsib[(j + 1) * STM_RMAX + v->cur[j + 1]];
    T.prefix[F - 1] = vsib[F * STM_RMAX + u];
    v->nsib[F] = u;
  } else {
    const int F = s.F;
    T.level = F;
    T.e = v->end[F];
    T.b = v->end[F] - s.t;
#if STM_MULTI
    for (int j = 0; j < F; ++j) T.prefix[j] = vsib[(j + 1) * STM_RMAX + v->cur[j + 1] % v->nr[j + 1]];
    T.tv[0] = 0;
    for (int d = 1; d <= F; ++d) T.tv[d] = (int16_t)(kp.mv[v->pv[d]].child_begin + v->cur[d] / v->nr[d]);
#else
    for (int j = 0; j < F; ++j) T.prefix[j] = vsib[(j + 1) * STM_RMAX + v->cur[j + 1]];
#endif
    v->end[F] = T.b;
  }
  return true;
}

__device__ __forceinline__ long long gtimer() {
  long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Failure detection (stm_tuning.watchdog_ms): true once the launch has run longer
// than watchdog_ns of wall time; the launch then aborts and reports STM_ETIMEOUT
// (work->overflow = 2), never a partial count.  STM_DEBUG builds also dump state.
__device__ __noinline__ bool watchdog(const StmKParams& kp, long long t0, const char* where) {
  if (!kp.watchdog_ns) return false;
  // once one warp has fired, every warp aborts at its next check
  if (*(volatile int*)&kp.work->overflow != 2 && gtimer() - t0 < kp.watchdog_ns) return false;
  W w = make_w(kp);
  if (w.lane == 0) {
    atomicExch(&w.kp->work->overflow, 2);
#if STM_DEBUG
    volatile WarpHdr* h = w.h;
    printf("WATCHDOG %s blk %d warp %d L=%d root=[%d,%d) nsib1=%d cur1=%d it1=%d end1=%d active=%d started=%d deficit=%d mask=%x poller=%d mail=%d\n",
           where, blockIdx.x, w.wid, h->L, h->root_it, h->root_end, h->nsib[1], h->cur[1], h->it[1], h->end[1],
           *(volatile int*)&w.kp->work->active, *(volatile int*)&w.kp->work->started,
           *(volatile int*)&w.kp->work->deficit, w.bh->idle_mask, w.bh->poller, h->mail_full);
#else
    (void)where;
#endif
  }
  __syncwarp();
  return true;
}

// Rebuild this warp's stack from a task (the receiver recomputes the sets of
// levels 1..T.level from the prefix).
__device__ __noinline__ void adopt_task(const StmKParams& kp, const StmTask& T) {
  W w = make_w(kp);
  if (T.level == 0) {
    HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
    if (w.lane == 0) {
      w.h->root_it = T.b;
      w.h->root_end = T.e;
      w.h->L = 0;
    }
    __syncwarp();
    return;
  }
  const int l = T.level;
  for (int i = 1; i <= l; ++i) {
    HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
    if (w.lane == 0) {
      SIB(w, i, 0) = T.prefix[i - 1];
#if STM_MULTI
      // the thief's frame i enumerates only the stolen path's child (virtual sibling ci)
      const StmMVert& pv = kp.mv[T.tv[i - 1]];
      const int ci = T.tv[i] - pv.child_begin;
      w.h->pv[i] = T.tv[i - 1];
      w.h->nr[i] = 1;
      w.h->nsib[i] = ci + 1;
      w.h->cur[i] = ci;
#else
      w.h->nsib[i] = 1;
      w.h->cur[i] = 0;
#endif
    }
    __syncwarp();
    if (i >= 2 || !STM_MULTI) {  // (i = 1: level-1 set nodes of directed plans, if any)
      int nb, ne, nst;
      bset(w, i - 1, w.h->cur[i - 1], nb, ne, nst);
      HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
      if (w.lane == 0)
        for (int s = nb; s < ne; ++s) NOFF(w, pregion(w, s), 0) = 0;
      __syncwarp();
      build_nodes(w, i - 1, 1, false);  // a stolen prefix is rebuilt as given
    }
    if (i == l && T.b < 0) {
      // a whole sibling (split kind 3): its bound-narrowed candidate range
      set_sibling(w, i, w.h->cur[i]);
    } else {
      const int len = src_len(w, i, w.h->cur[i]);
      HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
      if (w.lane == 0) {
        w.h->it[i] = (i == l) ? T.b : len;
        w.h->end[i] = (i == l) ? min(T.e, len) : len;
      }
      __syncwarp();
    }
  }
  HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
  if (w.lane == 0) w.h->L = l;
  __syncwarp();
  flush_instr(w);  // the rebuild's set operations count toward W
}

__device__ __forceinline__ volatile WarpHdr* warp_hdr(const W& w, int wid) {
  const int wb = warp_bytes(w.P->k, w.P->n_nodes, w.kp->ht_slots);
  return (volatile WarpHdr*)(stm_smem + sizeof(BlockHdr) + (size_t)wid * wb);
}

__device__ __forceinline__ void write_task(volatile StmTask* M, const StmTask& T) {
  M->level = T.level;
  M->b = T.b;
  M->e = T.e;
  for (int j = 0; j < STM_KMAX; ++j) {
    M->prefix[j] = T.prefix[j];
    M->tv[j] = T.tv[j];
  }
}
__device__ __forceinline__ void read_task(volatile StmTask* M, StmTask& T) {
  T.level = M->level;
  T.b = M->b;
  T.e = M->e;
  for (int j = 0; j < STM_KMAX; ++j) {
    T.prefix[j] = M->prefix[j];
    T.tv[j] = M->tv[j];
  }
}
__device__ __forceinline__ void bcast_task(StmTask& T) {
  T.level = bcast(T.level);
  T.b = bcast(T.b);
  T.e = bcast(T.e);
  for (int j = 0; j < STM_KMAX; ++j) {
    T.prefix[j] = bcast(T.prefix[j]);
    T.tv[j] = (int16_t)bcast(T.tv[j]);
  }
}

// Donor side of local work sharing (Sec. V-A, re-designed: the busy
// warp splits its own stack instead of an idle warp splitting it under a lock).
// Called by a busy warp that saw waiting warps in its block: claim one (clear its
// idle bit), give it the shallowest stealable part of this stack.
__device__ __noinline__ void share_local(const StmKParams& kp) {
  W w = make_w(kp);
  if (w.lane == 0 && pick_split(split_stop(kp, w.h), w.h).F >= 0) {
    unsigned want = (unsigned)*(volatile int*)&w.bh->idle_mask & ~(1u << w.wid);
    int target = -1;
    while (want && target < 0) {
      const int t = __ffs(want) - 1;
      want &= want - 1;
      if ((atomicAnd(&w.bh->idle_mask, ~(1 << t)) >> t) & 1) target = t;
    }
    if (target >= 0) {
      atomicAdd(&kp.work->active, 1);  // the claimed warp is busy from now on (termination)
      StmTask T;
      for (int j = 0; j < STM_KMAX; ++j) {
        T.prefix[j] = 0;
        T.tv[j] = 0;
      }
      split_stack(kp, w.h, w.sib, T);  // succeeds: only this warp changes its own stack
      volatile WarpHdr* th = warp_hdr(w, target);
      write_task(&th->mail, T);
      __threadfence_block();
      th->mail_full = 1;
      atomicAdd(&kp.work->n_local_steals, 1ull);
    }
  }
  __syncwarp();
}

// Donor side of global work sharing (Sec. V-B, re-designed for B200:
// a grid-wide task pool instead of per-block mailboxes).  Busy warps look at the pool's
// deficit (block pollers waiting minus queued tasks); a donor that claims one unit of it
// splits its own stack and queues the shallowest stealable part.
__device__ __noinline__ void maybe_push(const StmKParams& kp) {
  W w = make_w(kp);
  if (w.lane == 0 && *(volatile int*)&kp.work->deficit > 0 && pick_split(split_stop(kp, w.h), w.h).F >= 0) {
    if (atomicSub(&kp.work->deficit, 1) > 0) {
      StmTask T;
      for (int j = 0; j < STM_KMAX; ++j) {
        T.prefix[j] = 0;
        T.tv[j] = 0;
      }
      split_stack(kp, w.h, w.sib, T);    // succeeds: only this warp changes its own stack
      atomicAdd(&kp.work->active, 1);    // the queued task keeps the launch alive
      const unsigned long long t = atomicAdd(&kp.work->pool_tail, 1ull);
      StmPoolSlot* s = &kp.pool[t & (unsigned long long)kp.pool_mask];
      const int free_seq = (int)(2ull * (t >> kp.pool_shift));
      while (*(volatile int*)&s->seq != free_seq) __nanosleep(64);  // (the pool never fills: deficit)
      write_task(&s->task, T);
      __threadfence();
      atomicExch(&s->seq, free_seq + 1);
      atomicAdd(&kp.work->n_global_steals, 1ull);
    } else {
      atomicAdd(&kp.work->deficit, 1);
    }
  }
  __syncwarp();
}

// Pop one task from the pool (lane 0).  Returns false if the pool looked empty.
__device__ __forceinline__ bool pool_pop(const StmKParams& kp, StmTask& T) {
  volatile StmWork* vw = kp.work;
  for (;;) {
    const unsigned long long h = vw->pool_head, t = vw->pool_tail;
    if (h >= t) return false;
    if (atomicCAS(&kp.work->pool_head, h, h + 1) != h) continue;
    StmPoolSlot* s = &kp.pool[h & (unsigned long long)kp.pool_mask];
    const int full_seq = (int)(2ull * (h >> kp.pool_shift)) + 1;
    while (*(volatile int*)&s->seq != full_seq) __nanosleep(32);  // the pusher is writing it
    __threadfence();
    read_task(&s->task, T);
    atomicExch(&s->seq, full_seq + 1);  // free for the next round
    return true;
  }
}

// No more local work: returns true with new work adopted, false on termination.
// The warp leaves the active set and sets its bit in the block's idle mask (a busy warp
// of the block may then claim it and post a task into its mailbox).  One idle warp per
// block -- the poller -- also pops tasks from the grid-wide pool and detects termination:
// every warp started and `active` == 0 (no busy warp, no queued or claimed task).
__device__ __noinline__ bool acquire_work(const StmKParams& kp, long long t0) {
  W w = make_w(kp);
  if (try_chunk(kp)) return true;
  if (!kp.local_steal && !kp.global_steal) return false;
  BlockHdr* bh = w.bh;
  volatile WarpHdr* h = w.h;
  const int me = 1 << w.wid;
  if (w.lane == 0) {
    __threadfence();
    atomicSub(&kp.work->active, 1);
    if (kp.local_steal) atomicOr(&bh->idle_mask, me);
  }
  __syncwarp();
  bool poller = false;
  for (int spin = 0;; ++spin) {
    if ((spin & 63) == 63 && watchdog(kp, t0, "acquire")) return false;
    int full = 0, done = 0;
    if (w.lane == 0) {
      full = h->mail_full;
      done = *(volatile int*)&bh->done;
    }
    full = bcast(full);
    done = bcast(done);
    if (full) {  // a donor of this block claimed this warp (cleared its bit, counted it active)
      StmTask T;
      if (w.lane == 0) {
        __threadfence_block();
        read_task(&h->mail, T);
        h->mail_full = 0;
        h->steal_fails = 0;
        if (poller) {
          if (kp.global_steal) atomicSub(&kp.work->deficit, 1);
          atomicExch(&bh->poller, -1);
        }
      }
      bcast_task(T);
      adopt_task(kp, T);
      return true;
    }
    if (done) return false;
    int got = 0;
    StmTask T;
    if (w.lane == 0) {
      if (!poller && atomicCAS(&bh->poller, -1, w.wid) == -1) {
        poller = true;
        if (kp.global_steal) atomicAdd(&kp.work->deficit, 1);
      }
      if (poller) {
        volatile StmWork* vw = kp.work;
        if (vw->started == kp.total_warps && vw->active == 0) {
          atomicExch(&bh->done, 1);  // every warp of the grid is idle: nothing can appear any more
          done = 1;
        } else if (kp.global_steal && vw->pool_head < vw->pool_tail) {
          // leave local availability first (a donor may have claimed this warp already)
          const int old = kp.local_steal ? atomicAnd(&bh->idle_mask, ~me) : me;
          if (old & me) {
            if (pool_pop(kp, T)) {  // (the queued task's unit of `active` is now this warp's)
              got = 1;
              h->steal_fails = 0;
              atomicExch(&bh->poller, -1);  // (deficit: this poller leaves, one task less: net 0)
            } else if (kp.local_steal) {
              atomicOr(&bh->idle_mask, me);
            }
          }
        }
      }
    }
    poller = __shfl_sync(FULLMASK, (int)poller, 0) != 0;
    done = bcast(done);
    got = bcast(got);
    if (done) return false;
    if (got) {
      bcast_task(T);
      adopt_task(kp, T);
      return true;
    }
    if (w.lane == 0) {
      __nanosleep(32u << h->steal_fails);  // back off while no work arrives
      h->steal_fails = min(h->steal_fails + 1, kp.backoff_max);
    }
    __syncwarp();
  }
}

}  // namespace

// One main-loop iteration at frame F >= 1: the fused count of frame k-2, or the next
// batch of frame F (gather -> build frame F+1 -> descend), or the backtrack.  FC >= 0:
// F == FC is a compile-time constant (plan-specialised builds, STM_CPLAN: every plan
// lookup indexed by the frame folds to a constant and the node loops unroll).
template <int FC>
__device__ __forceinline__ void frame_step(W& w, const StmKParams& kp, int Fr, int k, int U, bool fused) {
  const int F = FC >= 0 ? FC : Fr;
#if STM_MULTI
  if (F == k - 2 && mvert(w, vert_of(w, F, w.h->cur[F])).n_build == 0 && w.h->cur[F] < w.h->nsib[F]) {
    fused_count_multi(w, F);
    if (w.h->cur[F] < w.h->nsib[F]) return;  // stopped at a child that builds sets
    HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
    if (w.lane == 0) w.h->L = F - 1;
    __syncwarp();
    return;
  }
#endif
  if (fused && F == k - 2) {
    PROF_BEGIN(5)
#if !STM_MULTI
    fused_count(w, F);
#endif
    PROF_END(5, 0)
    HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
    if (w.lane == 0) w.h->L = F - 1;
    __syncwarp();
    return;
  }
  // donors look at the pool's demand at frames < detect_level (they donate only work of
  // frames < stop_level: pick_split)
  if (pool_wanted(w) && kp.global_steal && F < kp.detect_level) {
    PROF_BEGIN(6)
    maybe_push(kp);
    PROF_END(6, 0)
  }
  int m = 0;
  bool back = false;
  for (;;) {
    if (w.h->cur[F] >= w.h->nsib[F]) { back = true; break; }
    if (w.h->it[F] < w.h->end[F]) {
      int Ub = U;
#if STM_MULTI
      {  // a frame that builds no set node has no per-sibling slice table: batch up to 32
        int nb, ne, nst;
        bset(w, F, w.h->cur[F], nb, ne, nst);
        if (nb == ne) Ub = STM_RMAX;
      }
#endif
      PROF_BEGIN(2)
      m = gather_batch(w, F, Ub);
      PROF_END(2, m)
      if (m > 0) break;
    }
    int nu = w.h->cur[F] + 1;
    if (nu >= w.h->nsib[F]) {
      HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
      if (w.lane == 0) w.h->cur[F] = nu;
      __syncwarp();
      back = true;
      break;
    }
    PROF_BEGIN(8)
    set_sibling(w, F, nu);
    PROF_END(8, 1)
  }
  if (back) {
    HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
    if (w.lane == 0) w.h->L = F - 1;
    __syncwarp();
    return;
  }
  // build frame F+1 from the batch
  PROF_BEGIN(3)
  m = build_nodes(w, F, m, true);
  PROF_END(3, m)
  if (m == 0) return;  // every sibling of the batch was pruned: gather the next one
  if (F + 1 == k - 1) {  // frame-count mode
    PROF_BEGIN(4)
    frame_count(w, m);
    PROF_END(4, m)
    return;
  }
  HDR_SYNC();  // every lane has read the header fields lane 0 rewrites
  if (w.lane == 0) {
#if STM_MULTI
    const int sv = vert_of(w, F, w.h->cur[F]);
    w.h->pv[F + 1] = sv;
    w.h->nr[F + 1] = m;
    w.h->nsib[F + 1] = m * kp.mv[sv].n_children;
#else
    w.h->nsib[F + 1] = m;
#endif
  }
  __syncwarp();
  PROF_BEGIN(9)
  set_sibling(w, F + 1, 0);
  PROF_END(9, 1)
  // (reads above are ordered before this write by a full-warp collective)
  if (w.lane == 0) w.h->L = F + 1;
  __syncwarp();
}

// ----------------------------------------------------------------------------
// the kernel
// ----------------------------------------------------------------------------
__device__ __forceinline__ void stm_count_body(const StmKParams& kp) {
  const StmPlan& P = STM_PLAN_OF(kp);
  BlockHdr* bh = (BlockHdr*)stm_smem;
  const int lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    bh->idle_mask = 0;
    bh->poller = -1;
    bh->done = 0;
  }
  for (int i = threadIdx.x; i < 256; i += blockDim.x) bh->lab2slot[i] = kp.lab2slot[i];
  W w = make_w(kp);
  if (lane == 0) {
    w.h->mail_full = 0;
    w.h->L = 0;
    w.h->root_it = 0;
    w.h->root_end = 0;
    w.h->exhausted = 0;
    w.h->donate_tick = 0;
    w.h->steal_fails = 0;
    w.h->first_dry = 0;
    w.h->gchk = 0;
    w.h->deep = 0;
    w.h->wd0 = gtimer();
    for (int i = 0; i < STM_KMAX; ++i) {
      w.h->nsib[i] = 0;
      w.h->cur[i] = 0;
      w.h->it[i] = 0;
      w.h->end[i] = 0;
    }
    // termination accounting (acquire_work): this warp is active, then it has started
    atomicAdd(&kp.work->active, 1);
    __threadfence();
    atomicAdd(&kp.work->started, 1);
  }
  __syncthreads();

  const int k = P.k;
  const int U = max(1, min(kp.unroll, STM_UMAX));
  const bool fused = !STM_MULTI && P.count_mode == STM_COUNT_FUSED;
  const long long t0 = clock64();
  const long long wd0 = gtimer();
  unsigned iter = 0;
  for (;;) {
    if ((++iter & 15) == 0 && watchdog(kp, wd0, "main")) break;
    // local work sharing: a busy warp serves the idle warps of its block (one shared-
    // memory load per iteration; the split runs only when a warp is waiting)
    PROF_CHK()
    if (kp.local_steal && waiting_warps(w)) share_local(kp);
    int L = w.h->L;
    if (L == 0) {
      PROF_BEGIN(0)
      int m = gather_roots(w);
      PROF_END(0, m)
      if (m > 0) {
        // (reads above are ordered before this write by a full-warp collective)
        if (w.lane == 0) {
#if STM_MULTI
          w.h->pv[1] = 0;
          w.h->nr[1] = m;
          w.h->nsib[1] = m * kp.mv[0].n_children;
#else
          w.h->nsib[1] = m;
#endif
          w.h->cur[1] = 0;
        }
        __syncwarp();
#if !STM_MULTI
        if (P.level_begin[1] != P.level_begin[2]) {
          // level-1 set nodes (directed plans: e.g. N+(v0) & N-(v0) for a mutual arc), built
          // per root (root_batch is 1 for such plans: offset 0 in every node region)
          HDR_SYNC();
          if (w.lane == 0)
            for (int s = P.level_begin[1]; s < P.level_begin[2]; ++s) NOFF(w, s, 0) = 0;
          __syncwarp();
          m = build_nodes(w, 0, m, true);
          if (m == 0) continue;  // the root cannot be extended: next root
        }
#endif
        PROF_BEGIN(1)
        set_sibling(w, 1, 0);
        PROF_END(1, 1)
        if (k == 2) {
          frame_count(w, m);  // counts N(root) per root
          continue;
        }
        // (reads above are ordered before this write by a full-warp collective)
        if (w.lane == 0) w.h->L = 1;
        __syncwarp();
      }
      if (m == 0) {
        // instrumented launches: time spent acquiring work (cursor, stealing, idle
        // waiting) vs the warp's whole lifetime -> idle/stealing fraction (north_star)
        const long long ta = (STM_INSTR && kp.count_bytes) ? clock64() : 0;
#if STM_PROFILE
        if (lane == 0) prof_timeline(w);  // busy until now
#endif
        PROF_BEGIN(7)
        const bool got = acquire_work(kp, wd0);
        PROF_END(7, got)
#if STM_PROFILE
        w.prof_chk = 0;  // idle time is not a busy interval
        w.prof_g = 0;
#endif
        if (STM_INSTR && kp.count_bytes) w.idle_cyc += (unsigned long long)(clock64() - ta);
        if (!got) break;
      }
      continue;
    }
#if STM_CPLAN
    switch (L) {  // a specialised copy per frame 1..k-2 (frames >= k-1 are never entered)
      case 1: frame_step<1>(w, kp, L, k, U, fused); break;
#if STM_CPLAN_K > 3
      case 2: frame_step<2>(w, kp, L, k, U, fused); break;
#endif
#if STM_CPLAN_K > 4
      case 3: frame_step<3>(w, kp, L, k, U, fused); break;
#endif
#if STM_CPLAN_K > 5
      case 4: frame_step<4>(w, kp, L, k, U, fused); break;
#endif
#if STM_CPLAN_K > 6
      case 5: frame_step<5>(w, kp, L, k, U, fused); break;
#endif
#if STM_CPLAN_K > 7
      case 6: frame_step<6>(w, kp, L, k, U, fused); break;
#endif
      default: break;
    }
#else
    frame_step<-1>(w, kp, L, k, U, fused);
#endif
  }
  if (lane == 0 && w.cnt) atomicAdd(&kp.work->count, w.cnt);
#if STM_PROFILE
  if (lane == 0) {
    for (int i = 0; i < STM_PROF_N; ++i) {
      atomicAdd(&kp.work->prof[3 * i], w.prof_cyc[i]);
      atomicAdd(&kp.work->prof[3 * i + 1], w.prof_cnt[i]);
      atomicAdd(&kp.work->prof[3 * i + 2], w.prof_items[i]);
    }
    const long long now = clock64();
    atomicAdd(&kp.work->prof[3 * STM_PROF_N], (unsigned long long)(now - t0));
    prof_timeline(w);
    prof_timeline_flush(w);
    // tail shape (clock64 is per SM; SMs start within a few us of each other)
    atomicMax(&kp.work->prof[3 * STM_PROF_N + 1], (unsigned long long)(now - t0));
    const long long fd = w.h->first_dry;
    atomicAdd(&kp.work->prof[3 * STM_PROF_N + 2], (unsigned long long)(fd ? fd - t0 : now - t0));
    atomicMax(&kp.work->prof[3 * STM_PROF_N + 3], (unsigned long long)(fd ? fd - t0 : now - t0));
  }
#endif
  if (STM_INSTR && kp.count_bytes) {
    flush_instr(w);
    if (lane == 0) {
      atomicAdd(&kp.work->idle_cycles, w.idle_cyc);
      atomicAdd(&kp.work->warp_cycles, (unsigned long long)(clock64() - t0));
    }
  }
  // The last block to finish publishes the async result record (stm_async_result):
  // every warp's count is ordered before its block's arrival by the fence.
  if (kp.result) {
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) {
      const unsigned done = atomicAdd(&kp.work->blocks_done, 1u);
      if (done == gridDim.x - 1) {
        __threadfence();
        volatile StmWork* vw = kp.work;
        const int ov = vw->overflow;
        kp.result[0] = ov ? 0ull : vw->count;
        kp.result[1] = ov == 2 ? 6ull /* STM_ETIMEOUT */ : ov ? 5ull /* STM_EOVERFLOW */ : 0ull;
        kp.result[2] = vw->n_chunks;
        kp.result[3] = vw->n_peer_chunks;
      }
    }
  }
}

// Two register budgets of the same kernel (stm_tuning.occupancy): 64 registers ->
// 32 resident warps per SM, or 32 registers (with spills) -> 64 warps per SM, which
// hides more DRAM latency when the graph does not fit in L2 (measured).
#ifdef STM_NVRTC
#define STM_KLINK extern "C"  // JIT builds: unmangled names for cudaLibraryGetKernel
#else
#define STM_KLINK
#endif
#if !defined(STM_JIT_VARIANT) || STM_JIT_VARIANT == 1
STM_KLINK __global__ void __launch_bounds__(STM_MAXT, 1) STM_SYM(stm_count_kernel)(const __grid_constant__ StmKParams kp) {
  stm_count_body(kp);
}
#endif
#if !defined(STM_JIT_VARIANT) || STM_JIT_VARIANT == 2
STM_KLINK __global__ void __launch_bounds__(STM_OCC_MAXT, 1) STM_SYM(stm_count_kernel_occ)(const __grid_constant__ StmKParams kp) {
  stm_count_body(kp);
}
#endif

#ifndef STM_NVRTC  // host side of the launch (never part of a JIT compile)

static const void* STM_SYM(kernel_fn)(int variant) {
  return variant == 2 ? (const void*)STM_SYM(stm_count_kernel_occ) : (const void*)STM_SYM(stm_count_kernel);
}

static int local_smem_bytes(int block_warps, int k, int n_nodes, int ht_slots) {
  return (int)sizeof(BlockHdr) + block_warps * warp_bytes(k, n_nodes, ht_slots);
}

#if !STM_INSTR && !STM_LIST && !STM_MULTI
int stm_drive_compiled() { return 0; }  // drive_ratio / hash sets: measured slower, removed
int stm_hash_compiled() { return 0; }

int stm_smem_bytes(int block_warps, int k, int n_nodes, int ht_slots) {
  return local_smem_bytes(block_warps, k, n_nodes, ht_slots);
}
#endif
#if STM_MULTI
int stm_smem_bytes_multi(int block_warps, int k, int n_regions) {
  return local_smem_bytes(block_warps, k, n_regions, 0);
}
#endif

int STM_SYM(stm_occupancy_fn)(const void* fn, int block_warps, int k, int n_nodes, int ht_slots, int carveout,
                              int* blocks_per_sm);
int STM_SYM(stm_launch_fn)(const void* fn, const StmKParams& kp, int grid, void* stream);

int STM_SYM(stm_occupancy)(int variant, int block_warps, int k, int n_nodes, int ht_slots, int carveout,
                           int* blocks_per_sm) {
  return STM_SYM(stm_occupancy_fn)(STM_SYM(kernel_fn)(variant), block_warps, k, n_nodes, ht_slots, carveout,
                                   blocks_per_sm);
}

int STM_SYM(stm_occupancy_fn)(const void* fn, int block_warps, int k, int n_nodes, int ht_slots, int carveout,
                              int* blocks_per_sm) {
  int smem = local_smem_bytes(block_warps, k, n_nodes, ht_slots);
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return (int)e;
  // The DFS stacks are the only shared-memory users: carve out just enough shared
  // memory for the register-limited number of resident blocks and leave the rest
  // of the unified 256 KB array to L1, which caches the binary-search probes.
  cudaFuncAttributes fa;
  e = cudaFuncGetAttributes(&fa, fn);
  if (e != cudaSuccess) return (int)e;
  const int threads = block_warps * 32;
  const int regs_per_warp = ((fa.numRegs * 32 + 255) / 256) * 256;
  int want = std::min(65536 / std::max(1, regs_per_warp * block_warps), 64 / block_warps);
  want = std::max(1, std::min(want, 32));
  const double need = (double)want * (smem + 1024);
  int pct = (int)std::ceil(100.0 * need / (228.0 * 1024.0));
  pct = std::max(0, std::min(100, pct));
  if (carveout != 0) pct = carveout;  // stm_tuning.carveout_pct: -1 = leave the driver default
  if (pct >= 0) {
    e = cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, pct);
    if (e != cudaSuccess) return (int)e;
  }
  (void)threads;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, fn, block_warps * 32, smem);
  return (int)e;
}

int STM_SYM(stm_launch)(int variant, const StmKParams& kp, int grid, void* stream) {
  return STM_SYM(stm_launch_fn)(STM_SYM(kernel_fn)(variant), kp, grid, stream);
}

int STM_SYM(stm_launch_fn)(const void* fn, const StmKParams& kp, int grid, void* stream) {
  int smem = local_smem_bytes(kp.block_warps, kp.plan.k, kp.plan.n_nodes, kp.ht_slots);
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return (int)e;
  void* args[] = {(void*)&kp};
  // cooperative launch (co-residency for the spin-waiting scheduler) with an optional
  // L2 access-policy window that keeps the hottest neighbour lists persisting in L2
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kp.block_warps * 32);
  cfg.dynamicSmemBytes = (size_t)smem;
  cfg.stream = (cudaStream_t)stream;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  int na = 1;
  if (kp.l2_window_bytes > 0) {
    at[1].id = cudaLaunchAttributeAccessPolicyWindow;
    at[1].val.accessPolicyWindow.base_ptr = (void*)kp.l2_window_base;
    at[1].val.accessPolicyWindow.num_bytes = (size_t)kp.l2_window_bytes;
    at[1].val.accessPolicyWindow.hitRatio = 1.0f;
    at[1].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    at[1].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    na = 2;
  }
  cfg.attrs = at;
  cfg.numAttrs = na;
  e = cudaLaunchKernelExC(&cfg, fn, args);
  return (int)e;
}
#endif  // !STM_NVRTC
