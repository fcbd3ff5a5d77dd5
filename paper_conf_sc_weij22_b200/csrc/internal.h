// internal.h -- host-side library internals (product code).
#pragma once
#include <stdint.h>

#include <string>
#include <utility>
#include <vector>

#include "../../include/stm.h"
#include "kernel.h"
#include "plan.h"

struct stm_plan {
  StmPlan dev;  // POD consumed by the kernel
  int k = 0;
  std::vector<std::pair<int, int>> edges;
  std::vector<int> labels;  // empty = unlabeled
  std::vector<std::pair<int, int>> restr;
  int64_t aut = 0;
  uint32_t flags = 0;
  bool order_free = false;  // restrictions hold for every total order of V (GK or none)
  std::string describe;
};

// records a thread-local error message and returns the status
stm_status stm_fail(stm_status s, const char* fmt, ...);

// Merged multi-pattern plan (motif census, NEXT-3): host copy of the trie that
// motif.cpp builds and runtime.cu uploads for the STM_MULTI kernel (kernel.h).
struct stm_merged {
  int k = 0;
  int n_patterns = 0;
  int n_regions = 0;                 // set-node storage regions per warp
  std::vector<StmMVert> verts;       // the trie, children contiguous (BFS numbering)
  std::vector<StmMNode> nodes;       // node pool
  bool order_free = true;            // every pattern uses order-free (GK) restrictions
};
// one persistent launch of the merged plan; counts[i] += count of pattern i
stm_status stm_launch_merged(const stm_graph* g, const stm_merged& m, const stm_tuning* t, void* stream,
                             uint64_t* counts);

// plan-specialised counting kernel of P for a register variant (jit.cpp): compiled with
// NVRTC on first use and cached; NULL (with *err) if it cannot be built
const void* stm_jit_kernel(const StmPlan& P, int variant, std::string* err);
int stm_jit_cache_size();
