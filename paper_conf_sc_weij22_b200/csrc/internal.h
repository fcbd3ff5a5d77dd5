// internal.h -- host-side library internals (product code).
#pragma once
#include <stdint.h>

#include <string>
#include <utility>
#include <vector>

#include "../../include/stm.h"
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
