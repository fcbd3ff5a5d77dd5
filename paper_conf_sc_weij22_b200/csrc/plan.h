// plan.h -- compiled pattern plan shared by the host compiler, the runtime and the
// kernel (product code only; the oracle never sees it).
//
// Notation (Sec. II-B): the matching order pi places pattern vertex
// pi[l] at level l; v_l is its image.  "Entering level l" means v_0..v_{l-1} are
// fixed and the candidate set of level l is computed ("getCandidates",
// PAPER.md:75-76).  A *set node* is a materialised set (the paper's C / C_21 sets,
// PAPER.md:136) defined by one operation
//
//         node = A  (op)  N(v_b)         op in {intersect, difference}
//
// where A is an earlier node or a raw neighbour list N(v_a).  Nodes carry a
// label mask (merged multi-label sets) and value bounds from the
// symmetry-breaking restrictions shared by all their consumers.  This encoding
// replaces the paper's (first-operand flag, op, dependency) triples
// (self-contradictory in the extracted text; reading R7).
#pragma once
#ifndef STM_NVRTC
#include <stdint.h>
#endif

#define STM_KMAX 8
#define STM_MAX_NODES 32
#ifndef STM_UMAX
#define STM_UMAX 32
#endif
// max siblings per unrolled frame (levels >= 2)
#define STM_RMAX 32        // max root siblings in frame 1

enum { STM_SRC_NODE = 0, STM_SRC_RAW = 1 };
enum { STM_OP_AND = 0, STM_OP_DIFF = 1, STM_OP_NONE = 2 };
enum { STM_COUNT_FUSED = 0,   // count over (sibling, candidate) pairs of frame k-2
       STM_COUNT_FRAME = 1 }; // frame k-1 is built; count one final op per sibling

#define STM_LAB_ANY 0xFFu

struct StmNode {
  int8_t level;     // computed when entering this level
  int8_t stage;     // dependency stage within the level (0 = operands from earlier levels)
  int8_t a_kind;    // STM_SRC_NODE / STM_SRC_RAW
  int8_t b;         // position code of N(v_b): j (+ 8 for the in-row of a directed plan)
  int8_t op;        // STM_OP_AND / STM_OP_DIFF
  uint8_t lab;      // label-slot mask (STM_LAB_ANY = no label filter)
  uint8_t lo;       // bitmask of positions j: keep w > v_j
  uint8_t hi;       // bitmask of positions j: keep w < v_j
  int16_t a;        // node index (merged plans: pool index) or position code of N(v_a)
  uint8_t pad[2];
};

// Candidate filter of one level: label, bounds, exclusions (injectivity for
// pattern non-neighbours).
struct StmFilter {
  uint8_t lab, lo, hi, excl;
};

struct StmSrc {
  int8_t kind;  // STM_SRC_NODE / STM_SRC_RAW
  int8_t pad;
  int16_t idx;  // node index (merged plans: pool index) or position code (j, + 8: in-row)
};

struct StmPlan {
  int32_t k;
  int32_t n_nodes;
  int32_t vertex_induced;
  int32_t count_mode;
  int32_t n_label_slots;             // distinct non-wildcard pattern labels
  int32_t label_value[STM_KMAX];     // slot -> pattern label value
  int32_t order[STM_KMAX];           // pi
  int8_t level_begin[STM_KMAX + 1];  // nodes of level l: [level_begin[l], level_begin[l+1])
  int8_t n_stages[STM_KMAX];
  StmNode nodes[STM_MAX_NODES];
  StmSrc cand[STM_KMAX];             // candidate source of levels 1..k-1
  StmFilter filt[STM_KMAX];          // candidate filter of levels 0..k-1
  // final (count) operation at level k-1: count |A op N(v_b)| under filt[k-1]
  StmSrc cnt_a;
  int8_t cnt_b;                      // position code, or -1 when op == STM_OP_NONE
  int8_t cnt_op;
  int8_t directed;                   // 1: raw operands name out- (code j) or in-rows (code j + 8)
  int8_t pad;
  // Candidate-set pruning: need[l] = the minimal size of level l's
  // candidate set (within its bounds) for any embedding to extend the prefix -- v_l itself
  // plus every later v_m that must also come from it; a sibling whose level-(l) set is
  // smaller is dropped before its frame is entered.  pretest[l] = 1: level l's candidate
  // source is an unbounded stage-0 node of level l with a bounded consumer -- its size
  // within the consumer's bounds is counted on bound-narrowed operands first, and the
  // level's sets are materialised only for the siblings that pass.
  int8_t need[STM_KMAX];
  int8_t pretest[STM_KMAX];
};
