// kernel_list.cu -- the listing build of the matching kernel (stm_match_list, SURVEY.md 8(f)
// NEXT-1): the same source with the last level emitting every embedding into a bounded
// device buffer (PAPER.md:75 Output(C, iter)) instead of only counting it.
#define STM_LIST 1
#include "kernel.cu"
