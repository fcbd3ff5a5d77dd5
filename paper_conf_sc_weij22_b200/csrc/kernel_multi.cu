// kernel_multi.cu -- the merged-census build of the persistent kernel (NEXT-3, pattern
// merging): kernel.cu with the trie plan access (STM_MULTI) and 8 unrolled
// siblings per frame (the trie's shared set regions multiply the per-warp stack).
#define STM_MULTI 1
#define STM_UMAX 8
#include "kernel.cu"
