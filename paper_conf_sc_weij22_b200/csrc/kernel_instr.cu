// kernel_instr.cu -- the instrumented build of the matching kernel (stm_tuning.instrument = 1):
// the same source with the algorithmic-byte and idle-cycle counters compiled in,
// so that the production kernels carry no counter registers.
#define STM_INSTR 1
#include "kernel.cu"
