// stm_nvrtc_prelude.h -- what the plan-specialised JIT compile of kernel.cu (runtime.cu
// jit_kernel, NVRTC: no system headers) needs from <cstdint> / <climits>.  Product code.
#pragma once
typedef signed char int8_t;
typedef unsigned char uint8_t;
typedef short int16_t;
typedef unsigned short uint16_t;
typedef int int32_t;
typedef unsigned int uint32_t;
typedef long long int64_t;
typedef unsigned long long uint64_t;
#define INT_MAX 2147483647
#define INT32_MAX 2147483647
#define INT32_MIN (-2147483647 - 1)
