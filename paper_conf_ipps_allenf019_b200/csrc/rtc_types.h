// rtc_types.h -- what the device headers need from the C/CUDA headers, also
// under NVRTC (the runtime compiler of user kernels, NEXT-3) which has no C
// library headers.
#pragma once
#ifdef __CUDACC_RTC__
typedef unsigned char uint8_t;
typedef unsigned short uint16_t;
typedef unsigned int uint32_t;
typedef unsigned long long uint64_t;
typedef int int32_t;
typedef long long int64_t;
#else
#include <cstddef>
#include <cstdint>
#include <cuda_runtime.h>
#endif
