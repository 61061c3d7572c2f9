// Development probe: FP32 throughput of scalar FFMA vs packed FFMA2 (fma.rn.f32x2)
// on sm_100a.  Each thread runs 8 independent FMA chains for ITER steps; the
// FFMA2 kernel does the same number of scalar FMAs as 4 packed chains.
#include <cuda_runtime.h>
#include <cstdio>

#define ITER 4096

__device__ __forceinline__ unsigned long long ffma2(unsigned long long a, unsigned long long b, unsigned long long c) {
  unsigned long long d;
  asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}

__global__ void k_ffma(float* out, float s) {
  float x[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) x[j] = threadIdx.x * 1e-3f + j;
  for (int i = 0; i < ITER; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) x[j] = __fmaf_rn(x[j], s, 0.5f);
  float r = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) r += x[j];
  out[blockIdx.x * blockDim.x + threadIdx.x] = r;
}

__global__ void k_ffma2(float* out, float s) {
  unsigned long long x[4];
  float2 f;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    f = make_float2(threadIdx.x * 1e-3f + 2 * j, threadIdx.x * 1e-3f + 2 * j + 1);
    x[j] = *reinterpret_cast<unsigned long long*>(&f);
  }
  float2 sv = make_float2(s, s), hv = make_float2(0.5f, 0.5f);
  const unsigned long long S = *reinterpret_cast<unsigned long long*>(&sv), H = *reinterpret_cast<unsigned long long*>(&hv);
  for (int i = 0; i < ITER; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) x[j] = ffma2(x[j], S, H);
  float r = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    f = *reinterpret_cast<float2*>(&x[j]);
    r += f.x + f.y;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = r;
}

int main() {
  float* out;
  cudaMalloc(&out, 148 * 8 * 256 * sizeof(float));
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const double fmas = 148.0 * 8 * 256 * ITER * 8;
  for (int rep = 0; rep < 2; ++rep) {
    float ms1, ms2;
    cudaEventRecord(a);
    k_ffma<<<148 * 8, 256>>>(out, 0.999f);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms1, a, b);
    cudaEventRecord(a);
    k_ffma2<<<148 * 8, 256>>>(out, 0.999f);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms2, a, b);
    if (rep) printf("FFMA  %.3f ms  %.1f TFLOP/s\nFFMA2 %.3f ms  %.1f TFLOP/s\n", ms1, 2 * fmas / ms1 / 1e9, ms2,
                    2 * fmas / ms2 / 1e9);
  }
  return 0;
}
