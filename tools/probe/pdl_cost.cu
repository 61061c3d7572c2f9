// Development probe: programmatic dependent launch (PDL) between back-to-back
// persistent worker kernels.  Each launch: 1184 CTAs x 256 threads, a prologue
// of two global round trips, then tasks of one 8-KB block copy each from a
// per-launch counter (B blocks), the counter of the NEXT launch pre-zeroed.
// Modes: plain launches; PDL (the next grid's CTAs start as this grid's CTAs
// run out of work and wait in griddepcontrol.wait); PDL with a CUDA event
// recorded between the launches (does the event break the overlap?).
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ unsigned long long ld_acq(const unsigned long long* p) {
  unsigned long long v; asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v;
}

template <bool PDL>
__global__ void __launch_bounds__(256, 8) k(unsigned* ctr, const unsigned long long* ctrl, const float4* src, float4* dst,
                                            unsigned B) {
  __shared__ unsigned s_g;
  if (threadIdx.x == 0) s_g = unsigned(ld_acq(ctrl)) + *(volatile unsigned*)(ctr + 64);
  __syncthreads();
  if (PDL) asm volatile("griddepcontrol.wait;" ::: "memory");   // the previous grid completed, memory visible
  for (;;) {
    if (threadIdx.x == 0) s_g = atomicAdd(ctr, 1u);
    __syncthreads();
    const unsigned g = s_g;
    __syncthreads();
    if (g >= B) break;
    for (int i = threadIdx.x; i < 512; i += 256) dst[size_t(g) * 512 + i] = src[size_t(g) * 512 + i];
  }
  if (PDL) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

template <bool PDL>
cudaError_t launch(unsigned* ctr, const unsigned long long* ctrl, const float4* s, float4* d, unsigned B, cudaStream_t st) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(1184);
  cfg.blockDim = dim3(256);
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = PDL ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, k<PDL>, ctr, ctrl, s, d, B);
}

int main() {
  const int N = 400;
  unsigned* ctr; unsigned long long* ctrl; float4 *s, *d;
  const unsigned Bmax = 16384;
  CK(cudaMalloc(&ctr, sizeof(unsigned) * 128 * (N + 1)));
  CK(cudaMalloc(&ctrl, 64));
  CK(cudaMemset(ctrl, 0, 64));
  CK(cudaMalloc(&s, size_t(Bmax) * 8192));
  CK(cudaMalloc(&d, size_t(Bmax) * 8192));
  cudaStream_t st; CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  cudaEvent_t a, b, mid[N];
  cudaEventCreate(&a); cudaEventCreate(&b);
  for (int i = 0; i < N; ++i) cudaEventCreate(&mid[i]);
  for (unsigned B : {16u, 2048u, 16384u}) {
    for (int mode = 0; mode < 3; ++mode) {
      for (int rep = 0; rep < 2; ++rep) {
        CK(cudaMemsetAsync(ctr, 0, sizeof(unsigned) * 128 * (N + 1), st));
        CK(cudaEventRecord(a, st));
        for (int i = 0; i < N; ++i) {
          unsigned* c = ctr + 128 * i;
          if (mode == 0) CK(launch<false>(c, ctrl, s, d, B, st));
          else CK(launch<true>(c, ctrl, s, d, B, st));
          if (mode == 2) CK(cudaEventRecord(mid[i], st));
        }
        CK(cudaEventRecord(b, st));
        CK(cudaEventSynchronize(b));
        float ms; cudaEventElapsedTime(&ms, a, b);
        if (rep == 1)
          printf("B %5u  %-16s %8.2f us per launch\n", B, mode == 0 ? "plain" : mode == 1 ? "PDL" : "PDL+event", ms * 1e3f / N);
      }
    }
  }
  CK(cudaGetLastError());
  return 0;
}
