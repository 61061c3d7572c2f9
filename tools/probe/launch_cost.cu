// Development probe: the fixed cost of a persistent-worker launch on B200.
// Back-to-back launches of near-empty kernels (1184 CTAs x 256 threads, the
// occupancy of an 8-CTA/SM worker) that add, one at a time, the steps of the
// slate worker's prologue/epilogue; mean time per launch over 200 launches.
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

struct Ctl { unsigned next; unsigned pad0[31]; unsigned long long done, live; unsigned started; unsigned pad1[27];
             unsigned long long live2; unsigned pad2[30]; unsigned long long ctrl; unsigned pad3[30]; };

__device__ __forceinline__ unsigned long long ld_acq(const unsigned long long* p) {
  unsigned long long v; asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ unsigned smid() { unsigned r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }

// mode bits: 1 fetch atomic (round trip) + barrier, 2 acquire load of ctrl, 4 three REDs on one line (join),
// 8 REDs at exit, 16 sys fence + mapped write by the last CTA, 32 rank LUT load, 64 REDs spread over lines
template <int MODE>
__global__ void __launch_bounds__(256, 8) k(Ctl* c, volatile unsigned* host, const unsigned short* lut, unsigned B) {
  __shared__ unsigned s_g;
  unsigned r = 0;
  if (threadIdx.x == 0) {
    if (MODE & 32) r = lut[smid()];
    if (MODE & 2) r += unsigned(ld_acq(&c->ctrl));
    if (MODE & 4) { atomicAdd(&c->live, 1ull); atomicAdd(&c->started, 1u); atomicAdd(&c->done, 1ull); }
    if (MODE & 64) { atomicAdd(&c->live, 1ull); atomicAdd(&c->started, 1u); atomicAdd(&c->live2, 1ull); }
    s_g = (MODE & 1) ? atomicAdd(&c->next, 1u) : B;
  }
  __syncthreads();
  if (s_g < B && threadIdx.x == 0) c->pad0[1] = r;
  if (threadIdx.x == 0) {
    if (MODE & 8) { atomicAdd(&c->live, ~0ull); }
    if (MODE & 16) {
      const unsigned long long o = atomicAdd(&c->done, 1ull << 32);
      if ((o >> 32) + 1 == gridDim.x) { __threadfence_system(); *host = 1; }
    }
  }
}

template <int MODE>
float run(Ctl* c, volatile unsigned* h, const unsigned short* lut, int grid, cudaStream_t st) {
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  for (int w = 0; w < 20; ++w) { cudaMemsetAsync(c, 0, sizeof(Ctl), st); k<MODE><<<grid, 256, 0, st>>>(c, h, lut, 16); }
  cudaEventRecord(a, st);
  for (int i = 0; i < 200; ++i) { cudaMemsetAsync(c, 0, sizeof(Ctl), st); k<MODE><<<grid, 256, 0, st>>>(c, h, lut, 16); }
  cudaEventRecord(b, st);
  cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  return ms * 1e3f / 200;
}

int main() {
  Ctl* c; unsigned short* lut; unsigned* h; unsigned* hd;
  CK(cudaMalloc(&c, sizeof(Ctl)));
  CK(cudaMalloc(&lut, 4096));
  CK(cudaMemset(lut, 0, 4096));
  CK(cudaHostAlloc(&h, 64, cudaHostAllocMapped));
  CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
  cudaStream_t st; CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  // memset-only baseline
  {
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a, st);
    for (int i = 0; i < 200; ++i) cudaMemsetAsync(c, 0, sizeof(Ctl), st);
    cudaEventRecord(b, st); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); printf("memset only            %.2f us\n", ms * 1e3f / 200);
  }
  for (int grid : {16, 148, 1184}) {
    printf("grid %4d: empty %.2f  fetch %.2f  +acq %.2f  +3red %.2f  +exit-red %.2f  +sysfence %.2f  +lut %.2f  spread-red %.2f  all %.2f us\n", grid,
           run<0>(c, hd, lut, grid, st), run<1>(c, hd, lut, grid, st), run<3>(c, hd, lut, grid, st),
           run<7>(c, hd, lut, grid, st), run<15>(c, hd, lut, grid, st), run<31>(c, hd, lut, grid, st),
           run<63>(c, hd, lut, grid, st), run<1 | 64>(c, hd, lut, grid, st), run<63 | 64>(c, hd, lut, grid, st));
  }
  CK(cudaGetLastError());
  return 0;
}
