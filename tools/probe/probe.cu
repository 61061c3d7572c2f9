// Early hardware probe (not product code): SM-id calibration, copy bandwidth vs
// number of SMs (the paper's Fig. 1 experiment, §II), and the latency of a
// cuStreamWriteValue64 control write observed by a spinning persistent kernel.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <chrono>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); return 1; } } while (0)

__device__ __forceinline__ unsigned smid() { unsigned r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }
__device__ __forceinline__ unsigned long long gtimer() { unsigned long long r; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(r)); return r; }

__global__ void k_smid(unsigned* out) {
  if (threadIdx.x == 0) out[blockIdx.x] = smid();
  // keep resident a little so the placement spreads
  unsigned long long t0 = gtimer();
  while (gtimer() - t0 < 20000) {}
}

__constant__ unsigned short c_rank[1024];

template <int UNROLL>
__global__ void __launch_bounds__(256) k_copy(const float4* __restrict__ src, float4* __restrict__ dst,
                                              unsigned long long n_chunks, unsigned chunk_vec,
                                              unsigned* counter, int lo, int hi) {
  __shared__ unsigned s_g;
  int r = c_rank[smid()];
  if (r < lo || r > hi) return;
  for (;;) {
    if (threadIdx.x == 0) s_g = atomicAdd(counter, 1u);
    __syncthreads();
    unsigned g = s_g;
    __syncthreads();
    if (g >= n_chunks) return;
    const float4* s = src + (size_t)g * chunk_vec;
    float4* d = dst + (size_t)g * chunk_vec;
    for (unsigned i = threadIdx.x; i < chunk_vec; i += 256 * UNROLL) {
      float4 v[UNROLL];
#pragma unroll
      for (int u = 0; u < UNROLL; ++u) {
        unsigned j = i + u * 256;
        if (j < chunk_vec) v[u] = __ldcs(s + j);
      }
#pragma unroll
      for (int u = 0; u < UNROLL; ++u) {
        unsigned j = i + u * 256;
        if (j < chunk_vec) __stcs(d + j, v[u]);
      }
    }
  }
}

// spins until *flag changes from its initial value, records globaltimer
__global__ void k_spin(volatile unsigned long long* flag, unsigned long long* host_mirror, unsigned long long init) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  unsigned long long v;
  do {
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(flag));
  } while (v == init);
  host_mirror[0] = v;
  host_mirror[1] = gtimer();
  __threadfence_system();
}

__global__ void k_fma(float* out, int iters) {
  float a = threadIdx.x * 1e-3f, b = 1.0001f, c0 = 0.f, c1 = 0.f, c2 = 0.f, c3 = 0.f, c4 = 0, c5 = 0, c6 = 0, c7 = 0;
  for (int i = 0; i < iters; ++i) {
    c0 = fmaf(a, b, c0); c1 = fmaf(a, b, c1); c2 = fmaf(a, b, c2); c3 = fmaf(a, b, c3);
    c4 = fmaf(a, b, c4); c5 = fmaf(a, b, c5); c6 = fmaf(a, b, c6); c7 = fmaf(a, b, c7);
  }
  if (c0 + c1 + c2 + c3 + c4 + c5 + c6 + c7 == 12345.f) out[0] = 1;
}

int main() {
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0));
  printf("name=%s sms=%d smem_per_sm=%zu smem_optin=%zu regs_per_sm=%d clock_khz=%d l2=%d\n", p.name, p.multiProcessorCount,
         p.sharedMemPerMultiprocessor, p.sharedMemPerBlockOptin, p.regsPerMultiprocessor, p.clockRate, p.l2CacheSize);
  int nsm = p.multiProcessorCount;
  // --- smid calibration
  int nprobe = nsm * 32;
  unsigned* d_ids; CK(cudaMalloc(&d_ids, nprobe * 4));
  k_smid<<<nprobe, 32>>>(d_ids);
  CK(cudaDeviceSynchronize());
  std::vector<unsigned> ids(nprobe); CK(cudaMemcpy(ids.data(), d_ids, nprobe * 4, cudaMemcpyDeviceToHost));
  std::vector<unsigned> u = ids; std::sort(u.begin(), u.end()); u.erase(std::unique(u.begin(), u.end()), u.end());
  printf("unique smids=%zu min=%u max=%u\n", u.size(), u.front(), u.back());
  printf("smids:"); for (auto x : u) printf(" %u", x); printf("\n");
  printf("first 160 block->smid:"); for (int i = 0; i < 160 && i < nprobe; ++i) printf(" %u", ids[i]); printf("\n");
  std::vector<unsigned short> rank(1024, 0xffff);
  for (size_t i = 0; i < u.size(); ++i) rank[u[i]] = (unsigned short)i;
  CK(cudaMemcpyToSymbol(c_rank, rank.data(), sizeof(unsigned short) * 1024));

  // --- FMA peak
  {
    float* o; CK(cudaMalloc(&o, 4));
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    int iters = 100000;
    k_fma<<<nsm * 8, 256>>>(o, 1000);
    cudaEventRecord(e0); k_fma<<<nsm * 8, 256>>>(o, iters); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double fl = 2.0 * 8 * iters * (double)nsm * 8 * 256;
    printf("fp32 fma: %.1f TFLOP/s (%.3f ms)\n", fl / ms / 1e9, ms);
  }

  // --- copy bandwidth vs SMs
  size_t bytes = (size_t)2 << 30;  // 2 GiB per array
  float4 *a, *b; CK(cudaMalloc(&a, bytes)); CK(cudaMalloc(&b, bytes));
  CK(cudaMemset(a, 0, bytes)); CK(cudaMemset(b, 0, bytes));
  unsigned* cnt; CK(cudaMalloc(&cnt, 4));
  unsigned chunk_vec = 4096;  // 64 KiB per task
  unsigned long long n_chunks = bytes / 16 / chunk_vec;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int sms_list[] = {4, 8, 12, 16, 24, 32, 40, 48, 56, 64, 74, 96, 112, 128, 148};
  for (int occ : {4, 8}) {
    for (int s : sms_list) {
      if (s > nsm) continue;
      float best = 1e9;
      for (int rep = 0; rep < 4; ++rep) {
        CK(cudaMemset(cnt, 0, 4));
        cudaEventRecord(e0);
        k_copy<4><<<nsm * occ, 256>>>(a, b, n_chunks, chunk_vec, cnt, 0, s - 1);
        cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
        float ms; cudaEventElapsedTime(&ms, e0, e1); best = std::min(best, ms);
      }
      printf("copy occ=%d sms=%3d  %.1f GB/s\n", occ, s, 2.0 * bytes / best / 1e6);
    }
  }
  // --- control-write latency
  {
    CUdevice dev; cuDeviceGet(&dev, 0);
    unsigned long long* flag; CK(cudaMalloc(&flag, 8)); CK(cudaMemset(flag, 0, 8));
    unsigned long long* hm; CK(cudaHostAlloc(&hm, 16, cudaHostAllocMapped));
    unsigned long long* dhm; CK(cudaHostGetDevicePointer(&dhm, hm, 0));
    cudaStream_t ks, cs; cudaStreamCreateWithFlags(&ks, cudaStreamNonBlocking);
    int lo, hi; cudaDeviceGetStreamPriorityRange(&lo, &hi);
    cudaStreamCreateWithPriority(&cs, cudaStreamNonBlocking, hi);
    std::vector<double> lat;
    for (int rep = 0; rep < 20; ++rep) {
      hm[0] = 0; hm[1] = 0;
      unsigned long long init = rep * 2;
      CK(cudaMemcpy(flag, &init, 8, cudaMemcpyHostToDevice));
      k_spin<<<1, 32, 0, ks>>>(flag, dhm, init);
      auto t0 = std::chrono::steady_clock::now();
      while (std::chrono::steady_clock::now() - t0 < std::chrono::microseconds(2000)) {}
      auto t1 = std::chrono::steady_clock::now();
      CUresult r = cuStreamWriteValue64(cs, (CUdeviceptr)flag, init + 1, 0);
      if (r != CUDA_SUCCESS) { printf("cuStreamWriteValue64 failed %d\n", (int)r); break; }
      while (((volatile unsigned long long*)hm)[0] != init + 1) {}
      auto t2 = std::chrono::steady_clock::now();
      lat.push_back(std::chrono::duration<double, std::micro>(t2 - t1).count());
      CK(cudaStreamSynchronize(ks));
    }
    std::sort(lat.begin(), lat.end());
    printf("ctrl write->observe host roundtrip us: min %.2f p50 %.2f max %.2f\n", lat.front(), lat[lat.size() / 2], lat.back());
  }
  return 0;
}
