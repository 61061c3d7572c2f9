// Development probe (not product code): WRITE and COPY bandwidth per SM on the
// first k SMs (%smid < k).  Question (round 2, C3): the copy tenant moves ~100
// GB/s of copy traffic per SM whatever its stage ring (3-6 CTAs/SM), while one
// SM reads 170+ GB/s by bulk copies (read_bw.cu) -- is the limit the SM's write
// path?  Variants: STG.128 streaming stores; cp.async.bulk shared->global
// stores from 1-4 issuing warps; a register copy (LDG.128 + STG.128).
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1); } } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return uint32_t(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ unsigned smid() { unsigned r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }

constexpr uint32_t kPiece = 65536;

template <int UNR>
__global__ void stg_write(float4* __restrict__ dst, uint32_t n_pieces, uint32_t* ctr, int k) {
  __shared__ uint32_t s_p;
  if ((int)smid() >= k) return;
  const uint32_t per = kPiece / 16;
  const float4 v = make_float4(1.f, 2.f, 3.f, 4.f);
  for (;;) {
    if (threadIdx.x == 0) s_p = atomicAdd(ctr, 1u);
    __syncthreads();
    const uint32_t p = s_p;
    __syncthreads();
    if (p >= n_pieces) break;
    float4* b = dst + size_t(p) * per;
#pragma unroll UNR
    for (uint32_t i = threadIdx.x; i < per; i += blockDim.x) __stcs(b + i, v);
  }
}

template <int UNR>
__global__ void reg_copy(const float4* __restrict__ src, float4* __restrict__ dst, uint32_t n_pieces, uint32_t* ctr, int k) {
  __shared__ uint32_t s_p;
  if ((int)smid() >= k) return;
  const uint32_t per = kPiece / 16;
  for (;;) {
    if (threadIdx.x == 0) s_p = atomicAdd(ctr, 1u);
    __syncthreads();
    const uint32_t p = s_p;
    __syncthreads();
    if (p >= n_pieces) break;
    const float4* s = src + size_t(p) * per;
    float4* d = dst + size_t(p) * per;
    for (uint32_t i = threadIdx.x; i < per; i += blockDim.x * UNR) {
      float4 v[UNR];
#pragma unroll
      for (int u = 0; u < UNR; ++u) v[u] = __ldcs(s + i + u * blockDim.x);
#pragma unroll
      for (int u = 0; u < UNR; ++u) __stcs(d + i + u * blockDim.x, v[u]);
    }
  }
}

// `issuers` warps, lane 0 of each keeps up to `depth` bulk stores of `bytes`
// from its own shared buffer in flight (the data is whatever is there)
__global__ void bulk_write(char* dst, uint32_t n_pieces, uint32_t* ctr, int k, uint32_t bytes, int depth) {
  extern __shared__ __align__(128) char sm[];
  if ((int)smid() >= k) return;
  if ((threadIdx.x & 31) != 0) return;
  const char* buf = sm + size_t(threadIdx.x >> 5) * bytes;
  const uint32_t cpp = kPiece / bytes;
  for (;;) {
    const uint32_t p = atomicAdd(ctr, 1u);
    if (p >= n_pieces) break;
    for (uint32_t sub = 0; sub < cpp; ++sub) {
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + size_t(p) * kPiece + size_t(sub) * bytes),
                   "r"(su32(buf)), "r"(bytes) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      if (depth == 2) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      else if (depth == 4) asm volatile("cp.async.bulk.wait_group.read 3;" ::: "memory");
      else asm volatile("cp.async.bulk.wait_group.read 7;" ::: "memory");
    }
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

// reads and writes on the same SMs at once: odd CTAs stream-read (LDG.128,
// summed), even CTAs stream-write (STG.128); each half has its own counter over
// its own buffer.  Is ~100 GB/s of copy traffic per SM (copy tenant) the sum of
// the two paths, or a limit of mixed traffic?
__global__ void mixed(const float4* __restrict__ src, float4* __restrict__ dst, uint32_t n_pieces, uint32_t* ctr, int k,
                      float* sink) {
  __shared__ uint32_t s_p;
  if ((int)smid() >= k) return;
  const bool rd = blockIdx.x & 1;
  uint32_t* c = ctr + (rd ? 1 : 0);
  const uint32_t per = kPiece / 16;
  float acc = 0.f;
  const float4 v = make_float4(1.f, 2.f, 3.f, 4.f);
  for (;;) {
    if (threadIdx.x == 0) s_p = atomicAdd(c, 1u);
    __syncthreads();
    const uint32_t p = s_p;
    __syncthreads();
    if (p >= n_pieces) break;
    if (rd) {
      const float4* b = src + size_t(p) * per;
      for (uint32_t i = threadIdx.x; i < per; i += blockDim.x * 4) {
        float4 x[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) x[u] = __ldcs(b + i + u * blockDim.x);
#pragma unroll
        for (int u = 0; u < 4; ++u) acc += x[u].x + x[u].y + x[u].z + x[u].w;
      }
    } else {
      float4* b = dst + size_t(p) * per;
      for (uint32_t i = threadIdx.x; i < per; i += blockDim.x) __stcs(b + i, v);
    }
  }
  if (acc == 1234.5f) sink[0] = acc;
}

int main() {
  const size_t total = size_t(2) << 30;
  char *src, *dst; CK(cudaMalloc(&src, total)); CK(cudaMalloc(&dst, total)); CK(cudaMemset(src, 1, total));
  char* flush; CK(cudaMalloc(&flush, 256u << 20));
  uint32_t* ctr; CK(cudaMalloc(&ctr, 4));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const uint32_t n_pieces = uint32_t(total / kPiece);
  int nsm = 0; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  CK(cudaFuncSetAttribute(bulk_write, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  auto timeit = [&](auto launch, int sms, const char* what, double traffic_per_byte) {
    float best = 1e9f;
    for (int r = 0; r < 3; ++r) {
      CK(cudaMemset(flush, r, 256u << 20));
      CK(cudaMemset(ctr, 0, 4));
      cudaEventRecord(e0); launch(); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
      CK(cudaGetLastError());
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
    }
    const double gbs = traffic_per_byte * total / (best * 1e-3) / 1e9;
    printf("sms %3d  %-44s %8.1f GB/s  %6.1f GB/s per SM (traffic)\n", sms, what, gbs, gbs / sms);
  };
  char name[128];
  float* sink; CK(cudaMalloc(&sink, 4));
  uint32_t* ctr2; CK(cudaMalloc(&ctr2, 8));
  for (int sms : {74, 37}) {
    // mixed: each half moves `total` bytes; traffic = 2 x total over the time both took
    for (int cps : {2, 4}) {
      snprintf(name, sizeof name, "mixed read+write %d CTA/SM x 512 thr", cps);
      timeit([&] {
        CK(cudaMemset(ctr2, 0, 8));
        mixed<<<nsm * cps, 512>>>((const float4*)src, (float4*)dst, n_pieces, ctr2, sms, sink);
      }, sms, name, 2.0);
    }
    for (int cps : {1, 2, 4}) {
      snprintf(name, sizeof name, "stg.128 %d CTA/SM x 512 thr", cps);
      timeit([&] { stg_write<4><<<nsm * cps, 512>>>((float4*)dst, n_pieces, ctr, sms); }, sms, name, 1.0);
    }
    for (int iss : {1, 2, 4}) for (uint32_t bytes : {16384u, 32768u}) for (int d : {2, 4, 8}) {
      if (size_t(bytes) * iss > 200 * 1024) continue;
      snprintf(name, sizeof name, "bulk s2g 1 CTA, %d issuers, %2u KB, depth %d", iss, bytes / 1024, d);
      timeit([&] { bulk_write<<<nsm, 32 * iss, size_t(bytes) * iss>>>(dst, n_pieces, ctr, sms, bytes, d); }, sms, name, 1.0);
    }
    for (int cps : {1, 2, 4}) {
      snprintf(name, sizeof name, "reg copy U4 %d CTA/SM x 512 thr", cps);
      timeit([&] { reg_copy<4><<<nsm * cps, 512>>>((const float4*)src, (float4*)dst, n_pieces, ctr, sms); }, sms, name, 2.0);
    }
  }
  return 0;
}
