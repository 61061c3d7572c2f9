// cluster_smid.cu -- which %smid pairs do the two CTAs of a 2-CTA cluster land on?
#include <cstdio>
#include <cuda_runtime.h>
__global__ void probe(unsigned* out) {
  unsigned smid, rank, cid;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(cid));
  if (threadIdx.x == 0) out[cid * 2 + rank] = smid;
  // hold the SM so every cluster gets its own pair
  unsigned long long t0, t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  do { asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); } while (t - t0 < 2000000ull);
}
int main() {
  unsigned* d; cudaMalloc(&d, 4096);
  cudaMemset(d, 0xff, 4096);
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = 2; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
  cfg.gridDim = dim3(148); cfg.blockDim = dim3(32); cfg.dynamicSmemBytes = 200 * 1024;
  cfg.attrs = at; cfg.numAttrs = 1;
  cudaLaunchKernelEx(&cfg, probe, d);
  cudaError_t e = cudaDeviceSynchronize();
  unsigned h[148];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  printf("err %s\n", cudaGetErrorString(e));
  int adjacent = 0, aligned = 0;
  for (int c = 0; c < 74; ++c) {
    unsigned a = h[2 * c], b = h[2 * c + 1];
    if ((a ^ 1u) == b) ++adjacent;
    if (a / 2 == b / 2) ++aligned;
    printf("%u:%u ", a, b);
  }
  printf("\nclusters %d, pairs {2t,2t+1}: %d\n", 74, aligned);
  return 0;
}
