// Development probe (not product code): HBM -> shared read bandwidth of
// cp.async.bulk per SM as a function of copy size and copies in flight.  One
// CTA per SM on the first `sms` SMs of the grid (others exit), one thread keeps
// `k` copies of `bytes` in flight through a ring of mbarriers; nobody reads
// the data.  Answers: how many bytes in flight does an SM need, and what is
// its ceiling, for the SpMV chunk ring (csrc/spmv_ws.cu).
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1); } } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return uint32_t(__cvta_generic_to_shared(p)); }

__global__ void bulk_read(const char* src, size_t per_cta, uint32_t bytes, int k, int sms, int streams_per_cta) {
  extern __shared__ __align__(128) char sm[];
  __shared__ uint64_t bar[16];
  if (blockIdx.x >= sms) return;
  if (threadIdx.x != 0) return;
  for (int i = 0; i < k; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[i])));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  const char* base = src + per_cta * blockIdx.x;
  const size_t n = per_cta / bytes;
  uint32_t par = 0;
  for (size_t i = 0; i < n + k; ++i) {
    const int s = int(i % k);
    if (i >= (size_t)k) {   // wait for the copy issued k ago on this slot
      const uint32_t ph = (par >> s) & 1u;
      asm volatile("{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n}" ::"r"(su32(&bar[s])), "r"(ph) : "memory");
      par ^= 1u << s;
    }
    if (i < n) {
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[s])), "r"(bytes) : "memory");
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(su32(sm + size_t(s) * bytes)),
                   "l"(base + i * bytes), "r"(bytes), "r"(su32(&bar[s])) : "memory");
    }
  }
}

// the same ring filled by one warp with cp.async (LDGSTS, 16 B per lane, L1/LSU
// path); each lane's copies of a slot signal the slot's mbarrier (count 32)
__global__ void lsu_read(const char* src, size_t per_cta, uint32_t bytes, int k, int sms) {
  extern __shared__ __align__(128) char sm[];
  __shared__ uint64_t bar[16];
  if (blockIdx.x >= sms || threadIdx.x >= 32) return;
  const uint32_t lane = threadIdx.x;
  if (lane == 0) {
    for (int i = 0; i < k; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 32;" ::"r"(su32(&bar[i])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  const char* base = src + per_cta * blockIdx.x;
  const size_t n = per_cta / bytes;
  uint32_t par = 0;
  for (size_t i = 0; i < n + k; ++i) {
    const int s = int(i % k);
    if (i >= (size_t)k) {
      const uint32_t ph = (par >> s) & 1u;
      asm volatile("{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n}" ::"r"(su32(&bar[s])), "r"(ph) : "memory");
      par ^= 1u << s;
    }
    if (i < n) {
      const char* g = base + i * bytes;
      char* d = sm + size_t(s) * bytes;
      for (uint32_t o = lane * 16; o < bytes; o += 512)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su32(d + o)), "l"(g + o) : "memory");
      asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(su32(&bar[s])) : "memory");
    }
  }
}

int main() {
  const size_t total = size_t(2) << 30;
  char* src; CK(cudaMalloc(&src, total));
  CK(cudaMemset(src, 1, total));
  char* flush; CK(cudaMalloc(&flush, 256 << 20));
  CK(cudaFuncSetAttribute(bulk_read, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  CK(cudaFuncSetAttribute(lsu_read, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int sms : {148, 74, 37}) {
    for (uint32_t bytes : {4096u, 16384u, 32768u}) {
      for (int k : {2, 4, 6, 8, 12}) {
        if (size_t(k) * bytes > 196 * 1024) continue;
        const size_t per_cta = (total / 148) / bytes * bytes;
        float best = 1e9;
        for (int r = 0; r < 4; ++r) {
          CK(cudaMemset(flush, r, 256 << 20));
          cudaEventRecord(e0);
          bulk_read<<<148, 32, k * bytes>>>(src, per_cta, bytes, k, sms, 1);
          cudaEventRecord(e1); CK(cudaEventSynchronize(e1)); CK(cudaGetLastError());
          float ms; cudaEventElapsedTime(&ms, e0, e1); if (r) best = ms < best ? ms : best;
        }
        const double gb = double(per_cta) * sms / 1e9;
        float best2 = 1e9;
        for (int r = 0; r < 4; ++r) {
          CK(cudaMemset(flush, r, 256 << 20));
          cudaEventRecord(e0);
          lsu_read<<<148, 32, k * bytes>>>(src, per_cta, bytes, k, sms);
          cudaEventRecord(e1); CK(cudaEventSynchronize(e1)); CK(cudaGetLastError());
          float ms; cudaEventElapsedTime(&ms, e0, e1); if (r) best2 = ms < best2 ? ms : best2;
        }
        printf("sms %3d  copy %6u B  in flight %2d (%4u KB)  bulk %7.1f GB/s (%6.1f per SM)  cp.async %7.1f GB/s (%6.1f per SM)\n",
               sms, bytes, k, unsigned(k * bytes / 1024), gb / best * 1e3, gb / best * 1e3 / sms, gb / best2 * 1e3,
               gb / best2 * 1e3 / sms);
      }
    }
  }
  return 0;
}
