// Development probe (not product code): CSR SpMV kernel designs on B200,
// timed at several SM counts (SM-restricted persistent workers, atomic task
// queue), to pick the tenant body.  Matrix: 2^20 rows x 16 nnz, banded.
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
#include <algorithm>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1); } } while (0)

__device__ __forceinline__ unsigned smid() { unsigned r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }

struct M { const int* rp; const int* col; const float* val; const float* x; float* y; int n; };

// A: original kernel, 8 lanes/row, one block = 32 rows
__global__ void __launch_bounds__(256) k_orig(M m) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, l = lane & 7;
  const int row = blockIdx.x * 32 + w * 4 + (lane >> 3);
  int lo = 0, hi = 0;
  if (row < m.n) { lo = m.rp[row] + l; hi = m.rp[row + 1]; }
  float acc = 0.f;
  for (int j = lo; j < hi; j += 8) acc = fmaf(__ldcs(m.val + j), __ldg(m.x + __ldcs(m.col + j)), acc);
  acc += __shfl_xor_sync(~0u, acc, 4); acc += __shfl_xor_sync(~0u, acc, 2); acc += __shfl_xor_sync(~0u, acc, 1);
  if (l == 0 && row < m.n) m.y[row] = acc;
}

// B: CTA worker, task of IT blocks, all rows of the task hoisted (U = IT)
template <int IT>
__global__ void __launch_bounds__(256) k_cta(M m, unsigned* ctr, int lo_sm, int hi_sm, int nblk) {
  __shared__ unsigned s_g;
  const int sm = smid();
  if (sm < lo_sm || sm > hi_sm) return;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, l = lane & 7, q = lane >> 3;
  for (;;) {
    if (threadIdx.x == 0) s_g = atomicAdd(ctr, IT);
    __syncthreads();
    const unsigned g = s_g;
    __syncthreads();
    if (g >= (unsigned)nblk) return;
    int lo[IT], hi[IT], c0[IT], c1[IT]; float v0[IT], v1[IT], acc[IT];
#pragma unroll
    for (int u = 0; u < IT; ++u) {
      const int row = (g + u) * 32 + w * 4 + q;
      lo[u] = hi[u] = 0; acc[u] = 0.f;
      if (row < m.n) { lo[u] = m.rp[row] + l; hi[u] = m.rp[row + 1]; }
    }
#pragma unroll
    for (int u = 0; u < IT; ++u) {
      c0[u] = lo[u] < hi[u] ? __ldcs(m.col + lo[u]) : 0; v0[u] = lo[u] < hi[u] ? __ldcs(m.val + lo[u]) : 0.f;
      c1[u] = lo[u] + 8 < hi[u] ? __ldcs(m.col + lo[u] + 8) : 0; v1[u] = lo[u] + 8 < hi[u] ? __ldcs(m.val + lo[u] + 8) : 0.f;
    }
#pragma unroll
    for (int u = 0; u < IT; ++u) {
      acc[u] = fmaf(v0[u], __ldg(m.x + c0[u]), acc[u]);
      acc[u] = fmaf(v1[u], __ldg(m.x + c1[u]), acc[u]);
      float a = acc[u];
      a += __shfl_xor_sync(~0u, a, 4); a += __shfl_xor_sync(~0u, a, 2); a += __shfl_xor_sync(~0u, a, 1);
      const int row = (g + u) * 32 + w * 4 + q;
      if (l == 0 && row < m.n) m.y[row] = a;
    }
  }
}

// C: warp worker: one warp = one whole block (8 sub-steps hoisted), task of IT blocks,
// next task's row pointers prefetched into registers (lookahead)
template <int IT>
__global__ void __launch_bounds__(256) k_warp(M m, unsigned* ctr, int lo_sm, int hi_sm, int nblk) {
  const int sm = smid();
  if (sm < lo_sm || sm > hi_sm) return;
  const int lane = threadIdx.x & 31, l = lane & 7, q = lane >> 3;
  unsigned g = 0;
  if (lane == 0) g = atomicAdd(ctr, IT);
  g = __shfl_sync(~0u, g, 0);
  while (g < (unsigned)nblk) {
    unsigned g2 = 0;
    if (lane == 0) g2 = atomicAdd(ctr, IT);     // lookahead fetch, result used after this task
    for (int u = 0; u < IT; ++u) {
      const unsigned x = g + u;
      if (x >= (unsigned)nblk) break;
      int lo[8], hi[8], c0[8], c1[8]; float v0[8], v1[8], acc[8];
#pragma unroll
      for (int t = 0; t < 8; ++t) {
        const int row = x * 32 + 4 * t + q;
        lo[t] = hi[t] = 0; acc[t] = 0.f;
        if (row < m.n) { lo[t] = m.rp[row] + l; hi[t] = m.rp[row + 1]; }
      }
#pragma unroll
      for (int t = 0; t < 8; ++t) {
        c0[t] = lo[t] < hi[t] ? __ldcs(m.col + lo[t]) : 0; v0[t] = lo[t] < hi[t] ? __ldcs(m.val + lo[t]) : 0.f;
        c1[t] = lo[t] + 8 < hi[t] ? __ldcs(m.col + lo[t] + 8) : 0; v1[t] = lo[t] + 8 < hi[t] ? __ldcs(m.val + lo[t] + 8) : 0.f;
      }
#pragma unroll
      for (int t = 0; t < 8; ++t) {
        acc[t] = fmaf(v0[t], __ldg(m.x + c0[t]), acc[t]);
        acc[t] = fmaf(v1[t], __ldg(m.x + c1[t]), acc[t]);
        float a = acc[t];
        a += __shfl_xor_sync(~0u, a, 4); a += __shfl_xor_sync(~0u, a, 2); a += __shfl_xor_sync(~0u, a, 1);
        const int row = x * 32 + 4 * t + q;
        if (l == 0 && row < m.n) m.y[row] = a;
      }
    }
    g = __shfl_sync(~0u, g2, 0);
  }
}

int main() {
  const int n = 1 << 20, nnzr = 16, band = 4096;
  std::mt19937 rng(1);
  std::vector<int> rp(n + 1), col((size_t)n * nnzr);
  std::vector<float> val((size_t)n * nnzr), x(n);
  for (int i = 0; i <= n; ++i) rp[i] = i * nnzr;
  for (int i = 0; i < n; ++i) {
    int lo = std::max(0, i - band), hi = std::min(n - 1, i + band);
    std::vector<int> c(nnzr);
    for (int k = 0; k < nnzr; ++k) c[k] = lo + (int)(rng() % (hi - lo + 1));
    std::sort(c.begin(), c.end());
    for (int k = 0; k < nnzr; ++k) { col[(size_t)i * nnzr + k] = c[k]; val[(size_t)i * nnzr + k] = 1.f; }
    x[i] = 1.f;
  }
  M m; m.n = n;
  int *drp, *dcol; float *dval, *dx, *dy; unsigned* ctr;
  CK(cudaMalloc(&drp, (n + 1) * 4)); CK(cudaMalloc(&dcol, col.size() * 4)); CK(cudaMalloc(&dval, val.size() * 4));
  CK(cudaMalloc(&dx, n * 4)); CK(cudaMalloc(&dy, n * 4)); CK(cudaMalloc(&ctr, 4));
  CK(cudaMemcpy(drp, rp.data(), (n + 1) * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dcol, col.data(), col.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dval, val.data(), val.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dx, x.data(), n * 4, cudaMemcpyHostToDevice));
  m.rp = drp; m.col = dcol; m.val = dval; m.x = dx; m.y = dy;
  const double bytes = 8.0 * n * nnzr + 12.0 * n;
  const int nblk = n / 32;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  float* flush; CK(cudaMalloc(&flush, 256 << 20));
  auto timeit = [&](auto launch) {
    float best = 1e9;
    for (int r = 0; r < 6; ++r) {
      CK(cudaMemset(flush, r, 256 << 20));
      CK(cudaMemset(ctr, 0, 4));
      cudaEventRecord(e0); launch(); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (r) best = std::min(best, ms);
    }
    return best;
  };
  float t = timeit([&] { k_orig<<<nblk, 256>>>(m); });
  printf("orig               148: %.4f ms %.0f GB/s\n", t, bytes / t / 1e6);
  int sms_list[] = {148, 111, 74, 49, 37};
  for (int s : sms_list) {
    int occ;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_cta<4>, 256, 0);
    t = timeit([&] { k_cta<4><<<148 * occ, 256>>>(m, ctr, 0, s - 1, nblk); });
    printf("cta U=4  occ=%d     %3d: %.4f ms %.0f GB/s\n", occ, s, t, bytes / t / 1e6);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_cta<8>, 256, 0);
    t = timeit([&] { k_cta<8><<<148 * occ, 256>>>(m, ctr, 0, s - 1, nblk); });
    printf("cta U=8  occ=%d     %3d: %.4f ms %.0f GB/s\n", occ, s, t, bytes / t / 1e6);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_warp<1>, 256, 0);
    t = timeit([&] { k_warp<1><<<148 * occ, 256>>>(m, ctr, 0, s - 1, nblk); });
    printf("warp IT=1 occ=%d    %3d: %.4f ms %.0f GB/s\n", occ, s, t, bytes / t / 1e6);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_warp<2>, 256, 0);
    t = timeit([&] { k_warp<2><<<148 * occ, 256>>>(m, ctr, 0, s - 1, nblk); });
    printf("warp IT=2 occ=%d    %3d: %.4f ms %.0f GB/s\n", occ, s, t, bytes / t / 1e6);
  }
  return 0;
}
