// Development probe: where does the slate worker's per-launch/per-task overhead
// come from?  Runs the real slate_worker<SpmvCsrReg> (library headers) beside the
// original kernel and stripped-down persistent variants, L2 flushed each run.
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#include <random>
#include <algorithm>
#include "../../paper_conf_ipps_allenf019_b200/csrc/slate_device.cuh"
#include "../../paper_conf_ipps_allenf019_b200/csrc/tenants.cuh"

using namespace slate;
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1); } } while (0)

// V0: minimal persistent CTA worker, same body (SpmvCsr::cta_task), one atomic per task
__global__ void __launch_bounds__(256) v0(slate_args_spmv a, unsigned* ctr, int nblk, int it) {
  __shared__ unsigned s_g;
  for (;;) {
    if (threadIdx.x == 0) s_g = atomicAdd(ctr, it);
    __syncthreads();
    const unsigned g = s_g;
    __syncthreads();
    if (g >= (unsigned)nblk) return;
    SpmvCsrReg::cta_task(a, g, min((unsigned)it, nblk - g), nullptr);
  }
}
// V1: V0 + the done counter (64-bit atomic with return) per task
__global__ void __launch_bounds__(256) v1(slate_args_spmv a, unsigned* ctr, unsigned long long* done, int nblk, int it) {
  __shared__ unsigned s_g;
  for (;;) {
    if (threadIdx.x == 0) s_g = atomicAdd(ctr, it);
    __syncthreads();
    const unsigned g = s_g;
    __syncthreads();
    if (g >= (unsigned)nblk) return;
    const unsigned n = min((unsigned)it, nblk - g);
    SpmvCsrReg::cta_task(a, g, n, nullptr);
    __syncthreads();
    if (threadIdx.x == 0) { unsigned long long o = atomicAdd(done, (1ull << 32) | n); if ((unsigned)o + n == (unsigned)nblk) done[1] = 1; }
  }
}

int main() {
  const int n = 1 << 20, nnzr = 16, band = 4096;
  std::mt19937 rng(1);
  std::vector<int> rp(n + 1), col((size_t)n * nnzr);
  std::vector<float> val((size_t)n * nnzr, 1.f), x(n, 1.f);
  for (int i = 0; i <= n; ++i) rp[i] = i * nnzr;
  for (int i = 0; i < n; ++i) {
    int lo = std::max(0, i - band), hi = std::min(n - 1, i + band);
    std::vector<int> c(nnzr);
    for (int k = 0; k < nnzr; ++k) c[k] = lo + (int)(rng() % (hi - lo + 1));
    std::sort(c.begin(), c.end());
    for (int k = 0; k < nnzr; ++k) col[(size_t)i * nnzr + k] = c[k];
  }
  int *drp, *dcol; float *dval, *dx, *dy;
  CK(cudaMalloc(&drp, (n + 1) * 4)); CK(cudaMalloc(&dcol, col.size() * 4)); CK(cudaMalloc(&dval, val.size() * 4));
  CK(cudaMalloc(&dx, n * 4)); CK(cudaMalloc(&dy, n * 4));
  CK(cudaMemcpy(drp, rp.data(), (n + 1) * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dcol, col.data(), col.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dval, val.data(), val.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dx, x.data(), n * 4, cudaMemcpyHostToDevice));
  slate_args_spmv a{(uint64_t)drp, (uint64_t)dcol, (uint64_t)dval, (uint64_t)dx, (uint64_t)dy, (uint32_t)n, (uint32_t)n};
  const int nblk = n / 32;
  unsigned* ctr; CK(cudaMalloc(&ctr, 4));
  unsigned long long* done; CK(cudaMalloc(&done, 16));
  TaskCtl* tc; CK(cudaMalloc(&tc, sizeof(TaskCtl)));
  uint64_t* ctrl; CK(cudaMalloc(&ctrl, 8));
  const uint64_t cv = pack_ctrl(1, 0, 147);
  CK(cudaMemcpy(ctrl, &cv, 8, cudaMemcpyHostToDevice));
  uint16_t* lut; CK(cudaMalloc(&lut, 2048));
  std::vector<uint16_t> hl(1024); for (int i = 0; i < 1024; ++i) hl[i] = (uint16_t)std::min(i, 147);
  CK(cudaMemcpy(lut, hl.data(), 2048, cudaMemcpyHostToDevice));
  float* flush; CK(cudaMalloc(&flush, 256 << 20));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const double bytes = 8.0 * n * nnzr + 12.0 * n;
  auto timeit = [&](const char* name, auto launch) {
    float best = 1e9, sum = 0; int cnt = 0;
    for (int r = 0; r < 8; ++r) {
      CK(cudaMemset(flush, r, 256 << 20));
      CK(cudaMemset(ctr, 0, 4)); CK(cudaMemset(done, 0, 16)); CK(cudaMemset(tc, 0, sizeof(TaskCtl)));
      cudaEventRecord(e0); launch(); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (r) { best = std::min(best, ms); sum += ms; ++cnt; }
    }
    printf("%-44s best %.4f ms  mean %.4f ms  %.0f GB/s\n", name, best, sum / cnt, bytes / best / 1e6);
  };
  timeit("original kernel (standalone<SpmvCsrReg>)", [&] { standalone<SpmvCsrReg><<<nblk, 256>>>(a); });
  for (int it : {4}) {
    int occ; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, v0, 256, 0);
    printf("v0 occ %d\n", occ);
    timeit("v0 persistent, 1 atomic/task", [&] { v0<<<148 * occ, 256>>>(a, ctr, nblk, it); });
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, v1, 256, 0);
    timeit("v1 + done atomic/task", [&] { v1<<<148 * occ, 256>>>(a, ctr, done, nblk, it); });
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, slate_worker<SpmvCsrReg>, 256, 0);
    printf("worker occ %d\n", occ);
    WorkerParams<slate_args_spmv> p{};
    p.args = a; p.gx = nblk; p.gy = 1; p.gz = 1; p.B = nblk; p.iters = it; p.occ = occ; p.bound_lo = 0; p.bound_hi = 147;
    p.n_ranks = 148; p.standby_timeout_ns = 200000; p.ctrl = ctrl; p.tc = tc; p.mirror = nullptr; p.cov = nullptr; p.rank_of = lut;
    timeit("slate_worker<SpmvCsrReg> (the real one)", [&] { slate_worker<SpmvCsrReg><<<148 * occ, 256>>>(p); });
    auto variant = [&](const char* name, auto kern, int it2) {
      int o; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, kern, 256, 0);
      WorkerParams<slate_args_spmv> q = p; q.occ = o; q.iters = it2;
      char buf[96]; snprintf(buf, sizeof buf, "%s occ %d", name, o);
      timeit(buf, [&] { kern<<<148 * o, 256>>>(q); });
    };
    variant("U8 mb4 (SpmvCsr now)", slate_worker<SpmvCsrT<8, 4>>, 8);
    variant("U4 mb6", slate_worker<SpmvCsrT<4, 6>>, 4);
    variant("U3 mb8", slate_worker<SpmvCsrT<3, 8>>, 3);
  }
  return 0;
}
