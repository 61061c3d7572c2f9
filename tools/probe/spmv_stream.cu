// Development probe (not product code): the warp-specialised SpMV worker
// (csrc/spmv_ws.cu) against the register body it replaces, as the original
// kernel and as slate workers bound to s SMs (the library's own sources), L2
// flushed before every run.  Also checks that all produce bit-identical y.
// Matrix: C2's, 2^20 x nnzr banded +-4096, random values.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include \
//        tools/probe/spmv_stream.cu -o tools/probe/spmv_stream
#include <cuda_runtime.h>
#include <cstdio>
#include <cstring>
#include <vector>
#include <string>
#include <random>
#include <algorithm>
#include "../../paper_conf_ipps_allenf019_b200/csrc/slate_device.cuh"
#include "../../paper_conf_ipps_allenf019_b200/csrc/tenants.cuh"
#include "../../paper_conf_ipps_allenf019_b200/csrc/spmv_ws.cu"

using namespace slate;
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1); } } while (0)

#ifdef SLATE_SPMV_PROFILE
static void* spmv_prof_ptr() { void* p; CK(cudaGetSymbolAddress(&p, spmv::spmv_prof)); return p; }
#endif
int main(int argc, char** argv) {
  const int n = 1 << 20, band = 4096;
  const int nnzr = argc > 1 ? atoi(argv[1]) : 16;
  std::mt19937 rng(1);
  std::uniform_real_distribution<float> U(-1.f, 1.f);
  std::vector<int> rp(n + 4), col((size_t)n * nnzr + 4);
  std::vector<float> val((size_t)n * nnzr + 4), x(n);
  for (int i = 0; i <= n; ++i) rp[i] = i * nnzr;
  for (int i = 0; i < n; ++i) {
    int lo = std::max(0, i - band), hi = std::min(n - 1, i + band);
    std::vector<int> c(nnzr);
    for (int k = 0; k < nnzr; ++k) c[k] = lo + (int)(rng() % (hi - lo + 1));
    std::sort(c.begin(), c.end());
    for (int k = 0; k < nnzr; ++k) { col[(size_t)i * nnzr + k] = c[k]; val[(size_t)i * nnzr + k] = U(rng); }
    x[i] = U(rng);
  }
  int *drp, *dcol; float *dval, *dx, *dy;
  CK(cudaMalloc(&drp, rp.size() * 4)); CK(cudaMalloc(&dcol, col.size() * 4)); CK(cudaMalloc(&dval, val.size() * 4));
  CK(cudaMalloc(&dx, n * 4)); CK(cudaMalloc(&dy, n * 4));
  CK(cudaMemcpy(drp, rp.data(), rp.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dcol, col.data(), col.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dval, val.data(), val.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dx, x.data(), n * 4, cudaMemcpyHostToDevice));
  slate_args_spmv a{(uint64_t)drp, (uint64_t)dcol, (uint64_t)dval, (uint64_t)dx, (uint64_t)dy, (uint32_t)n, (uint32_t)n};
  const int nblk = n / 32;
  TaskCtl* tc; CK(cudaMalloc(&tc, sizeof(TaskCtl)));
  uint64_t* ctrl; CK(cudaMalloc(&ctrl, 8));
  uint16_t* lut; CK(cudaMalloc(&lut, 2048));
  // identity-ish LUT: rank = smid (ranks >= 148 never in range)
  std::vector<uint16_t> hl(1024); for (int i = 0; i < 1024; ++i) hl[i] = (uint16_t)std::min(i, 1023);
  CK(cudaMemcpy(lut, hl.data(), 2048, cudaMemcpyHostToDevice));
  float* flush; CK(cudaMalloc(&flush, 256 << 20));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const double bytes = 8.0 * n * nnzr + 12.0 * n;
  std::vector<float> ref(n), out(n);
  bool have_ref = false;
  auto check = [&](const char* name) {
    CK(cudaMemcpy(out.data(), dy, n * 4, cudaMemcpyDeviceToHost));
    if (!have_ref) { ref = out; have_ref = true; return; }
    if (memcmp(ref.data(), out.data(), n * 4)) {
      int bad = 0; for (int i = 0; i < n; ++i) bad += ref[i] != out[i];
      printf("  !! %s differs from the first variant in %d rows\n", name, bad);
    }
  };
  auto timeit = [&](const char* name, int sms, auto launch) {
    float best = 1e9, sum = 0; int cnt = 0;
    for (int r = 0; r < 8; ++r) {
      CK(cudaMemset(dy, 0, n * 4));
      CK(cudaMemset(flush, r, 256 << 20));
      CK(cudaMemset(tc, 0, sizeof(TaskCtl)));
      const uint64_t cv = pack_ctrl(1, 0, sms - 1);
      CK(cudaMemcpy(ctrl, &cv, 8, cudaMemcpyHostToDevice));
      cudaEventRecord(e0); launch(); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
      CK(cudaGetLastError());
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (r) { best = std::min(best, ms); sum += ms; ++cnt; }
    }
    check(name);
    printf("%-40s sms %3d  best %.4f ms  mean %.4f ms  %5.0f GB/s\n", name, sms, best, sum / cnt, bytes / best / 1e6);
  };
  const KindOps ws = spmv_ws_ops();
  CK(cudaFuncSetAttribute(ws.worker_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, ws.smem));
  timeit("original (SpmvSeg)", 148, [&] { standalone<SpmvSeg><<<nblk, SpmvSeg::kThreads>>>(a); });
  auto worker = [&](const char* name, auto kern, int threads, int smem, uint32_t iters, int sms) {
    int o; CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, kern, threads, smem));
    WorkerParams<slate_args_spmv> p{};
    p.args = a; p.gx = nblk; p.gy = 1; p.gz = 1; p.B = nblk; p.iters = iters; p.occ = o; p.bound_lo = 0;
    p.bound_hi = 1023; p.n_ranks = 148; p.standby_timeout_ns = 200000; p.ctrl = ctrl; p.tc = tc; p.mirror = nullptr;
    p.cov = nullptr; p.rank_of = lut;
    char buf[96]; snprintf(buf, sizeof buf, "%s it %u occ %d", name, iters, o);
    timeit(buf, sms, [&] { kern<<<148 * o, threads, smem>>>(p); });
  };
  auto ws_worker = [&](uint32_t iters, int sms) {
    WorkerCommon w{};
    w.gx = nblk; w.gy = 1; w.gz = 1; w.B = nblk; w.iters = iters; w.occ = 1; w.bound_lo = 0; w.bound_hi = 1023;
    w.n_ranks = 148; w.standby_timeout_ns = 200000; w.ctrl = ctrl; w.tc = tc; w.mirror = nullptr; w.cov = nullptr;
    w.rank_of = lut;
    char buf[96]; snprintf(buf, sizeof buf, "worker, warp-specialised it %u", iters);
    timeit(buf, sms, [&] { CK(ws.launch_worker(w, &a, 148, 0)); });
  };
  const uint32_t IT = getenv("SPMV_ITERS") ? atoi(getenv("SPMV_ITERS")) : 32;
  for (int sms : {148, 111, 74, 56, 37}) {
    ws_worker(IT, sms);
    if (sms == 148) { ws_worker(16, sms); ws_worker(8, sms); ws_worker(1, sms); }
  }
#ifdef SLATE_SPMV_TRACE
  ws_worker(IT, 74);
  static unsigned long long t[4][3][64][4];
  CK(cudaMemcpyFromSymbol(t, spmv::spmv_trace, sizeof(t)));
  unsigned long long t0 = ~0ull;
  for (int c = 0; c < 4; ++c) for (int r = 0; r < 3; ++r) for (int i = 0; i < 64; ++i) if (t[c][r][i][0] && t[c][r][i][0] < t0) t0 = t[c][r][i][0];
  const char* names[] = {"task: wait empty", "task: empty ok", "task: fetched g", "task: window issued"};
  for (int c = 0; c < 2; ++c) {
    std::vector<std::pair<unsigned long long, std::string>> ev;
    for (int r = 0; r < 3; ++r) for (int i = 0; i < 64; ++i) {
      auto* e = t[c][r][i]; if (!e[0]) continue;
      char buf[128]; int k = (int)e[1];
      const char* nm = k < 4 ? names[k] : k == 10 ? "chunk: task rp ok" : k == 11 ? "chunk: slot free -> issue" : k == 20 ? "comp: slot full" : k == 21 ? "comp: start" : "comp: end";
      snprintf(buf, sizeof buf, "%-28s %llu %llu", nm, e[2], e[3]);
      ev.push_back({e[0], buf});
    }
    std::sort(ev.begin(), ev.end());
    for (auto& x : ev) printf("cta %d %9.3f us  %s\n", c, (x.first - t0) / 1e3, x.second.c_str());
  }
#endif
#ifdef SLATE_SPMV_PROFILE
  for (int sms : {148, 74, 37}) {
  static long long pr[148][32][5];
  CK(cudaMemset(spmv_prof_ptr(), 0, sizeof(pr)));
  ws_worker(IT, sms);
  CK(cudaMemcpyFromSymbol(pr, spmv::spmv_prof, sizeof(pr)));
  printf("-- %d SMs\n", sms);
  for (int c = 0; c < 148; ++c) for (int w : {0, 15}) {
    if (!pr[c][w][4] || (c % 16 != 0)) continue;
    long long* o = pr[c][w];
    printf("cta %3d warp %2d: total %7lld clk  wait-full %6.1f%%  first-chunk %5.1f%%  compute %5.1f%%  chunks %lld  (%.0f clk/chunk compute)\n",
           c, w, o[0], 100.0 * o[1] / o[0], 100.0 * o[2] / o[0], 100.0 * o[3] / o[0], o[4], o[4] ? double(o[3]) / o[4] : 0.0);
  }
  }
#endif
  return 0;
}
