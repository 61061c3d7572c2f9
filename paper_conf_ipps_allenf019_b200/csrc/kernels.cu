// kernels.cu -- instantiates the worker and standalone kernels for every tenant
// kind and exposes a small host-side dispatch table to the runtime.
#include <cstring>
#include "kernels.h"
#include "slate_device.cuh"
#include "tenants.cuh"
#include "gemm_tc.cuh"
#include "spmv_ws.cuh"

namespace slate {

__global__ void calibrate_kernel(uint32_t* out, uint32_t spin_ns) {
  if (threadIdx.x == 0) out[blockIdx.x] = smid();
  const uint64_t t0 = globaltimer();
  while (globaltimer() - t0 < spin_ns) {
  }
}

namespace {

template <class Tn>
cudaError_t launch_worker_t(const WorkerCommon& w, const void* args, uint32_t grid, cudaStream_t st) {
  WorkerParams<typename Tn::Args> p;
  std::memcpy(&p.args, args, sizeof(typename Tn::Args));
  p.gx = w.gx; p.gy = w.gy; p.gz = w.gz; p.B = w.B; p.iters = w.iters; p.occ = w.occ;
  p.bound_lo = w.bound_lo; p.bound_hi = w.bound_hi; p.n_ranks = w.n_ranks;
  p.standby_timeout_ns = w.standby_timeout_ns;
  p.base_epoch = w.base_epoch;
  p.is_topup = w.is_topup;
  p.gate_first = w.gate_first;
  p.ranklog = w.ranklog;
  p.pdl_early = 0;
  p.ctrl = w.ctrl; p.tc = w.tc; p.mirror = w.mirror; p.cov = w.cov; p.rank_of = w.rank_of;
  void* kargs[] = {&p};
  return launch_kernel(reinterpret_cast<const void*>(&slate_worker<Tn>), dim3(grid), dim3(Tn::kThreads), kargs,
                       Tn::kSmem, st, w.pdl);
}

template <class Tn>
cudaError_t launch_standalone_t(const void* args, dim3 grid, cudaStream_t st) {
  typename Tn::Args a;
  std::memcpy(&a, args, sizeof(a));
  void* kargs[] = {&a};
  return cudaLaunchKernel(reinterpret_cast<const void*>(&standalone<Tn>), grid, dim3(Tn::kThreads), kargs,
                          Tn::kSmemStandalone, st);
}

// Black-Scholes: the few-scenario worker (task-level body) or the
// many-scenario one, per launch; same occupancy (64 registers, 4 CTAs/SM)
cudaError_t launch_worker_bs(const WorkerCommon& w, const void* args, uint32_t grid, cudaStream_t st) {
  const slate_args_bs* a = static_cast<const slate_args_bs*>(args);
  return a->n_scen <= BlackScholesShort::kPipelineMaxScen ? launch_worker_t<BlackScholesShort>(w, args, grid, st)
                                                           : launch_worker_t<BlackScholes>(w, args, grid, st);
}

template <class Tn>
KindOps make_ops(uint32_t default_iters) {
  KindOps o;
  o.worker_fn = reinterpret_cast<const void*>(&slate_worker<Tn>);
  o.standalone_fn = reinterpret_cast<const void*>(&standalone<Tn>);
  o.threads = Tn::kThreads;
  o.smem = Tn::kSmem;
  o.smem_standalone = Tn::kSmemStandalone;
  o.args_size = sizeof(typename Tn::Args);
  o.default_iters = default_iters;
  o.max_auto_iters = Tn::kMaxIters;
  o.tasks_per_worker = Tn::kTasksPerWorker;
  o.launch_worker = &launch_worker_t<Tn>;
  o.launch_standalone = &launch_standalone_t<Tn>;
  o.topup_anytime = true;
  o.pdl_ok = true;
  return o;
}

}  // namespace

const KindOps* kind_ops(uint32_t kind) {
  static KindOps table[SLATE_KIND_MAX_];
  static bool init = false;
  if (!init) {
    table[SLATE_KIND_TRIAD] = make_ops<Triad>(0);
    table[SLATE_KIND_COPY] = make_ops<Copy>(0);
    table[SLATE_KIND_SGEMM_NAIVE] = make_ops<SgemmNaive>(0);
    table[SLATE_KIND_SPMV_CSR] = spmv_ws_ops();
    table[SLATE_KIND_BLACKSCHOLES] = make_ops<BlackScholes>(0);
    table[SLATE_KIND_BLACKSCHOLES].launch_worker = &launch_worker_bs;
    table[SLATE_KIND_STENCIL2D] = make_ops<Stencil2D>(0);
    table[SLATE_KIND_GEMM_BF16] = gemm_tc_ops();
    table[SLATE_KIND_TRANSPOSE] = make_ops<Transpose>(0);
    table[SLATE_KIND_SGEMM_TILED] = make_ops<SgemmTiled>(0);
    table[SLATE_KIND_QRNG] = make_ops<Qrng>(0);
    table[SLATE_KIND_GAUSS_FAN1] = make_ops<GaussFan1>(0);
    table[SLATE_KIND_GAUSS_FAN2] = make_ops<GaussFan2>(0);
    init = true;
  }
  if (kind == 0 || kind >= SLATE_KIND_MAX_) return nullptr;
  return table[kind].worker_fn ? &table[kind] : nullptr;
}

// host <-> device clock offset: the host raises flag[i] (mapped memory) at a
// known host time; the kernel stamps %globaltimer the moment it sees it.
__global__ void clock_probe_kernel(volatile uint32_t* flag, volatile unsigned long long* stamp, int rounds) {
  if (threadIdx.x || blockIdx.x) return;
  for (int i = 0; i < rounds; ++i) {
    flag[2 * i + 1] = 1;                       // ready for round i
    __threadfence_system();
    const unsigned long long t0 = globaltimer();
    while (flag[2 * i] == 0) {
      if (globaltimer() - t0 > 2000000ull) {   // 2 ms: no host on the other side (e.g. a profiler replay)
        stamp[i] = 1ull;
        return;
      }
    }
    stamp[i] = globaltimer();
    __threadfence_system();
  }
}

cudaError_t launch_clock_probe(volatile uint32_t* flag, volatile unsigned long long* stamp, int rounds,
                               cudaStream_t st) {
  clock_probe_kernel<<<1, 32, 0, st>>>(flag, stamp, rounds);
  return cudaGetLastError();
}

cudaError_t launch_calibrate(uint32_t* out, uint32_t blocks, uint32_t spin_ns, cudaStream_t st) {
  calibrate_kernel<<<blocks, 64, 0, st>>>(out, spin_ns);
  return cudaGetLastError();
}

}  // namespace slate
