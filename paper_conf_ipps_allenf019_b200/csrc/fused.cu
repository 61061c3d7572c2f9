// fused.cu -- NEXT-1: instantiations of the fused co-run worker (fused.cuh)
// for the pairs of generic-worker kinds that share a CTA shape (256 threads,
// no per-CTA state), and the host-side launcher.
#include <cstring>
#include "kernels.h"
#include "fused.cuh"
#include "tenants.cuh"

namespace slate {
namespace {

template <class Tn>
void fill(WorkerParams<typename Tn::Args>& p, const WorkerCommon& w, const void* args) {
  std::memcpy(&p.args, args, sizeof(typename Tn::Args));
  p.gx = w.gx; p.gy = w.gy; p.gz = w.gz; p.B = w.B; p.iters = w.iters; p.occ = w.occ;
  p.bound_lo = w.bound_lo; p.bound_hi = w.bound_hi; p.n_ranks = w.n_ranks;
  p.standby_timeout_ns = w.standby_timeout_ns;
  p.base_epoch = w.base_epoch;
  p.is_topup = 0;
  p.gate_first = 0;
  p.ranklog = w.ranklog;
  p.pdl_early = 0;
  p.ctrl = w.ctrl; p.tc = w.tc; p.mirror = w.mirror; p.cov = w.cov; p.rank_of = w.rank_of;
}

template <class TA, class TB>
struct Pair {
  static constexpr int kSmem = TA::kSmem > TB::kSmem ? TA::kSmem : TB::kSmem;
  static cudaError_t launch(const WorkerCommon& wa, const void* aa, const WorkerCommon& wb, const void* ab,
                            uint32_t grow, uint32_t grid, cudaStream_t st) {
    FusedParams<TA, TB> p;
    fill<TA>(p.a, wa, aa);
    fill<TB>(p.b, wb, ab);
    p.grow_on_drain = grow;
    p.speculative = 0;
    void* kargs[] = {&p};
    return cudaLaunchKernel(reinterpret_cast<const void*>(&slate_fused<TA, TB>), dim3(grid), dim3(TA::kThreads), kargs,
                            kSmem, st);
  }
  static const void* fn() { return reinterpret_cast<const void*>(&slate_fused<TA, TB>); }
};

struct Entry {
  const void* fn = nullptr;
  int threads = 0, smem = 0;
  cudaError_t (*launch)(const WorkerCommon&, const void*, const WorkerCommon&, const void*, uint32_t, uint32_t,
                        cudaStream_t) = nullptr;
};

template <class TA, class TB>
Entry entry() {
  Entry e;
  e.fn = Pair<TA, TB>::fn();
  e.threads = TA::kThreads;
  e.smem = Pair<TA, TB>::kSmem;
  e.launch = &Pair<TA, TB>::launch;
  return e;
}

// the kinds a fused pair may combine, and their tenant types
template <int K> struct KindT;
template <> struct KindT<SLATE_KIND_TRIAD> { using T = Triad; };
template <> struct KindT<SLATE_KIND_SGEMM_NAIVE> { using T = SgemmNaive; };
template <> struct KindT<SLATE_KIND_SGEMM_TILED> { using T = SgemmTiled; };
template <> struct KindT<SLATE_KIND_BLACKSCHOLES> { using T = BlackScholes; };
template <> struct KindT<SLATE_KIND_STENCIL2D> { using T = Stencil2D; };
template <> struct KindT<SLATE_KIND_TRANSPOSE> { using T = Transpose; };

const Entry* table(uint32_t a, uint32_t b) {
  static Entry t[SLATE_KIND_MAX_][SLATE_KIND_MAX_];
  static bool init = false;
  if (!init) {
#define SLATE_FUSE(A, B) t[A][B] = entry<KindT<A>::T, KindT<B>::T>();
#define SLATE_FUSE_ROW(A)                                                                            \
  SLATE_FUSE(A, SLATE_KIND_TRIAD) SLATE_FUSE(A, SLATE_KIND_SGEMM_NAIVE) SLATE_FUSE(A, SLATE_KIND_SGEMM_TILED) \
  SLATE_FUSE(A, SLATE_KIND_BLACKSCHOLES) SLATE_FUSE(A, SLATE_KIND_STENCIL2D) SLATE_FUSE(A, SLATE_KIND_TRANSPOSE)
    SLATE_FUSE_ROW(SLATE_KIND_TRIAD)
    SLATE_FUSE_ROW(SLATE_KIND_SGEMM_NAIVE)
    SLATE_FUSE_ROW(SLATE_KIND_SGEMM_TILED)
    SLATE_FUSE_ROW(SLATE_KIND_BLACKSCHOLES)
    SLATE_FUSE_ROW(SLATE_KIND_STENCIL2D)
    SLATE_FUSE_ROW(SLATE_KIND_TRANSPOSE)
#undef SLATE_FUSE_ROW
#undef SLATE_FUSE
    init = true;
  }
  if (a >= SLATE_KIND_MAX_ || b >= SLATE_KIND_MAX_) return nullptr;
  return t[a][b].fn ? &t[a][b] : nullptr;
}

}  // namespace

bool fused_supported(uint32_t kind_a, uint32_t kind_b) { return table(kind_a, kind_b) != nullptr; }

cudaError_t fused_shape(uint32_t kind_a, uint32_t kind_b, const void** fn, int* threads, int* smem) {
  const Entry* e = table(kind_a, kind_b);
  if (!e) return cudaErrorInvalidValue;
  *fn = e->fn;
  *threads = e->threads;
  *smem = e->smem;
  return cudaSuccess;
}

cudaError_t launch_fused(uint32_t kind_a, uint32_t kind_b, const WorkerCommon& wa, const void* args_a,
                         const WorkerCommon& wb, const void* args_b, uint32_t grow_on_drain, uint32_t grid,
                         cudaStream_t st) {
  const Entry* e = table(kind_a, kind_b);
  if (!e) return cudaErrorInvalidValue;
  return e->launch(wa, args_a, wb, args_b, grow_on_drain, grid, st);
}

}  // namespace slate
