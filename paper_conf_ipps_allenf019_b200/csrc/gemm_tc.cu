// gemm_tc.cu -- the tensor-core tenant: C (fp32) = A (bf16, m x k, K-major) x B^T
// (B bf16, n x k, K-major), one 128 x 128 output tile per original block
// (BASELINE configs 3 and 4).
//
// sm_100a design: warp-specialised, one CTA per SM.
//   warp 0  TMA producer: 64-wide K slices of A and B (SWIZZLE_128B boxes of
//           128 x 64 bf16) into a 6-stage shared-memory ring; it also makes
//           the slate task decision (resize word + task counter) at each tile
//           boundary and hands tile indices to the other roles.
//   warp 1  MMA issuer: one elected thread issues tcgen05.mma (M=128, N=128,
//           K=16, bf16 -> fp32) into a double-buffered TMEM accumulator and
//           commits to mbarriers.
//   warp 2  TMEM allocator (256 columns).
//   warps 4-7 epilogue: tcgen05.ld 32x32b -> registers -> fp32 stores; it
//           counts the tile done (blocks_done) only after its stores.
// The standalone kernel K(B,T) runs exactly one tile per CTA from blockIdx with
// the same code and the same MMA sequence, so outputs are bit-identical.
#include <cstring>
#include <cuda.h>
#include "gemm_tc.cuh"
#include "slate_device.cuh"

namespace slate {
namespace gemm {

#ifndef SLATE_GEMM_BN
#define SLATE_GEMM_BN 256
#endif
constexpr int BM = 128, BN = SLATE_GEMM_BN, BK = 64;   // tile and K slice
constexpr int kStageBytes = (BM + BN) * BK * 2;        // 32 KiB (BN 128) / 48 KiB (BN 256)
constexpr int kStages = (6 * 32768) / kStageBytes;     // ~192 KiB ring
constexpr int kThreads = 256;
constexpr int kTmemCols = 2 * BN;                      // two fp32 accumulators of BN columns
constexpr int kSmemBytes = 1024 /*align slack*/ + kStages * kStageBytes + 256 /*barriers*/;

struct Params {
  CUtensorMap tma_a;     // 64-B aligned members first
  CUtensorMap tma_b;
  slate_args_gemm args;
  uint32_t gx, gy, B, iters, occ, bound_lo, bound_hi, n_ranks, standby_timeout_ns;
  const uint64_t* ctrl;
  TaskCtl* tc;
  HostMirror* mirror;
  uint32_t* cov;
  const uint16_t* rank_of;
};

// ------------------------------------------------------------------ PTX wrappers
__device__ __forceinline__ uint32_t s_u32(const void* p) { return uint32_t(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(s_u32(b)), "r"(n) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(s_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(s_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "W_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra W_%=;\n}" ::"r"(s_u32(b)),
      "r"(parity)
      : "memory");
}
// operand panels are re-read by neighbouring tiles: keep them in L2 (evict-last;
// evict-normal for B measured no different)
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, int x, int y, uint64_t* bar) {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%2, "
      "%3}], [%4], %5;" ::"r"(s_u32(dst)),
      "l"(map), "r"(x), "r"(y), "r"(s_u32(bar)), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap* m) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(m) : "memory");
}
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(s_u32(bar))
               : "memory");
}
__device__ __forceinline__ void tc_mma(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc)
      : "memory");
}
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, "
      "%16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]),
        "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]),
        "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// UMMA shared-memory descriptor, K-major, SWIZZLE_128B: start address >> 4,
// LBO 1 (unused for swizzled K-major), SBO = 1024 B (8 rows x 128 B), version 1
// (sm_100), layout SWIZZLE_128B (2) in bits 61-63.
__device__ __forceinline__ uint64_t sw128_desc(uint32_t saddr) {
  const uint64_t lo = uint64_t((saddr >> 4) & 0x3FFFu) | (uint64_t(1) << 16);
  const uint64_t hi = uint64_t(1024 >> 4) | (uint64_t(1) << 14) | (uint64_t(2) << 29);
  return lo | (hi << 32);
}
// instruction descriptor: D fp32, A bf16, B bf16, both K-major, N = BN, M = BM
constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | (uint32_t(BN >> 3) << 17) | (uint32_t(BM >> 4) << 24);

// Original block b -> output tile (m, n): grouped rasterisation, kGroupM tile
// rows per group swept column by column, so the ~148 tiles in flight share a
// few A row panels and B column panels in L2 (a property of the tenant kernel:
// standalone and slate use the same map; every tile is computed exactly once).
// 16 rows of 128x256 tiles: each B column panel is fetched from DRAM 64/16 = 4
// times at 8192^3; ncu DRAM reads 0.91 GB per launch (8 rows: 1.33 GB; 32
// rows: 1.20 GB, the 64 MB of A panels no longer stay resident).
#ifndef SLATE_GEMM_GROUP_M
#define SLATE_GEMM_GROUP_M 16
#endif
constexpr uint32_t kGroupM = SLATE_GEMM_GROUP_M;
__device__ __forceinline__ void tile_of(uint32_t b, uint32_t gx, uint32_t gy, uint32_t& m0, uint32_t& n0) {
  const uint32_t per_group = kGroupM * gx;
  const uint32_t first_m = (b / per_group) * kGroupM;
  const uint32_t rows = min(gy - first_m, kGroupM);
  const uint32_t r = b % per_group;
  m0 = (first_m + r % rows) * BM;
  n0 = (r / rows) * BN;
}

struct Smem {
  uint64_t full[kStages], empty[kStages];
  uint64_t tmem_full[2], tmem_empty[2];
  uint64_t tq_full[2], tq_empty[2];
  uint64_t drain;
  uint32_t tileq[2];
  volatile uint32_t kb_limit[2];   // k-slices the producer issues for the tile in queue slot j
  volatile uint32_t aborted[2];    // the tile in accumulator b was abandoned (Q28): no store
  uint32_t tmem_base;
  uint32_t go, rank, retired;
};

__device__ __forceinline__ bool mbar_try(uint64_t* b, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(s_u32(b)), "r"(parity)
      : "memory");
  return ok != 0;
}

// ------------------------------------------------------------------ the kernel
template <bool kSlate>
__global__ void __launch_bounds__(kThreads, 1) gemm_kernel(const __grid_constant__ Params p) {
  extern __shared__ __align__(1024) char smem_raw[];
  // 1024-B aligned ring (SWIZZLE_128B atoms), barriers after it
  char* ring = reinterpret_cast<char*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  Smem& S = *reinterpret_cast<Smem*>(ring + kStages * kStageBytes);
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint64_t c = 0;

  if constexpr (kSlate) {
    // ---- Lst1 binding + standby (shared with every tenant: slate_device.cuh)
    if (threadIdx.x == 0) {
      const uint32_t r = p.rank_of[smid()];
      S.rank = r;
      S.retired = 0;
      S.go = prologue(p, r, c) ? 1u : 0u;
    }
    __syncthreads();
    if (!S.go) return;
  }
  if (threadIdx.x == 32) {
    for (int i = 0; i < kStages; ++i) {
      mbar_init(&S.full[i], 1);
      mbar_init(&S.empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&S.tmem_full[i], 1);
      mbar_init(&S.tmem_empty[i], 1);
      mbar_init(&S.tq_full[i], 1);
      mbar_init(&S.tq_empty[i], 1 + 4);   // MMA thread + one lane of each epilogue warp
      S.aborted[i] = 0;
    }
    mbar_init(&S.drain, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0 && lane == 0) {
    prefetch_tmap(&p.tma_a);
    prefetch_tmap(&p.tma_b);
  }
  if (warp == 2) {   // TMEM: only CTAs that work hold it (standby CTAs returned above)
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(s_u32(&S.tmem_base)),
                 "n"(kTmemCols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = S.tmem_base;
  const uint32_t num_kb = p.args.k / BK;

  if (warp == 0) {
    // ===================== producer + slate task decisions =====================
    if (lane == 0) {
      uint32_t t = 0, it = 0;   // tiles handed out, k-slices issued
      bool stop = false;
      while (!stop) {
        uint32_t g = 0xffffffffu, n = 1;
        if constexpr (kSlate) {
          // task boundary: resize word, returned tasks, then the counter
          c = ld_acquire_u64(p.ctrl);
          if (!in_range(p, S.rank, c) && try_retire(p.tc)) {
            S.retired = 1;
          } else {
            bool leave;
            g = take_returned(p.tc, false, leave);            // an abandoned tile first (Q28)
            if (g == 0xffffffffu) {
              const uint32_t f = atomicAdd(&p.tc->next, p.iters);   // Lst2 (2)
              if (f < p.B) {
                g = f;
                n = min(p.iters, p.B - f);
                if (f == 0) p.tc->t_first = globaltimer();
              } else {
                g = take_returned(p.tc, true, leave);          // drained: leave unless one was returned
              }
            }
          }
        } else {
          g = t == 0 ? blockIdx.y * gridDim.x + blockIdx.x : 0xffffffffu;
        }
        if (g == 0xffffffffu) break;
        // a task = n consecutive tiles (SLATE_ITERS), handed out one by one;
        // bit 31 marks the last tile of the task (tasks_done counts tasks)
        for (uint32_t i = 0; i < n && !stop; ++i) {
          const uint32_t tile = g + i;
          const uint32_t j = t & 1, u = t >> 1;
          mbar_wait(&S.tq_empty[j], (u & 1) ^ 1);
          S.kb_limit[j] = num_kb;
          S.tileq[j] = tile | (i + 1 == n ? 0x80000000u : 0u);
          mbar_arrive(&S.tq_full[j]);
          ++t;
          uint32_t m0, n0;
          tile_of(tile, p.gx, p.gy, m0, n0);
          for (uint32_t kb = 0; kb < num_kb; ++kb, ++it) {
            if constexpr (kSlate) {
              // Q28: a worker that left the range abandons its tile mid-way (if it
              // is not the last live worker) and gives the tile back; nothing of it
              // is stored.  Checked every 16 K slices (~4-8 us).
              if ((kb & 15) == 15 && n == 1) {
                const uint64_t c2 = ld_acquire_u64(p.ctrl);
                if (!in_range(p, S.rank, c2) && try_retire(p.tc, true)) {
                  give_back_task(p.tc, tile);
                  c = c2;
                  S.retired = 1;
                  S.kb_limit[j] = kb;            // the MMA consumes the kb slices issued, then aborts
                  stop = true;
                  break;
                }
              }
            }
            const uint32_t s = it % kStages, r = it / kStages;
            mbar_wait(&S.empty[s], (r & 1) ^ 1);
            char* sa = ring + s * kStageBytes;
            char* sb = sa + BM * BK * 2;
            mbar_expect_tx(&S.full[s], kStageBytes);
            tma_load_2d(sa, &p.tma_a, int(kb * BK), int(m0), &S.full[s]);
            tma_load_2d(sb, &p.tma_b, int(kb * BK), int(n0), &S.full[s]);
          }
        }
      }
      // sentinel: the other roles stop after the tiles already handed out
      const uint32_t j = t & 1, u = t >> 1;
      mbar_wait(&S.tq_empty[j], (u & 1) ^ 1);
      S.tileq[j] = 0xffffffffu;
      mbar_arrive(&S.tq_full[j]);
    }
  } else if (warp == 1) {
    // ===================== MMA issuer (one thread) =====================
    if (lane == 0) {
      uint32_t t = 0, it = 0;
      for (;;) {
        const uint32_t j = t & 1, u = t >> 1;
        mbar_wait(&S.tq_full[j], u & 1);
        const uint32_t g = S.tileq[j];
        if (g == 0xffffffffu) {
          mbar_arrive(&S.tq_empty[j]);
          break;
        }
        const uint32_t b = t & 1, v = t >> 1;
        mbar_wait(&S.tmem_empty[b], (v & 1) ^ 1);     // the epilogue has drained this accumulator
        tc_fence_after();
        const uint32_t d = tmem + b * BN;
        bool abandoned = false;
        for (uint32_t kb = 0; kb < num_kb; ++kb, ++it) {
          const uint32_t s = it % kStages, r = it / kStages;
          while (!mbar_try(&S.full[s], r & 1)) {
            if (kb >= S.kb_limit[j]) { abandoned = true; break; }   // Q28: no more slices will come
          }
          if (abandoned) break;
          tc_fence_after();
          const uint32_t sa = s_u32(ring + s * kStageBytes);
          const uint32_t sb = sa + BM * BK * 2;
#pragma unroll
          for (uint32_t kk = 0; kk < BK / 16; ++kk)   // K = 16 per instruction: +32 B in the swizzled row
            tc_mma(d, sw128_desc(sa + kk * 32), sw128_desc(sb + kk * 32), kIdesc, (kb | kk) != 0);
          tc_commit(&S.empty[s]);                      // frees the stage when these MMAs complete
        }
        mbar_arrive(&S.tq_empty[j]);
        if (abandoned) {
          tc_commit(&S.drain);                          // the issued MMAs finish before TMEM is let go
          mbar_wait(&S.drain, 0);
          S.aborted[b] = 1;
          mbar_arrive(&S.tmem_full[b]);                 // wake the epilogue: nothing to store
        } else {
          tc_commit(&S.tmem_full[b]);                   // accumulator ready
        }
        ++t;
      }
    }
  } else if (warp >= 4) {
    // ===================== epilogue: TMEM -> registers -> global =====================
    const uint32_t ew = warp - 4;                      // TMEM lanes 32*ew .. 32*ew + 31
    uint32_t t = 0;
    for (;;) {
      const uint32_t j = t & 1, u = t >> 1;
      mbar_wait(&S.tq_full[j], u & 1);
      const uint32_t entry = S.tileq[j];
      __syncwarp();
      if (lane == 0) mbar_arrive(&S.tq_empty[j]);
      if (entry == 0xffffffffu) break;
      const uint32_t g = entry & 0x7fffffffu;
      const bool last_of_task = (entry >> 31) != 0;
      const uint32_t b = t & 1, v = t >> 1;
      mbar_wait(&S.tmem_full[b], v & 1);
      tc_fence_after();
      if (S.aborted[b]) {                               // abandoned tile (Q28): nothing stored or counted
        asm volatile("bar.sync 1, 128;" ::: "memory");
        if (ew == 0 && lane == 0) {
          S.aborted[b] = 0;
          mbar_arrive(&S.tmem_empty[b]);
        }
        ++t;
        continue;
      }
      uint32_t m0, n0;
      tile_of(g, p.gx, p.gy, m0, n0);
      const uint32_t row = m0 + ew * 32 + lane;
      float* crow = reinterpret_cast<float*>(p.args.C) + uint64_t(row) * p.args.n + n0;
#pragma unroll 1
      for (uint32_t cb = 0; cb < BN / 32; ++cb) {
        uint32_t r[32];
        tmem_ld32(tmem + ((ew * 32) << 16) + b * BN + cb * 32, r);
        float4* dst = reinterpret_cast<float4*>(crow + cb * 32);
#pragma unroll
        for (int q = 0; q < 8; ++q)
          __stcs(dst + q, make_float4(__uint_as_float(r[4 * q]), __uint_as_float(r[4 * q + 1]),
                                      __uint_as_float(r[4 * q + 2]), __uint_as_float(r[4 * q + 3])));
      }
      tc_fence_before();
      asm volatile("bar.sync 1, 128;" ::: "memory");   // the 4 epilogue warps finished this tile
      if (ew == 0 && lane == 0) {
        mbar_arrive(&S.tmem_empty[b]);
        if constexpr (kSlate) {
          if (p.cov) atomicAdd(&p.cov[g], 1u);
          count_done(p, 1u, last_of_task ? 1u : 0u);
        }
      }
      ++t;
    }
  }
  __syncthreads();
  if (warp == 2) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(kTmemCols) : "memory");
  }
  if constexpr (kSlate) {
    if (warp == 0) {
      c = __shfl_sync(0xffffffffu, c, 0);
      if (lane == 0) atomicAdd(&p.tc->live_rank[S.rank], 0xffffffffu);
      if (S.retired) check_shrink_done(p, c, lane);
    }
  }
}

// ------------------------------------------------------------------ host side
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess) fn = (EncodeTiledFn)f;
  }
  return fn;
}

// a rows x k bf16 K-major matrix, boxes of box_rows rows x 64 columns, 128-B swizzle
static bool make_map(CUtensorMap* m, const void* base, uint32_t rows, uint32_t k, uint32_t box_rows) {
  EncodeTiledFn enc = encode_fn();
  if (!enc) return false;
  const cuuint64_t dims[2] = {k, rows};
  const cuuint64_t strides[1] = {cuuint64_t(k) * 2};
  const cuuint32_t box[2] = {BK, box_rows};
  const cuuint32_t estr[2] = {1, 1};
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, estr,
             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

static cudaError_t fill(Params& p, const void* args) {
  std::memset(&p, 0, sizeof(p));
  std::memcpy(&p.args, args, sizeof(p.args));
  if (!make_map(&p.tma_a, reinterpret_cast<const void*>(p.args.A), p.args.m, p.args.k, BM) ||
      !make_map(&p.tma_b, reinterpret_cast<const void*>(p.args.B), p.args.n, p.args.k, BN))
    return cudaErrorInvalidValue;
  return cudaSuccess;
}

static cudaError_t launch_worker(const WorkerCommon& w, const void* args, uint32_t grid, cudaStream_t st) {
  Params p;
  cudaError_t e = fill(p, args);
  if (e != cudaSuccess) return e;
  p.gx = w.gx; p.gy = w.gy; p.B = w.B; p.iters = w.iters; p.occ = w.occ;
  p.bound_lo = w.bound_lo; p.bound_hi = w.bound_hi; p.n_ranks = w.n_ranks;
  p.standby_timeout_ns = w.standby_timeout_ns;
  p.ctrl = w.ctrl; p.tc = w.tc; p.mirror = w.mirror; p.cov = w.cov; p.rank_of = w.rank_of;
  void* kargs[] = {&p};
  return cudaLaunchKernel(reinterpret_cast<const void*>(&gemm_kernel<true>), dim3(grid), dim3(kThreads), kargs,
                          kSmemBytes, st);
}

static cudaError_t launch_standalone(const void* args, dim3 grid, cudaStream_t st) {
  Params p;
  cudaError_t e = fill(p, args);
  if (e != cudaSuccess) return e;
  p.gx = grid.x; p.gy = grid.y; p.B = grid.x * grid.y;
  void* kargs[] = {&p};
  return cudaLaunchKernel(reinterpret_cast<const void*>(&gemm_kernel<false>), grid, dim3(kThreads), kargs, kSmemBytes,
                          st);
}

}  // namespace gemm

KindOps gemm_tc_ops() {
  KindOps o;
  o.worker_fn = reinterpret_cast<const void*>(&gemm::gemm_kernel<true>);
  o.standalone_fn = reinterpret_cast<const void*>(&gemm::gemm_kernel<false>);
  o.threads = gemm::kThreads;
  o.smem = gemm::kSmemBytes;
  o.smem_standalone = gemm::kSmemBytes;
  o.args_size = sizeof(slate_args_gemm);
  o.default_iters = 1;   // one tile per task: resize latency ~ one tile (SURVEY §7 hard part 3)
  o.max_auto_iters = 1;
  o.tile_n = gemm::BN;
  o.launch_worker = &gemm::launch_worker;
  o.launch_standalone = &gemm::launch_standalone;
  return o;
}

}  // namespace slate
