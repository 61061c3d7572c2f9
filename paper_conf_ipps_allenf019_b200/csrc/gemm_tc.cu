// gemm_tc.cu -- the tensor-core tenant: C (fp32) = A (bf16, m x k, K-major) x B^T
// (B bf16, n x k, K-major), one 256 x 256 output tile per original block
// (BASELINE configs 3 and 4).
//
// sm_100a design: a CTA PAIR (cluster of 2 on one TPC) per tile,
// one CTA per SM, cta_group::2 MMA (M = 256, N = 256, K = 16).  CTA r of the
// pair stages A rows [128 r, 128 r + 128) and B rows [128 r, 128 r + 128) of the
// tile; the pair's MMA reads both CTAs' shared memory and leaves rows
// [128 r, 128 r + 128) of the accumulator in CTA r's TMEM.  Per SM this halves
// the B bytes per FLOP (32 KiB stages instead of 48 KiB), so the ring holds
// kStages = 7 K slices (~1.9 us of MMA work) instead of 4: what lets the GEMM
// ride out the memory latency a co-running HBM-bound tenant causes (DESIGN.md
// §8), and what brings the shared-memory traffic per MMA under the SM's
// 128 B/clk.
//   warp 0  TMA producer.  Leader CTA: the slate task decision (resize word,
//           returned tiles, task counter) at each tile boundary, hands tile
//           indices to both CTAs, issues its halves of each K slice and arms
//           the pair's full barrier for both; peer CTA: issues its halves of
//           exactly the slices the leader issued (lock-step through
//           `lead_issued`, so an abandoned tile leaves both rings aligned).
//   warp 1  MMA issuer (leader CTA only): one thread issues tcgen05.mma.cta_group::2
//           into a double-buffered TMEM accumulator (2 x 256 columns) and
//           multicasts its commits to both CTAs' barriers.
//   warp 2  TMEM allocator (cta_group::2, 512 columns).
//   warps 4-7 epilogue (both CTAs): tcgen05.ld 32x32b -> registers -> fp32
//           stores of the CTA's 128 rows; the second CTA of the pair to finish
//           a tile counts it done.
// The standalone kernel K(B,T) runs exactly one tile per cluster with the same
// code and the same MMA sequence, so outputs are bit-identical.
#include <cstring>
#include <cuda.h>
#include "gemm_tc.cuh"
#include "slate_device.cuh"

namespace slate {
namespace gemm {

constexpr int BM = 128;                 // A rows per CTA (the pair's tile has 2 * BM)
constexpr int BN = 256;                 // tile columns (each CTA stages BN / 2 rows of B)
constexpr int BK = 64;                  // K slice (one SWIZZLE_128B atom of bf16)
constexpr int kTileM = 2 * BM;
constexpr int kHalfBytes = BM * BK * 2;                 // 16 KiB: one operand half of one slice
constexpr int kStageBytes = 2 * kHalfBytes;             // A half + B half per CTA
constexpr int kPairStageBytes = 2 * kStageBytes;        // what the leader's full barrier expects
#ifndef SLATE_GEMM_TMA_STORE
#define SLATE_GEMM_TMA_STORE 1
#endif
#ifndef SLATE_GEMM_STAGES
#define SLATE_GEMM_STAGES (SLATE_GEMM_TMA_STORE ? 6 : 7)
#endif
constexpr int kStages = SLATE_GEMM_STAGES;
constexpr int kThreads = 256;
constexpr int kTmemCols = 2 * BN;                       // two fp32 accumulators of BN columns
// epilogue staging for the TMA store of C: per epilogue warp two 32 x 32 fp32
// boxes (4 KiB each, SWIZZLE_128B), so a box is written while the previous one drains
constexpr int kBoxBytes = 32 * 32 * 4;
constexpr int kStagingBytes = SLATE_GEMM_TMA_STORE ? 4 * 2 * kBoxBytes : 0;
constexpr int kSmemBytes = 1024 /*align slack*/ + kStages * kStageBytes + kStagingBytes + 512 /*barriers*/;
static_assert(kSmemBytes <= 232448, "shared memory budget");

struct Params {
  CUtensorMap tma_a;     // 64-B aligned members first
  CUtensorMap tma_b;
  CUtensorMap tma_c;     // fp32 C, boxes of 32 x 32, SWIZZLE_128B (epilogue TMA store)
  slate_args_gemm args;
  uint32_t gx, gy, B, iters, occ, bound_lo, bound_hi, n_ranks, standby_timeout_ns, base_epoch;
  uint32_t is_topup, gate_first, ranklog;   // as WorkerParams (slate_device.cuh)
  const uint64_t* ctrl;
  TaskCtl* tc;
  HostMirror* mirror;
  uint32_t* cov;
  const uint16_t* rank_of;
};

// ------------------------------------------------------------------ PTX wrappers
__device__ __forceinline__ uint32_t s_u32(const void* p) { return uint32_t(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ uint32_t cta_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
// shared::cluster address of the same variable in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t mapa(const void* p, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(s_u32(p)), "r"(rank));
  return r;
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ void st_cluster(uint32_t raddr, uint32_t v) {
  asm volatile("st.relaxed.cluster.shared::cluster.u32 [%0], %1;" ::"r"(raddr), "r"(v) : "memory");  // racecheck: mbarrier-ordered (every use is followed by a remote arrive or a cluster barrier)
}
// the leader's progress word in the peer's shared memory: only ever raised
// (K slices issued, bit 31 when it stopped), so the writer is an atomic max and
// the reader an atomic read -- both cluster-scope atomics, no plain access
__device__ __forceinline__ void red_max_cluster(uint32_t raddr, uint32_t v) {
  asm volatile("red.relaxed.cluster.shared::cluster.max.u32 [%0], %1;" ::"r"(raddr), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_relaxed_cluster(const volatile uint32_t* p) {
  uint32_t v;
  asm volatile("atom.relaxed.cluster.shared::cta.or.b32 %0, [%1], 0;" : "=r"(v) : "r"(s_u32((const void*)p)) : "memory");
  return v;
}
// a 32-bit word of another CTA's shared memory (after a cluster barrier)
__device__ __forceinline__ uint32_t ld_shared_cluster(uint32_t raddr) {
  uint32_t v;
  asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(raddr) : "memory");
  return v;
}
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(s_u32(b)), "r"(n) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(s_u32(b)) : "memory");
}
// after observing a barrier phase that a remote CTA completed with a release
// arrive: makes that CTA's earlier shared-memory writes visible (once per tile)
__device__ __forceinline__ void fence_cluster() { asm volatile("fence.acq_rel.cluster;" ::: "memory"); }
__device__ __forceinline__ void mbar_arrive_remote(uint32_t raddr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(raddr) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(s_u32(b)), "r"(bytes) : "memory");
}
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
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "W_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra W_%=;\n}" ::"r"(s_u32(b)),
      "r"(parity)
      : "memory");
}
// One CTA's half of a K slice; the bytes are counted on the LEADER's barrier
// (`bar` is a shared::cluster address in CTA 0).  Operand panels are re-read by
// neighbouring tiles: keep them in L2 (evict-last).
__device__ __forceinline__ void tma_load_half(void* dst, const CUtensorMap* map, int x, int y, uint32_t bar) {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint "
      "[%0], [%1, {%2, %3}], [%4], %5;" ::"r"(s_u32(dst)),
      "l"(map), "r"(x), "r"(y), "r"(bar), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap* m) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(m) : "memory");
}
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
// completion of the pair's issued MMAs -> the barrier at this offset in BOTH CTAs
__device__ __forceinline__ void tc_commit_pair(uint64_t* bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          s_u32(bar)),
      "h"(uint16_t(3))
      : "memory");
}
// ... -> the barrier in the leader only
__device__ __forceinline__ void tc_commit_local(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(s_u32(bar))
               : "memory");
}
__device__ __forceinline__ void tc_mma(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
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
// instruction descriptor: D fp32, A bf16, B bf16, both K-major, N = BN, M = 2 * BM (the pair)
constexpr uint32_t kIdesc =
    (1u << 4) | (1u << 7) | (1u << 10) | (uint32_t(BN >> 3) << 17) | (uint32_t(kTileM >> 4) << 24);

// Original block b -> output tile (m, n): grouped rasterisation, kGroupM tile
// rows per group swept column by column, so the ~74 tiles in flight share a
// few A row panels and B column panels in L2 (a property of the tenant kernel:
// standalone and slate use the same map; every tile is computed exactly once).
// 8 rows of 256 x 256 tiles = 2048 rows of A per group: each B column panel is
// fetched from DRAM 4 times at 8192^3 (measured with 128-row tiles: 16 rows
// 0.91 GB of DRAM reads per launch, 8 rows 1.33 GB, 32 rows 1.20 GB; with the
// current 256 x 256 CTA-pair tiles, profiles/r1_gemm_groupm_sweep.md: 4 rows
// 1.36 GB, 8 rows 0.94 GB, 16 rows 1.29 GB, 32 rows 2.45 GB, and 8 is also the
// fastest solo and in the C3 co-run).
#ifndef SLATE_GEMM_GROUP_M
#define SLATE_GEMM_GROUP_M 8
#endif
constexpr uint32_t kGroupM = SLATE_GEMM_GROUP_M;
__device__ __forceinline__ void tile_of(uint32_t b, uint32_t gx, uint32_t gy, uint32_t& m0, uint32_t& n0) {
  const uint32_t per_group = kGroupM * gx;
  const uint32_t first_m = (b / per_group) * kGroupM;
  const uint32_t rows = min(gy - first_m, kGroupM);
  const uint32_t r = b % per_group;
  m0 = (first_m + r % rows) * kTileM;
  n0 = (r / rows) * BN;
}

struct Smem {
  uint64_t full[kStages], empty[kStages];
  uint64_t tmem_full[2], tmem_empty[2];
  uint64_t tq_full[2], tq_empty[2];
  uint64_t drain;
  uint32_t tileq[2];
  volatile uint32_t kb_limit[2];   // k-slices issued for the tile in queue slot j
  volatile uint32_t aborted[2];    // the tile in accumulator b was abandoned (Q28): no store
  volatile uint32_t lead_issued;   // (peer) K slices the leader has issued so far; bit 31: it stopped
  uint32_t done_cnt[2];            // (leader) epilogues finished per accumulator, x2 per tile
  uint32_t tmem_base;
  uint32_t go, rank, peer_rank, retired;
};
static_assert(sizeof(Smem) <= 512, "barrier area");

// ------------------------------------------------------------------ slate bookkeeping for a pair
// The pair is one worker: it works only if BOTH SMs are in the range, it holds
// one unit of `live` and one of live_rank on each of its two ranks.
template <class P>
__device__ __forceinline__ bool pair_in_range(const P& p, uint32_t r0, uint32_t r1, uint64_t c) {
  return in_range(p, r0, c) && in_range(p, r1, c);
}
// Lst1 prologue for the pair (leader thread): slate_device.cuh's prologue with
// the pair's range test; the staffing target counts pairs.
template <class P>
__device__ bool pair_prologue(const P& p, uint32_t r0, uint32_t r1, uint64_t& c_out) {
  TaskCtl* tc = p.tc;
  uint64_t t0 = 0;
  uint32_t backoff = 256;
  if (p.gate_first) {   // top-up of a launch that has no start event: wait until it started
    // bounded: the gated launch may be queued behind other work and need the
    // very SM slots this top-up's waiting CTAs hold; a launch that starts later
    // reads the resize word by itself (its own grid is a full wave), so the
    // top-up may leave without joining
    const uint64_t tg = globaltimer();
    while (ld_relaxed_u64(&tc->t_first) == 0 && ld_relaxed_u32(&tc->next) < p.B) {
      if (globaltimer() - tg > p.standby_timeout_ns) return false;
      __nanosleep(512);
    }
  }
  for (;;) {
    const uint64_t c = ld_acquire_u64(p.ctrl);
    if (ld_relaxed_u32(&tc->next) >= p.B) return false;
    bool join = pair_in_range(p, r0, r1, c);
    if (!join) {
      const uint32_t live = uint32_t(ld_relaxed_u64(&tc->live_pending));
      const uint32_t target = (ctrl_hi(c) - ctrl_lo(c) + 1) / 2;
      if (live >= target) return false;
      if (t0 == 0) t0 = globaltimer();
      if (live == 0 && globaltimer() - t0 > p.standby_timeout_ns) join = true;
    }
    if (join) {
      atomicAdd(&tc->live_pending, 1ull);
      atomicAdd(&tc->live_rank[r0], 1u);
      atomicAdd(&tc->live_rank[r1], 1u);
      atomicAdd(&tc->started, 1u);
      const uint32_t e = ctrl_epoch(c);
      if (e > p.base_epoch && ld_relaxed_u32(&tc->join_epoch) < e && atomicMax(&tc->join_epoch, e) < e && p.mirror) {
        publish_mirror(&tc->join_word, &p.mirror->join, mirror_pack(e, globaltimer()));
      }
      c_out = c;
      return true;
    }
    __nanosleep(backoff);
    if (backoff < 4096) backoff <<= 1;
  }
}

// ------------------------------------------------------------------ the kernel
template <bool kSlate>
__global__ void __launch_bounds__(kThreads, 1) gemm_kernel(const __grid_constant__ Params p) {
  extern __shared__ __align__(1024) char smem_raw[];
  // 1024-B aligned ring (SWIZZLE_128B atoms), barriers after it; identical
  // offsets in both CTAs (the pair's MMA reads the peer at the leader's offsets)
  char* ring = reinterpret_cast<char*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  char* staging = ring + kStages * kStageBytes;
  Smem& S = *reinterpret_cast<Smem*>(staging + kStagingBytes);
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t crank = cta_rank();
  const bool leader = crank == 0;
  uint64_t c = 0;

  if (threadIdx.x == 32) {
    for (int i = 0; i < kStages; ++i) {
      mbar_init(&S.full[i], 1);      // leader: its expect_tx arrival + both CTAs' bytes
      mbar_init(&S.empty[i], 1);     // the pair's MMA commit (multicast)
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&S.tmem_full[i], 1);       // MMA commit (multicast) or the abort arrive
      mbar_init(&S.tmem_empty[i], 2);      // (leader) both CTAs' epilogues
      mbar_init(&S.tq_full[i], 1);         // the leader's producer
      mbar_init(&S.tq_empty[i], 10);       // (leader) MMA + 4 + 4 epilogue warps + peer producer
      S.aborted[i] = 0;
      S.done_cnt[i] = 0;
    }
    mbar_init(&S.drain, 1);
    S.lead_issued = 0;
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if constexpr (kSlate) {
    if (threadIdx.x == 0) {
      S.rank = p.rank_of[smid()];
      S.retired = 0;
    }
  }
  cluster_sync();   // the peer's rank is written (and both CTAs run) before any DSMEM access
  if constexpr (kSlate) {
    // ---- Lst1 binding + standby, by the leader for the pair
    if (leader && threadIdx.x == 0) {
      S.peer_rank = ld_shared_cluster(mapa(&S.rank, 1));
      const uint32_t go = pair_prologue(p, S.rank, S.peer_rank, c) ? 1u : 0u;
      S.go = go;
      st_cluster(mapa(&S.go, 1), go);
    }
    cluster_sync();
    if (!S.go) {
      if (threadIdx.x == 0) leave_main(p);   // every CTA of the grid counts (slate_device.cuh)
      return;
    }
  }
  if (warp == 0 && lane == 0) {
    prefetch_tmap(&p.tma_a);
    prefetch_tmap(&p.tma_b);
    if (SLATE_GEMM_TMA_STORE) prefetch_tmap(&p.tma_c);
  }
  if (warp == 2) {   // TMEM of both SMs, allocated by warp 2 of each CTA
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(s_u32(&S.tmem_base)),
                 "n"(kTmemCols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = S.tmem_base;
  const uint32_t num_kb = (p.args.k + BK - 1) / BK;   // a ragged last slice: zero-filled past k
  const uint32_t full0 = mapa(&S.full[0], 0);       // the leader's full barriers (shared::cluster)

  if (warp == 0 && lane == 0 && leader) {
    // ===================== leader producer + slate task decisions =====================
    const uint32_t r_tq_full[2] = {mapa(&S.tq_full[0], 1), mapa(&S.tq_full[1], 1)};
    const uint32_t r_tileq[2] = {mapa(&S.tileq[0], 1), mapa(&S.tileq[1], 1)};
    const uint32_t r_issued = mapa((const void*)&S.lead_issued, 1);
    uint32_t t = 0, it = 0;   // tiles handed out, k-slices issued
    bool stop = false;
    auto hand_out = [&](uint32_t entry) {
      const uint32_t j = t & 1, u = t >> 1;
      mbar_wait(&S.tq_empty[j], (u & 1) ^ 1);
      fence_cluster();                             // the peer's reads of slot j happened
      S.kb_limit[j] = num_kb;
      S.tileq[j] = entry;  // racecheck: mbarrier-ordered
      st_cluster(r_tileq[j], entry);
      mbar_arrive(&S.tq_full[j]);
      mbar_arrive_remote(r_tq_full[j]);
      ++t;
      return j;
    };
    while (!stop) {
      uint32_t g = 0xffffffffu, n = 1;
      if constexpr (kSlate) {
        // task boundary: resize word, returned tasks, then the counter
        c = ld_acquire_u64(p.ctrl);
        const bool inr = pair_in_range(p, S.rank, S.peer_rank, c);
        if (!inr && try_retire(p.tc)) {
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
          if (g != 0xffffffffu) log_task(p, g, S.rank, c, !inr);   // the leader's rank (the pair is in or out together)
        }
      } else {
        g = t == 0 ? blockIdx.y * (gridDim.x >> 1) + (blockIdx.x >> 1) : 0xffffffffu;
      }
      if (g == 0xffffffffu) break;
      // a task = n consecutive tiles (SLATE_ITERS), handed out one by one;
      // bit 31 marks the last tile of the task (tasks_done counts tasks)
      for (uint32_t i = 0; i < n && !stop; ++i) {
        const uint32_t tile = g + i;
        const uint32_t j = hand_out(tile | (i + 1 == n ? 0x80000000u : 0u));
        uint32_t m0, n0;
        tile_of(tile, p.gx, p.gy, m0, n0);
        for (uint32_t kb = 0; kb < num_kb; ++kb, ++it) {
          if constexpr (kSlate) {
            // Q28: a pair that left the range abandons its tile mid-way (if it is
            // not the last live worker) and gives the tile back; nothing of it is
            // stored.  Checked every 16 K slices (~4-5 us).
            if ((kb & 15) == 15 && n == 1) {
              const uint64_t c2 = ld_acquire_u64(p.ctrl);
              if (!pair_in_range(p, S.rank, S.peer_rank, c2) && try_retire(p.tc, true)) {
                give_back_task(p.tc, tile);
                c = c2;
                S.retired = 1;
                S.kb_limit[j] = kb;            // the MMA consumes the kb slices issued, then aborts
                red_max_cluster(r_issued, it | 0x80000000u);   // ... and the peer issues exactly those
                stop = true;
                break;
              }
            }
          }
          const uint32_t s = it % kStages, r = it / kStages;
          mbar_wait(&S.empty[s], (r & 1) ^ 1);
          char* sa = ring + s * kStageBytes;
          mbar_expect_tx(&S.full[s], kPairStageBytes);
          tma_load_half(sa, &p.tma_a, int(kb * BK), int(m0), full0 + s * 8);
          tma_load_half(sa + kHalfBytes, &p.tma_b, int(kb * BK), int(n0), full0 + s * 8);
          red_max_cluster(r_issued, it + 1);   // one location, so the peer sees the counts in order
        }
      }
    }
    hand_out(0xffffffffu);   // sentinel: every role of both CTAs stops after the tiles handed out
  } else if (warp == 0 && lane == 0) {
    // ===================== peer producer: the leader's slices, in lock-step =====================
    const uint32_t tq_empty0 = mapa(&S.tq_empty[0], 0);
    uint32_t t = 0, it = 0;
    for (;;) {
      const uint32_t j = t & 1, u = t >> 1;
      mbar_wait(&S.tq_full[j], u & 1);
      fence_cluster();
      const uint32_t entry = S.tileq[j];
      mbar_arrive_remote(tq_empty0 + j * 8);
      ++t;
      if (entry == 0xffffffffu) break;
      uint32_t m0, n0;
      tile_of(entry & 0x7fffffffu, p.gx, p.gy, m0, n0);
      bool cut = false;
      for (uint32_t kb = 0; kb < num_kb; ++kb, ++it) {
        // the leader issued slice #it of the pair's sequence, or stopped before it
        for (;;) {
          const uint32_t li = ld_relaxed_cluster(&S.lead_issued);
          if ((li & 0x7fffffffu) > it) break;
          if (li >> 31) { cut = true; break; }
        }
        if (cut) break;
        const uint32_t s = it % kStages, r = it / kStages;
        mbar_wait(&S.empty[s], (r & 1) ^ 1);
        char* sa = ring + s * kStageBytes;
        tma_load_half(sa, &p.tma_a, int(kb * BK), int(m0 + BM), full0 + s * 8);
        tma_load_half(sa + kHalfBytes, &p.tma_b, int(kb * BK), int(n0 + BN / 2), full0 + s * 8);
      }
    }
  } else if (warp == 1 && lane == 0 && leader) {
    // ===================== MMA issuer (leader, one thread) =====================
    const uint32_t r_aborted[2] = {mapa((const void*)&S.aborted[0], 1), mapa((const void*)&S.aborted[1], 1)};
    const uint32_t r_tmem_full[2] = {mapa(&S.tmem_full[0], 1), mapa(&S.tmem_full[1], 1)};
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
      mbar_wait(&S.tmem_empty[b], (v & 1) ^ 1);     // both epilogues drained this accumulator
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
        const uint32_t sb = sa + kHalfBytes;
#pragma unroll
        for (uint32_t kk = 0; kk < BK / 16; ++kk)   // K = 16 per instruction: +32 B in the swizzled row
          tc_mma(d, sw128_desc(sa + kk * 32), sw128_desc(sb + kk * 32), kIdesc, (kb | kk) != 0);
        tc_commit_pair(&S.empty[s]);                 // frees the stage in both CTAs when these complete
      }
      mbar_arrive(&S.tq_empty[j]);
      if (abandoned) {
        tc_commit_local(&S.drain);                   // the issued MMAs finish before TMEM is let go
        mbar_wait(&S.drain, 0);
        S.aborted[b] = 1;
        st_cluster(r_aborted[b], 1u);
        mbar_arrive(&S.tmem_full[b]);                // wake both epilogues: nothing to store
        mbar_arrive_remote(r_tmem_full[b]);
      } else {
        tc_commit_pair(&S.tmem_full[b]);             // accumulator ready in both CTAs
      }
      ++t;
    }
  } else if (warp >= 4) {
    // ===================== epilogue (both CTAs): TMEM -> registers -> global =====================
    const uint32_t ew = warp - 4;                    // TMEM lanes 32*ew .. 32*ew + 31
    const uint32_t tq_empty0 = mapa(&S.tq_empty[0], 0);
    const uint32_t tmem_empty0 = mapa(&S.tmem_empty[0], 0);
    const uint32_t done_cnt0 = mapa(&S.done_cnt[0], 0);
    uint32_t t = 0;
    for (;;) {
      const uint32_t j = t & 1, u = t >> 1;
      mbar_wait(&S.tq_full[j], u & 1);
      if (!leader) fence_cluster();
      const uint32_t entry = S.tileq[j];  // racecheck: mbarrier-ordered
      __syncwarp();
      if (lane == 0) mbar_arrive_remote(tq_empty0 + j * 8);
      if (entry == 0xffffffffu) break;
      const uint32_t g = entry & 0x7fffffffu;
      const bool last_of_task = (entry >> 31) != 0;
      const uint32_t b = t & 1, v = t >> 1;
      mbar_wait(&S.tmem_full[b], v & 1);
      tc_fence_after();
      if (!leader) fence_cluster();                   // the leader's abort flag
      if (S.aborted[b]) {                              // abandoned tile (Q28): nothing stored or counted
        asm volatile("bar.sync 1, 128;" ::: "memory");
        if (ew == 0 && lane == 0) {
          S.aborted[b] = 0;
          mbar_arrive_remote(tmem_empty0 + b * 8);
        }
        ++t;
        continue;
      }
      uint32_t m0, n0;
      tile_of(g, p.gx, p.gy, m0, n0);
#if SLATE_GEMM_TMA_STORE
      // TMEM -> registers -> swizzled staging box -> TMA store (coalesced by the
      // bulk engine; the LSU only writes shared memory)
      const uint32_t y0 = m0 + crank * BM + ew * 32;
#pragma unroll 1
      for (uint32_t cb = 0; cb < BN / 32; ++cb) {
        uint32_t r[32];
        tmem_ld32(tmem + ((ew * 32) << 16) + b * BN + cb * 32, r);
        char* box = staging + (ew * 2 + (cb & 1)) * kBoxBytes;
        if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");   // box drained
        __syncwarp();
#pragma unroll
        for (int q = 0; q < 8; ++q)   // row `lane`, 16-B chunk q at chunk position q ^ (row % 8)
          *reinterpret_cast<uint4*>(box + lane * 128 + ((q ^ (lane & 7)) << 4)) =
              make_uint4(r[4 * q], r[4 * q + 1], r[4 * q + 2], r[4 * q + 3]);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncwarp();
        if (lane == 0) {
          uint64_t pol;
          asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
          asm volatile(
              "cp.async.bulk.tensor.2d.global.shared::cta.bulk_group.L2::cache_hint [%0, {%1, %2}], [%3], %4;" ::"l"(
                  &p.tma_c),
              "r"(int(n0 + cb * 32)), "r"(int(y0)), "r"(s_u32(box)), "l"(pol)
              : "memory");
          asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
      }
      tc_fence_before();
      asm volatile("bar.sync 1, 128;" ::: "memory");   // the 4 epilogue warps of this CTA read TMEM
      if (ew == 0 && lane == 0) mbar_arrive_remote(tmem_empty0 + b * 8);
      if constexpr (kSlate) {
        if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");   // this warp's C is written
        asm volatile("bar.sync 1, 128;" ::: "memory");
        if (ew == 0 && lane == 0) {
          // the second CTA of the pair to finish counts the tile
          __threadfence();
          uint32_t old;
          asm volatile("atom.acq_rel.cluster.shared::cluster.add.u32 %0, [%1], 1;"
                       : "=r"(old)
                       : "r"(done_cnt0 + b * 4)
                       : "memory");
          if (old & 1u) {
            if (p.cov) atomicAdd(&p.cov[g], 1u);
            count_done(p, 1u, last_of_task ? 1u : 0u);
          }
        }
      }
#else
      const uint32_t row = m0 + crank * BM + ew * 32 + lane;
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
      asm volatile("bar.sync 1, 128;" ::: "memory");   // the 4 epilogue warps of this CTA finished
      if (ew == 0 && lane == 0) {
        mbar_arrive_remote(tmem_empty0 + b * 8);
        if constexpr (kSlate) {
          // the second CTA of the pair to finish counts the tile (its stores and,
          // by the acq_rel atomic, the other CTA's happen before)
          __threadfence();
          uint32_t old;
          asm volatile("atom.acq_rel.cluster.shared::cluster.add.u32 %0, [%1], 1;"
                       : "=r"(old)
                       : "r"(done_cnt0 + b * 4)
                       : "memory");
          if (old & 1u) {
            if (p.cov) atomicAdd(&p.cov[g], 1u);
            count_done(p, 1u, last_of_task ? 1u : 0u);
          }
        }
      }
#endif
      ++t;
    }
    if (SLATE_GEMM_TMA_STORE && lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  __syncthreads();
  cluster_sync();   // no CTA of the pair leaves while the other may still address it
  if (warp == 2) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(kTmemCols) : "memory");
  }
  if constexpr (kSlate) {
    if (warp == 0 && leader) {
      c = __shfl_sync(0xffffffffu, c, 0);
      if (lane == 0) {
        atomicAdd(&p.tc->live_rank[S.rank], 0xffffffffu);
        atomicAdd(&p.tc->live_rank[S.peer_rank], 0xffffffffu);
      }
      if (S.retired) check_shrink_done(p, c, lane);
    }
    // after the shrink bookkeeping; tiles are counted done one by one by the
    // epilogue, so the CTA completing the grid can wait for a top-up's tiles
    if (threadIdx.x == 0) leave_main(p);
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

// a rows x k bf16 K-major matrix, boxes of 128 rows x 64 columns, 128-B swizzle
static bool make_map(CUtensorMap* m, const void* base, uint32_t rows, uint32_t k) {
  EncodeTiledFn enc = encode_fn();
  if (!enc) return false;
  const cuuint64_t dims[2] = {k, rows};
  const cuuint64_t strides[1] = {cuuint64_t(k) * 2};
  const cuuint32_t box[2] = {BK, BM};
  const cuuint32_t estr[2] = {1, 1};
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, estr,
             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// C: m x n fp32 row-major, boxes of 32 x 32, 128-B swizzle (the epilogue's staging layout)
static bool make_map_c(CUtensorMap* m, void* base, uint32_t rows, uint32_t n) {
  EncodeTiledFn enc = encode_fn();
  if (!enc) return false;
  const cuuint64_t dims[2] = {n, rows};
  const cuuint64_t strides[1] = {cuuint64_t(n) * 4};
  const cuuint32_t box[2] = {32, 32};
  const cuuint32_t estr[2] = {1, 1};
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, base, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
             CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) ==
         CUDA_SUCCESS;
}

static cudaError_t fill(Params& p, const void* args) {
  std::memset(&p, 0, sizeof(p));
  std::memcpy(&p.args, args, sizeof(p.args));
  if (!make_map(&p.tma_a, reinterpret_cast<const void*>(p.args.A), p.args.m, p.args.k) ||
      !make_map(&p.tma_b, reinterpret_cast<const void*>(p.args.B), p.args.n, p.args.k) ||
      !make_map_c(&p.tma_c, reinterpret_cast<void*>(p.args.C), p.args.m, p.args.n))
    return cudaErrorInvalidValue;
  return cudaSuccess;
}

static cudaError_t launch_pairs(const void* fn, Params& p, dim3 grid, cudaStream_t st) {
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.gridDim = grid;
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = kSmemBytes;
  cfg.stream = st;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  void* kargs[] = {&p};
  return cudaLaunchKernelExC(&cfg, fn, kargs);
}

static cudaError_t launch_worker(const WorkerCommon& w, const void* args, uint32_t grid, cudaStream_t st) {
  Params p;
  cudaError_t e = fill(p, args);
  if (e != cudaSuccess) return e;
  p.gx = w.gx; p.gy = w.gy; p.B = w.B; p.iters = w.iters; p.occ = w.occ;
  p.bound_lo = w.bound_lo; p.bound_hi = w.bound_hi; p.n_ranks = w.n_ranks;
  p.standby_timeout_ns = w.standby_timeout_ns;
  p.base_epoch = w.base_epoch;
  p.is_topup = w.is_topup;
  p.gate_first = w.gate_first;
  p.ranklog = w.ranklog;
  p.ctrl = w.ctrl; p.tc = w.tc; p.mirror = w.mirror; p.cov = w.cov; p.rank_of = w.rank_of;
  return launch_pairs(reinterpret_cast<const void*>(&gemm_kernel<true>), p, dim3((grid + 1) & ~1u), st);
}

// K(B,T): one cluster (CTA pair) per original block (gx x gy tiles)
static cudaError_t launch_standalone(const void* args, dim3 grid, cudaStream_t st) {
  Params p;
  cudaError_t e = fill(p, args);
  if (e != cudaSuccess) return e;
  p.gx = grid.x; p.gy = grid.y; p.B = grid.x * grid.y;
  return launch_pairs(reinterpret_cast<const void*>(&gemm_kernel<false>), p, dim3(2 * grid.x, grid.y), st);
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
  o.tile_m = gemm::kTileM;
  o.tile_n = gemm::BN;
  o.launch_worker = &gemm::launch_worker;
  o.topup_anytime = true;   // leave_main: the CTA completing the grid waits for every tile
  o.launch_standalone = &gemm::launch_standalone;
  return o;
}

}  // namespace slate
