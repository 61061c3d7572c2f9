// spmv_ws.cu -- the slate worker of the CSR SpMV kind, warp-specialised for
// sm_100a (DESIGN.md §5 "SpMV tenant").
//
// What it computes is the original kernel's (tenants.cuh SpmvSeg): a row's
// nonzeros in aligned 16-byte segments, lane q of the row's 4-lane group
// summing segments s0+q, s0+q+4, ... ascending as one fmaf chain, then a xor
// 2, 1 butterfly.  Only where the operands come from differs (shared memory
// here, global memory there), so y is bit-identical to the original kernel's
// (tests/test_gpu_parity.py).
//
// Why a separate worker: the original kernel is bound by the L1 gather of x
// (one 128-B line per lane per instruction: ~1 nonzero per SM clock) and, at
// the co-run's SM share, by the bytes each SM can keep in flight (a register
// pipeline holds ~45 KB per SM; at HBM's loaded latency that is ~25 GB/s per
// SM -- measured, round 2).  Here one CTA per SM runs three roles (the
// structure of the GEMM tenant: the slate protocol lives in a producer warp):
//   * task warp (warp 16) -- the slate worker proper: Lst1 binding and standby
//     (prologue), at every task boundary the resize word (retire, Lst1 P:L185)
//     and the task counter (Lst2 (2) P:L208), taken one task ahead
//     (speculative boundary); then the task's row-pointer slice, loaded by the
//     whole warp into one of four slice buffers, and the bounds of its x window,
//     read off the task's nonzeros: [first column of its first row, last column
//     of its last row] widened to the buffer's capacity (a banded or
//     near-diagonal matrix then finds every column in it; a column outside is
//     read from global memory, so the window decides speed, never the result);
//   * chunk warp (warp 17, lane 0) -- per task the x window (cp.async.bulk,
//     L2 -> shared, two buffers), then the task's nonzeros as chunks of 512 rows
//     (16 original blocks) through a 2-slot ring: columns and values of
//     [rp[r0], rp[r0+256]) by cp.async.bulk (HBM -> shared, evict-first), up to
//     128 KB in flight per SM (two 32-KB copies per chunk: a bulk copy costs
//     the SM's copy engine a fixed ~190 ns, so fewer, larger copies win --
//     256-row chunks in a 4-slot ring: 52.7 us per C2 launch on 74 SMs, 128-row
//     in 8 slots: 68.8, 512-row in 2 slots: 46.6; round 2);
//   * compute warps 0..15 -- per chunk, four passes of 8 rows, 4 lanes per row:
//     one 128-bit shared load of columns and one of values per lane and
//     segment, x from the window.
// The task warp runs up to three tasks ahead of the compute warps and the chunk
// warp keeps up to four chunks in flight, so HBM sees a stream instead of one
// round-trip chain per task.
//
// Resize: the task boundary is where the task warp re-reads the
// resize word; a CTA that left the range stops fetching, its compute warps
// finish the tasks it already holds (at most four), then it retires.  Nothing
// is abandoned, so coverage is exactly-once by construction.
#include <cstring>
#include "kernels.h"
#include "slate_device.cuh"
#include "tenants.cuh"
#include "spmv_ws.cuh"

namespace slate {
namespace spmv {

#ifndef SLATE_SPMV_WARPS
#define SLATE_SPMV_WARPS 16
#endif
constexpr int kComputeWarps = SLATE_SPMV_WARPS;
constexpr int kCompute = 32 * kComputeWarps;
constexpr int kThreads = kCompute + 64;          // + task warp + chunk warp
constexpr int kTaskWarp = kComputeWarps, kChunkWarp = kComputeWarps + 1;
#ifndef SLATE_SPMV_CHUNK_BLOCKS
#define SLATE_SPMV_CHUNK_BLOCKS 16   // 512-row chunks: two 32-KB bulk copies each, four passes per warp (measured best, round 2)
#endif
#ifndef SLATE_SPMV_SLOTS
#define SLATE_SPMV_SLOTS 2
#endif
#ifndef SLATE_SPMV_WIN
#define SLATE_SPMV_WIN 9232         // 1024 rows of a +-4096 band (9216) + alignment slack
#endif
constexpr int kChunkBlocks = SLATE_SPMV_CHUNK_BLOCKS;   // blocks per chunk
constexpr int kChunkRows = 32 * kChunkBlocks;
constexpr int kPassRows = 8;                     // rows per warp pass (4 lanes per row)
constexpr int kPasses = kChunkRows / (kPassRows * kComputeWarps);
static_assert(kPasses * kPassRows * kComputeWarps == kChunkRows, "rows per chunk");
constexpr int kMaxTaskBlocks = 32;               // task-size cap (1024 rows)
constexpr int kSlots = SLATE_SPMV_SLOTS;         // chunk ring depth
constexpr int kCap = kChunkRows * 16 + 8;        // nonzeros per slot (16 per row + alignment)
constexpr int kSlotBytes = 2 * kCap * 4;         // col + val
#ifndef SLATE_SPMV_RPBUFS
#define SLATE_SPMV_RPBUFS 4
#endif
constexpr int kRpBufs = SLATE_SPMV_RPBUFS;       // row-pointer slices: the task warp runs <= kRpBufs-1 tasks ahead
constexpr int kRpInts = 32 * kMaxTaskBlocks + 4; // rp slice of one task (rounded to 16 B)
#ifndef SLATE_SPMV_WINBUFS
#define SLATE_SPMV_WINBUFS 2
#endif
constexpr int kWinBufs = SLATE_SPMV_WINBUFS;
constexpr int kWin = SLATE_SPMV_WIN;              // x window per task (floats)
constexpr int kHdrBytes = 1024;
constexpr int kSmemBytes = kHdrBytes + kSlots * kSlotBytes + kRpBufs * kRpInts * 4 + kWinBufs * kWin * 4;
static_assert(kSmemBytes <= 227 * 1024, "one CTA per SM");
static_assert(kSlotBytes % 16 == 0 && (kRpInts * 4) % 16 == 0 && (kWin * 4) % 16 == 0, "16-B bulk granules");

struct TaskMeta {                 // written by the task warp before its rp arrive
  uint32_t g, n;                  // original blocks [g, g+n); n = 0: stop (sentinel)
  int32_t wlo;                    // x window: columns [wlo, wlo + wlen)
  uint32_t wlen;
};
struct ChunkMeta {                // written by the chunk warp before its slot arrive
  uint32_t tb;                    // rp buffer of the chunk's task; 0xffffffff: stop (sentinel)
  uint32_t wb;                    // x-window buffer of the chunk's task
  uint32_t row0;                  // first row of the chunk within the task
  uint32_t nblk;                  // blocks in the chunk
  int32_t a0;                     // nonzero index of col_s[0] (16-B aligned)
  uint32_t mode;                  // 0 staged, 1 col/val from global memory (the chunk exceeds the slot)
  uint32_t first, last;           // first / last chunk of its task
};
struct Hdr {
  uint64_t slot_full[kSlots], slot_empty[kSlots];
  uint64_t rp_full[kRpBufs], rp_empty[kRpBufs];
  uint64_t win_full[kWinBufs], win_empty[kWinBufs];
  TaskMeta tmeta[kRpBufs];
  ChunkMeta cmeta[kSlots];
  uint32_t go, rank, retired;
  uint64_t ctrl;                  // the resize word last acted on (task warp)
};
static_assert(sizeof(Hdr) <= kHdrBytes, "header");

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
// x is re-read by every task (L2-resident): no evict-first hint
__device__ __forceinline__ void bulk_g2s_keep(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))  // racecheck: mbarrier-ordered
               : "memory");
}

#ifndef SLATE_SPMV_PF
#define SLATE_SPMV_PF 0   // experiment (measured: no gain, profiles/r2_spmv_limits.md)
#endif
__device__ __forceinline__ void bulk_prefetch_l2(const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(src), "r"(bytes) : "memory");
}

#ifdef SLATE_SPMV_TRACE
// development trace (tools/probe/spmv_stream.cu): per CTA < 4 and role, 64 events {t, kind, a, b}
__device__ unsigned long long spmv_trace[4][3][64][4];
__device__ __forceinline__ void trace(int role, uint32_t& n, uint32_t kind, uint32_t a0, uint32_t b0) {
  if (blockIdx.x < 4 && n < 64) {
    unsigned long long* r = spmv_trace[blockIdx.x][role][n++];
    r[0] = globaltimer(); r[1] = kind; r[2] = a0; r[3] = b0;
  }
}
#define TRACE(role, kind, a0, b0) trace(role, tn, kind, a0, b0)
#define TRACE_DECL uint32_t tn = 0
#else
#define TRACE(role, kind, a0, b0)
#define TRACE_DECL
#endif

#ifdef SLATE_SPMV_PROFILE
__device__ long long spmv_prof[148][32][5];   // per CTA, compute warp: {total, wait full, first-chunk waits, compute, chunks}
#endif

struct Smem {
  Hdr* h;
  char* slots;
  char* rpb;
  char* win;
  __device__ __forceinline__ int32_t* col(int s) const { return reinterpret_cast<int32_t*>(slots + s * kSlotBytes); }
  __device__ __forceinline__ float* val(int s) const {
    return reinterpret_cast<float*>(slots + s * kSlotBytes + kCap * 4);
  }
  __device__ __forceinline__ int32_t* rp(int b) const { return reinterpret_cast<int32_t*>(rpb + b * kRpInts * 4); }
  __device__ __forceinline__ float* xw(int b) const { return reinterpret_cast<float*>(win + b * kWin * 4); }
};

// ------------------------------------------------------------------ compute warps
// Rows of one chunk: kPasses passes of 8 rows per compute warp, 4 lanes per
// row; every pass's shared-memory loads are issued before the first FMA.  x
// comes from the task's window, or global memory for a column outside it.
#ifndef SLATE_SPMV_EARLY_RELEASE
#define SLATE_SPMV_EARLY_RELEASE 1
#endif
// Returns true when it already released the slot (arrived on `empty`): a warp
// whose rows all fit their first segment is done with the slot once its
// columns and values are in registers, so the chunk warp can refill the slot
// while the warp still gathers x and accumulates (the gathers are ~55% of the
// chunk's shared-memory work; profiles/r2_spmv_limits.md).
__device__ __forceinline__ bool compute_chunk(const slate_args_spmv& a, const Smem& S, const ChunkMeta& m,
                                              const TaskMeta& tm, int s, int nnz, uint64_t* empty) {
  bool released = false;
  const float* __restrict__ xg = reinterpret_cast<const float*>(a.x);
  const int32_t* rp = S.rp(int(m.tb)) + m.row0;          // rp of the chunk's first row
  const float* xw = S.xw(int(m.wb));
  const int32_t wlo = tm.wlo;
  const uint32_t wlen = tm.wlen;
  const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int q = int(lane & 3);
  const uint32_t row_first = tm.g * 32 + m.row0;        // global row of rp[0]
  const uint32_t nrows = min(m.nblk * 32, a.n_rows - row_first);
  auto xval = [&](int c) -> float {
    const uint32_t d = uint32_t(c - wlo);
    return d < wlen ? xw[d] : __ldg(xg + c);  // racecheck: mbarrier-ordered
  };
  const int csafe = wlen ? wlo : 0;   // a column with a finite x, for the entries outside a row
  constexpr int U = kPasses;
  int lo[U], hi[U];
  float acc[U];
  bool longrow = false;
#pragma unroll
  for (int u = 0; u < U; ++u) {
    const uint32_t lr = (u * kComputeWarps + w) * kPassRows + (lane >> 2);
    const bool in = lr < nrows;
    lo[u] = in ? rp[lr] : 0;  // racecheck: mbarrier-ordered
    hi[u] = in ? rp[lr + 1] : 0;  // racecheck: mbarrier-ordered
    longrow |= ((lo[u] >> 2) + 4) * 4 < hi[u];   // segments past the lane's first
  }
  if (m.mode == 0) {
    const int32_t* col = S.col(s);
    const float* val = S.val(s);
    const int32_t a0 = m.a0;   // the slot holds entries [a0, ...), a0 a multiple of 4
    auto seg = [&](int base) {
      spmvseg::Seg r;
      r.c = *reinterpret_cast<const int4*>(col + (base - a0));  // racecheck: mbarrier-ordered
      r.v = *reinterpret_cast<const float4*>(val + (base - a0));  // racecheck: mbarrier-ordered
      return r;
    };
    spmvseg::Seg sg[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {   // a lane with no entry of its row reads nothing (its offset may be negative)
      const int base = ((lo[u] >> 2) + q) * 4;
      if (base < hi[u]) sg[u] = seg(base);
      else sg[u] = spmvseg::Seg{make_int4(0, 0, 0, 0), make_float4(0.f, 0.f, 0.f, 0.f)};
    }
    if (SLATE_SPMV_EARLY_RELEASE && !__any_sync(0xffffffffu, longrow)) {
      // every lane's slot reads are issued above; the warp barrier orders them
      // before lane 0's release arrive (as at the end of a chunk)
      __syncwarp();
      if ((threadIdx.x & 31) == 0) mbar_arrive(empty);
      released = true;
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int base = ((lo[u] >> 2) + q) * 4;
      acc[u] = spmvseg::fma_seg(0.f, sg[u], base, lo[u], hi[u], csafe, xval);
    }
    if (__any_sync(0xffffffffu, longrow)) {
#pragma unroll
      for (int u = 0; u < U; ++u)   // rows longer than 16: the rest of the chain, still ascending
        for (int base = ((lo[u] >> 2) + q + 4) * 4; base < hi[u]; base += 16)
          acc[u] = spmvseg::fma_seg(acc[u], seg(base), base, lo[u], hi[u], csafe, xval);
    }
  } else {
    // the chunk's nonzeros did not fit the slot: the same chain from global memory
    const int* col = reinterpret_cast<const int*>(a.col);
    const float* val = reinterpret_cast<const float*>(a.val);
#pragma unroll
    for (int u = 0; u < U; ++u) acc[u] = spmvseg::row_tail(0.f, col, val, nnz, lo[u], hi[u], q, 0, csafe, xval);
  }
#pragma unroll
  for (int u = 0; u < U; ++u) {
    const float v = spmvseg::reduce4(acc[u]);
    const uint32_t lr = (u * kComputeWarps + w) * kPassRows + (lane >> 2);
    if (q == 0 && lr < nrows) __stcs(reinterpret_cast<float*>(a.y) + row_first + lr, v);
  }
  return released;
}

// ------------------------------------------------------------------ the worker
__global__ void __launch_bounds__(kThreads, 1) spmv_worker(const __grid_constant__ WorkerParams<slate_args_spmv> p) {
  extern __shared__ __align__(128) char smem_raw[];
  Smem S;
  S.h = reinterpret_cast<Hdr*>(smem_raw);
  S.slots = smem_raw + kHdrBytes;
  S.rpb = S.slots + kSlots * kSlotBytes;
  S.win = S.rpb + kRpBufs * kRpInts * 4;
  Hdr& H = *S.h;
  const slate_args_spmv& a = p.args;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (threadIdx.x == kTaskWarp * 32) {
    for (int i = 0; i < kSlots; ++i) {
      mbar_init(&H.slot_full[i], 1);              // the chunk warp's expect_tx arrive (+ bytes)
      mbar_init(&H.slot_empty[i], kComputeWarps); // every compute warp
    }
    for (int i = 0; i < kRpBufs; ++i) {
      mbar_init(&H.rp_full[i], 32);               // every lane of the task warp (plain loads + stores)
      mbar_init(&H.rp_empty[i], kComputeWarps);   // every compute warp, after the task's last chunk
    }
    for (int i = 0; i < kWinBufs; ++i) {
      mbar_init(&H.win_full[i], 1);               // the chunk warp's expect_tx arrive (+ x bytes)
      mbar_init(&H.win_empty[i], kComputeWarps);
    }
    fence_mbar_init();
    // ---- Lst1: bind to the SM, standby while under-staffed
    const uint32_t r = p.rank_of[smid()];
    uint64_t c = 0;
    H.rank = r;
    H.retired = 0;
    H.go = prologue(p, r, c) ? 1u : 0u;
    H.ctrl = c;
  }
  __syncthreads();
  if (!H.go) {
    if (threadIdx.x == 0) leave_main(p);
    return;
  }
  // a PDL launch: the previous kernel on the stream has completed after this
  // wait.  When that kernel is this one with the same arguments (pdl_early:
  // y overlaps no input, and the previous launch writes y only), the task and
  // chunk warps start on the inputs at once -- the row-pointer slices, the x
  // window and the first chunks are in flight while the previous launch
  // finishes -- and only the compute warps, which write y, wait.
  if (!p.pdl_early || (warp != kTaskWarp && warp != kChunkWarp)) pdl_wait();
  const int nnz = __ldg(reinterpret_cast<const int*>(a.rowptr) + a.n_rows);

  if (warp == kTaskWarp) {
    // ===================== task warp: the slate task protocol + row-pointer slices =====================
    uint64_t c = H.ctrl;
    const uint32_t rank = H.rank;
    __syncwarp();   // every lane has read H.ctrl before lane 0 may rewrite it (the stop sentinel)
    TRACE_DECL;
    // Speculative boundary (as the generic worker's kSpeculative mode): the
    // decision for task t+1 -- retire, or the counter atomic -- is taken when
    // task t's slice is fetched, from the resize word loaded one boundary
    // earlier, so neither round trip sits on the task warp's critical path; a
    // resize is honoured within two task boundaries.
    uint64_t c_pre = c;                   // the resize word for the next boundary (lane 0)
    uint32_t g_next = 0xffffffffu;        // raw counter value fetched for the next task (lane 0)
    bool next_ret = false;
    if (lane == 0) {                      // the first boundary is not speculative
      const bool inr = in_range(p, rank, c);
      if (!inr && try_retire(p.tc)) {
        next_ret = true;
        pdl_trigger();                                                 // this CTA fetches no more
      } else {
        g_next = atomicAdd(&p.tc->next, p.iters);                     // Lst2 (2)
        if (g_next + p.iters >= p.B) pdl_trigger();                   // every task is handed out
        log_task(p, g_next, rank, c, !inr);
      }
      c_pre = ld_acquire_u64(p.ctrl);
    }
    bool prev_valid = false;              // task t-1: slice in shared memory, not yet published
    int prev_b = 0;
    uint32_t prev_g = 0, prev_n = 0;
    int32_t prev_e0 = 0, prev_e1 = 0;
    for (uint32_t t = 0;; ++t) {
      const int b = int(t % kRpBufs);
      uint32_t g = 0xffffffffu, chg = 0;
      if (lane == 0) {
        TRACE(0, 0, t, 0);
        // resolve the fetch taken at the previous boundary
        if (next_ret) {
          H.retired = 1;
        } else if (g_next < p.B) {
          g = g_next;
          TRACE(0, 2, t, g);
          if (g == 0) p.tc->t_first = globaltimer();
        } else {
          atomicAdd(&p.tc->live_pending, ~0ull);                        // drained: live -= 1
        }
        // task boundary for task t+1, taken now
        next_ret = false;
        g_next = 0xffffffffu;
        if (g != 0xffffffffu) {
          chg = ctrl_epoch(c_pre) != ctrl_epoch(c);
          c = c_pre;
          const bool inr = in_range(p, rank, c);
          if (!inr && try_retire(p.tc)) {
            next_ret = true;
            pdl_trigger();
          } else {
            g_next = atomicAdd(&p.tc->next, p.iters);                 // Lst2 (2); result used next round
            if (g_next + p.iters >= p.B) pdl_trigger();
            log_task(p, g_next, rank, c, !inr);
          }
          c_pre = ld_acquire_u64(p.ctrl);
        }
        mbar_wait(&H.rp_empty[b], ((t / kRpBufs) & 1) ^ 1);         // task t-4 fully consumed
        TRACE(0, 1, t, 0);
      }
      g = __shfl_sync(0xffffffffu, g, 0);
      chg = __shfl_sync(0xffffffffu, chg, 0);
      c = __shfl_sync(0xffffffffu, c, 0);
      if (chg) check_shrink_done(p, c, lane);
      // Two tasks in flight (one round trip per task instead of two): this
      // iteration loads task t's row-pointer slice while lane 0 loads the two
      // column indices that bound task t-1's x window (its slice arrived in the
      // previous iteration), then publishes t-1.  Tasks are published in order.
      const uint32_t n = g == 0xffffffffu ? 0u : min(p.iters, p.B - g);
      const uint32_t r0 = g * 32, r1 = g == 0xffffffffu ? r0 : min(r0 + n * 32, a.n_rows);
      const uint32_t cnt = g == 0xffffffffu ? 0u : r1 - r0 + 1, n4 = cnt / 4;
      const int32_t* rpg = reinterpret_cast<const int32_t*>(a.rowptr) + r0;
      int32_t* rps = S.rp(b);
      constexpr int kV = (kRpInts / 4 + 31) / 32;
      int4 v[kV];
#pragma unroll
      for (int k = 0; k < kV; ++k)
        if (lane + 32 * k < n4) v[k] = __ldg(reinterpret_cast<const int4*>(rpg) + lane + 32 * k);
      const bool tail = lane < cnt - n4 * 4;
      const int32_t vt = tail ? __ldg(rpg + n4 * 4 + lane) : 0;
      if (prev_valid) {
        if (lane == 0) {
          // the x window from task t-1's first and last nonzero
          int32_t wlo = 0;
          uint32_t wlen = 0;
          if (prev_e1 > prev_e0) {
            const int32_t* colg = reinterpret_cast<const int32_t*>(a.col);
            const int32_t cf = __ldg(colg + prev_e0), cl = __ldg(colg + prev_e1 - 1);
            const int32_t cmin = min(cf, cl), cmax = max(cf, cl);
            const int32_t ncols = int32_t(a.n_cols);
            const int32_t span = cmax - cmin + 1;
            int32_t lo = span >= kWin ? cmin : cmin - (kWin - span) / 2;
            lo = max(0, min(lo, ncols - kWin)) & ~3;
            wlo = lo;
            // whole granules inside x; columns past the window read global memory
            wlen = uint32_t(max(0, min(kWin, ncols - lo)) & ~3);
          }
          TaskMeta& tp = H.tmeta[prev_b];
          tp.g = prev_g; tp.n = prev_n; tp.wlo = wlo; tp.wlen = wlen;  // racecheck: mbarrier-ordered
        }
        mbar_arrive(&H.rp_full[prev_b]);              // each lane after its stores (count 32)
        prev_valid = false;
      }
      TaskMeta& tm = H.tmeta[b];
      if (g == 0xffffffffu) {
        if (lane == 0) {
          tm.g = 0; tm.n = 0; tm.wlo = 0; tm.wlen = 0;  // racecheck: mbarrier-ordered
          H.ctrl = c;                                 // the word the CTA acted on last
        }
        mbar_arrive(&H.rp_full[b]);                   // sentinel: publishes the stop
        break;
      }
#pragma unroll
      for (int k = 0; k < kV; ++k)
        if (lane + 32 * k < n4) reinterpret_cast<int4*>(rps)[lane + 32 * k] = v[k];  // racecheck: mbarrier-ordered
      if (tail) rps[n4 * 4 + lane] = vt;  // racecheck: mbarrier-ordered
      __syncwarp();
      prev_valid = true;
      prev_b = b;
      prev_g = g;
      prev_n = n;
      prev_e0 = rps[0];
      prev_e1 = rps[r1 - r0];
#if SLATE_SPMV_PF
      {
        // experiment: the task's columns and values into L2 now, up to three
        // tasks before the chunk warp copies them (four lanes, one bulk
        // prefetch each: the two halves of both arrays)
        const int32_t e0 = prev_e0 & ~3, e1 = min((prev_e1 + 3) & ~3, nnz & ~3);
        const int32_t half = ((e1 - e0) / 2) & ~3;
        const int32_t o = e0 + ((lane & 1) ? half : 0);
        const int32_t len = (lane & 1) ? (e1 - e0 - half) : half;
        if (lane < 4 && len > 0)
          bulk_prefetch_l2(lane < 2 ? static_cast<const void*>(reinterpret_cast<const int32_t*>(a.col) + o)
                                    : static_cast<const void*>(reinterpret_cast<const float*>(a.val) + o),
                           uint32_t(len) * 4);
      }
#endif
    }
  } else if (warp == kChunkWarp) {
    // ===================== chunk warp: nonzeros of each task through the slot ring =====================
    if (lane == 0) {
      TRACE_DECL;
      uint32_t q = 0;   // chunks issued
      for (uint32_t t = 0;; ++t) {
        const int b = int(t % kRpBufs), wb = int(t % kWinBufs);
        mbar_wait(&H.rp_full[b], (t / kRpBufs) & 1);
        TRACE(1, 10, t, 0);
        const TaskMeta tm = H.tmeta[b];
        if (tm.n) {                                   // the task's x window (task t-2 is done with the buffer)
          mbar_wait(&H.win_empty[wb], ((t / kWinBufs) & 1) ^ 1);
          mbar_expect_tx(&H.win_full[wb], tm.wlen * 4);
          if (tm.wlen)
            bulk_g2s_keep(S.xw(wb), reinterpret_cast<const float*>(a.x) + tm.wlo, tm.wlen * 4, &H.win_full[wb]);
        }
        const uint32_t nch = tm.n ? (tm.n + kChunkBlocks - 1) / kChunkBlocks : 1;
        for (uint32_t k = 0; k < nch; ++k, ++q) {
          const int s = int(q % kSlots);
          mbar_wait(&H.slot_empty[s], ((q / kSlots) & 1) ^ 1);
          TRACE(1, 11, q, 0);
          ChunkMeta& m = H.cmeta[s];
          if (tm.n == 0) {
            m.tb = 0xffffffffu;  // racecheck: mbarrier-ordered
            mbar_expect_tx(&H.slot_full[s], 0);
            break;
          }
          const uint32_t row0 = k * kChunkRows;
          const uint32_t nblk = min(uint32_t(kChunkBlocks), tm.n - k * kChunkBlocks);
          const uint32_t r0 = tm.g * 32 + row0;
          const uint32_t nrows = min(nblk * 32, a.n_rows - r0);
          const int32_t* rp = S.rp(b) + row0;
          const int32_t e0 = rp[0], e1 = rp[nrows];
          // [a0, a1) in whole 16-B granules; at the end of the matrix the
          // granule past nnz may lie outside the arrays: its entries are loaded
          // by this thread instead
          const bool end = r0 + nrows == a.n_rows;
          const int32_t a0 = e0 & ~3, a1 = end ? (e1 & ~3) : ((e1 + 3) & ~3);
          m.tb = uint32_t(b); m.wb = uint32_t(wb); m.row0 = row0; m.nblk = nblk; m.a0 = a0;  // racecheck: mbarrier-ordered
          m.first = k == 0; m.last = k + 1 == nch;  // racecheck: mbarrier-ordered
          if (max(a1, e1) - a0 > kCap) {
            m.mode = 1;
            mbar_expect_tx(&H.slot_full[s], 0);
          } else {
            m.mode = 0;  // racecheck: mbarrier-ordered
            for (int32_t j = max(a1, a0); j < e1; ++j) {
              S.col(s)[j - a0] = __ldg(reinterpret_cast<const int32_t*>(a.col) + j);
              S.val(s)[j - a0] = __ldg(reinterpret_cast<const float*>(a.val) + j);
            }
            const uint32_t bytes = uint32_t(max(a1 - a0, 0)) * 4;
            mbar_expect_tx(&H.slot_full[s], 2 * bytes);
            if (bytes) {
#ifndef SLATE_SPMV_SPLIT
#define SLATE_SPMV_SPLIT 1   // experiment: each array's chunk as this many bulk copies
#endif
              const uint32_t piece = ((bytes + SLATE_SPMV_SPLIT - 1) / SLATE_SPMV_SPLIT + 15) & ~15u;
              for (uint32_t o = 0; o < bytes; o += piece) {
                const uint32_t nb = min(piece, bytes - o);
                bulk_g2s(reinterpret_cast<char*>(S.col(s)) + o, reinterpret_cast<const char*>(a.col) + uint64_t(a0) * 4 + o,
                         nb, &H.slot_full[s]);
                bulk_g2s(reinterpret_cast<char*>(S.val(s)) + o, reinterpret_cast<const char*>(a.val) + uint64_t(a0) * 4 + o,
                         nb, &H.slot_full[s]);
              }
            }
          }
        }
        if (tm.n == 0) break;
      }
    }
  } else {
    // ===================== compute warps =====================
    uint32_t q = 0, t = 0, my_blocks = 0, my_tasks = 0;
    TRACE_DECL;
#ifdef SLATE_SPMV_PROFILE
    long long pf_wait = 0, pf_first = 0, pf_comp = 0, pf_t0 = clock64();
#endif
    for (;; ++q) {
      const int s = int(q % kSlots);
#ifdef SLATE_SPMV_PROFILE
      long long c0 = clock64();
#endif
      mbar_wait(&H.slot_full[s], (q / kSlots) & 1);
#ifdef SLATE_SPMV_PROFILE
      long long c1 = clock64();
      pf_wait += c1 - c0;
#endif
      if (threadIdx.x == 0) TRACE(2, 20, q, 0);
      const ChunkMeta m = H.cmeta[s];  // racecheck: mbarrier-ordered
      if (m.tb == 0xffffffffu) break;
      const int b = int(m.tb);
      if (m.first) {
        mbar_wait(&H.rp_full[b], (t / kRpBufs) & 1);
        mbar_wait(&H.win_full[m.wb], (t / kWinBufs) & 1);
      }
      const TaskMeta tm = H.tmeta[b];  // racecheck: mbarrier-ordered
      if (threadIdx.x == 0) TRACE(2, 21, q, 0);
#ifdef SLATE_SPMV_PROFILE
      long long c2 = clock64();
      pf_first += c2 - c1;
#endif
      const bool released = compute_chunk(a, S, m, tm, s, nnz, &H.slot_empty[s]);
      __syncwarp();
#ifdef SLATE_SPMV_PROFILE
      pf_comp += clock64() - c2;
#endif
      if (threadIdx.x == 0) TRACE(2, 22, q, 0);
      if (lane == 0) {
        if (!released) mbar_arrive(&H.slot_empty[s]);
        if (m.last) {
          mbar_arrive(&H.rp_empty[b]);
          mbar_arrive(&H.win_empty[m.wb]);
        }
      }
      if (threadIdx.x == 0) {
        my_blocks += m.nblk;
        if (p.cov)
          for (uint32_t i = 0; i < m.nblk; ++i) atomicAdd(&p.cov[tm.g + m.row0 / 32 + i], 1u);
      }
      if (m.last) {
        ++t;
        ++my_tasks;
      }
    }
    if (threadIdx.x == 0 && my_blocks) count_done(p, my_blocks, my_tasks);
#ifdef SLATE_SPMV_PROFILE
    if (lane == 0 && blockIdx.x < 148) {
      long long* o = spmv_prof[blockIdx.x][warp];
      o[0] = clock64() - pf_t0; o[1] = pf_wait; o[2] = pf_first; o[3] = pf_comp; o[4] = q;
    }
#endif
  }
  __syncthreads();
  if (warp == kTaskWarp) {
    if (lane == 0) atomicAdd(&p.tc->live_rank[H.rank], 0xffffffffu);   // live_rank -= 1
    if (H.retired) check_shrink_done(p, H.ctrl, lane);
    if (lane == 0) leave_main(p);   // after the shrink bookkeeping (see slate_device.cuh)
  }
}

// y = [y, y + 4 n_rows) against x and rowptr (col and val: a caller aliasing y
// onto them writes its own matrix and is outside the kind's contract)
static bool outputs_disjoint(const void* args) {
  const slate_args_spmv* a = static_cast<const slate_args_spmv*>(args);
  auto apart = [](uint64_t p0, uint64_t n0, uint64_t p1, uint64_t n1) { return p0 + n0 <= p1 || p1 + n1 <= p0; };
  const uint64_t ny = 4ull * a->n_rows;
  return apart(a->y, ny, a->x, 4ull * a->n_cols) && apart(a->y, ny, a->rowptr, 4ull * (a->n_rows + 1ull));
}

static cudaError_t launch_worker(const WorkerCommon& w, const void* args, uint32_t grid, cudaStream_t st) {
  WorkerParams<slate_args_spmv> p;
  std::memcpy(&p.args, args, sizeof(p.args));
  p.gx = w.gx; p.gy = w.gy; p.gz = w.gz; p.B = w.B; p.iters = w.iters; p.occ = w.occ;
  p.bound_lo = w.bound_lo; p.bound_hi = w.bound_hi; p.n_ranks = w.n_ranks;
  p.standby_timeout_ns = w.standby_timeout_ns;
  p.base_epoch = w.base_epoch;
  p.is_topup = w.is_topup;
  p.gate_first = w.gate_first;
  p.ranklog = w.ranklog;
  p.pdl_early = w.pdl_early;
  p.ctrl = w.ctrl; p.tc = w.tc; p.mirror = w.mirror; p.cov = w.cov; p.rank_of = w.rank_of;
  void* kargs[] = {&p};
  return launch_kernel(reinterpret_cast<const void*>(&spmv_worker), dim3(grid), dim3(kThreads), kargs, kSmemBytes, st,
                       w.pdl);
}

static cudaError_t launch_standalone(const void* args, dim3 grid, cudaStream_t st) {
  slate_args_spmv a;
  std::memcpy(&a, args, sizeof(a));
  void* kargs[] = {&a};
  return cudaLaunchKernel(reinterpret_cast<const void*>(&standalone<SpmvSeg>), grid, dim3(SpmvSeg::kThreads),
                          kargs, 0, st);
}

}  // namespace spmv

KindOps spmv_ws_ops() {
  KindOps o;
  o.worker_fn = reinterpret_cast<const void*>(&spmv::spmv_worker);
  o.standalone_fn = reinterpret_cast<const void*>(&standalone<SpmvSeg>);
  o.threads = spmv::kThreads;
  o.smem = spmv::kSmemBytes;
  o.smem_standalone = 0;
  o.args_size = sizeof(slate_args_spmv);
  o.default_iters = 0;
  o.max_auto_iters = spmv::kMaxTaskBlocks;
  o.max_iters = spmv::kMaxTaskBlocks;        // the task buffer holds the rp slice of <= 32 blocks
  o.tasks_per_worker = 6;
  o.launch_worker = &spmv::launch_worker;
  o.launch_standalone = &spmv::launch_standalone;
  o.topup_anytime = true;   // leave_main: the last main CTA waits for every block
  o.pdl_ok = true;          // griddepcontrol.wait before the first task
  o.pdl_early_ok = true;    // producer warps may start before the wait (y written only, see spmv_worker)
  o.outputs_disjoint = &spmv::outputs_disjoint;
  return o;
}

}  // namespace slate
