// spmv_ws.cu -- the slate worker of the CSR SpMV kind, warp-specialised for
// sm_100a (DESIGN.md §5 "SpMV tenant").
//
// What it computes is the original kernel's (tenants.cuh SpmvSeg): a row's
// nonzeros in aligned 16-byte segments, lane q of the row's 4-lane group
// summing segments s0+q, s0+q+4, ... ascending as one fmaf chain, then a xor
// 2, 1 butterfly.  Only where x comes from differs (a shared-memory window
// here, global memory there), so y is bit-identical to the original kernel's
// (tests/test_gpu_parity.py).
//
// Why a separate worker.  Per SM the kernel must move ~136 bytes per row
// (16 nonzeros: 64 B of columns, 64 B of values, rp, y) while gathering 16
// random x values per row.  Gathered from global memory, x costs one L1 tag
// per lane (~1 nonzero per SM clock, the original kernel's bound); gathered
// from a shared-memory window it costs a few bank wavefronts per warp load.
// The columns and values stream through registers by 128-bit loads (one L1
// wavefront per 128 B, no shared-memory round trip), software-pipelined: a
// compute warp has the next group's loads in flight while it computes the
// current group, so each SM keeps ~64 KB in flight -- what HBM needs to run
// near its peak from half the chip (the co-run split).
//
// One CTA per SM, two roles:
//   * task warp (warp 16) -- the slate worker proper: Lst1 binding and standby
//     (prologue), at every task boundary the resize word (retire, Lst1 P:L185)
//     and the task counter (Lst2 (2) P:L208), taken one task ahead
//     (speculative boundary); then the task's row-pointer slice into one of
//     four slice buffers and the task's x window -- [first column of its first
//     row, last column of its last row] widened to the buffer (a banded or
//     near-diagonal matrix then finds every column in it; a column outside is
//     read from global memory, so the window decides speed, never the result)
//     -- by one bulk copy (L2 -> shared, cp.async.bulk) into one of three windows;
//   * compute warps 0..14 -- the 128 passes of 8 rows of a task (4 lanes per
//     row) dealt round-robin, 9 per warp in three groups of three: the columns
//     and values of the next group (this task's, or the next task's first) are
//     loaded while the current group is computed.
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

constexpr int kComputeWarps = 15;                  // + the task warp = 16 warps: 128 registers per thread
constexpr int kThreads = 32 * kComputeWarps + 32;
constexpr int kTaskWarp = kComputeWarps;
constexpr int kMaxTaskBlocks = 32;                 // task-size cap (1024 rows)
constexpr int kTaskRows = 32 * kMaxTaskBlocks;
constexpr int kPassRows = 8;                       // rows per warp pass (4 lanes per row)
constexpr int kTaskPasses = kTaskRows / kPassRows; // 128 passes per task, dealt round-robin to the warps
constexpr int kU = 3;                              // passes per group (loads in flight together)
constexpr int kGroups = (kTaskPasses + kComputeWarps * kU - 1) / (kComputeWarps * kU);   // 3 groups per warp
constexpr int kRpBufs = 4;                         // row-pointer slices: the task warp runs <= 3 tasks ahead
constexpr int kRpInts = kTaskRows + 4;             // rp slice of one task (rounded to 16 B)
constexpr int kWinBufs = 3;                        // the task warp issues windows up to two tasks ahead
constexpr int kWin = 10240;                        // x window per task (floats): 1024 rows of a +-4096 band
constexpr int kHdrBytes = 512;
constexpr int kSmemBytes = kHdrBytes + kRpBufs * kRpInts * 4 + kWinBufs * kWin * 4;
static_assert(kSmemBytes <= 227 * 1024, "one CTA per SM");
static_assert((kRpInts * 4) % 16 == 0 && (kWin * 4) % 16 == 0, "16-B bulk granules");

struct TaskMeta {                 // written by the task warp before its rp arrive
  uint32_t g, n;                  // original blocks [g, g+n); n = 0: stop (sentinel)
  int32_t wlo;                    // x window: columns [wlo, wlo + wlen)
  uint32_t wlen;
};
struct Hdr {
  uint64_t rp_full[kRpBufs], rp_empty[kRpBufs], rp_tx[kRpBufs];
  uint64_t win_full[kWinBufs], win_empty[kWinBufs];
  TaskMeta tmeta[kRpBufs];
  uint32_t go, rank, retired;
  int32_t nnz;
  uint32_t blocks, tasks;         // counted by compute warp 0 (it runs a part of every task the CTA took)
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
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}

struct Smem {
  Hdr* h;
  char* rpb;
  char* win;
  __device__ __forceinline__ int32_t* rp(int b) const { return reinterpret_cast<int32_t*>(rpb + b * kRpInts * 4); }
  __device__ __forceinline__ float* xw(int b) const { return reinterpret_cast<float*>(win + b * kWin * 4); }
};

// one group of kU passes of a compute warp: per lane, its row's first segment
// (loads in flight until compute_group reads them; the row bounds are re-read
// from the task's rp slice then, to keep two groups within the register budget)
struct Group {
  spmvseg::Seg s[kU];
};
__device__ __forceinline__ void row_bounds(const int32_t* rps, uint32_t nrows, uint32_t lr, int& lo, int& hi) {
  const bool in = lr < nrows;
  lo = in ? rps[lr] : 0;
  hi = in ? rps[lr + 1] : 0;
}

// the row (within its task) of lane `lane` in pass u of group `grp` of warp w
__device__ __forceinline__ uint32_t task_row(uint32_t w, uint32_t lane, int grp, int u) {
  return (w + kComputeWarps * uint32_t(grp * kU + u)) * kPassRows + (lane >> 2);
}

// issue the loads of group `grp` of task `tm` (its rp slice `rps`)
__device__ __forceinline__ void load_group(Group& G, const slate_args_spmv& a, const int32_t* rps,
                                           const TaskMeta& tm, uint32_t w, uint32_t lane, int grp, int nnz) {
  const int* __restrict__ col = reinterpret_cast<const int*>(a.col);
  const float* __restrict__ val = reinterpret_cast<const float*>(a.val);
  const uint32_t nrows = min(tm.n * 32u, a.n_rows - tm.g * 32u);
  const int q = int(lane & 3);
#pragma unroll
  for (int u = 0; u < kU; ++u) {
    const uint32_t lr = task_row(w, lane, grp, u);
    int lo, hi;
    row_bounds(rps, nrows, lr, lo, hi);
    const int base = ((lo >> 2) + q) * 4;
    G.s[u] = spmvseg::load(col, val, base, nnz, base < hi);
  }
}

// compute group `grp` of task `tm` with x from window `xw` (columns [wlo, wlo + wlen))
__device__ __forceinline__ void compute_group(const Group& G, const slate_args_spmv& a, const int32_t* rps,
                                              const float* xw, const TaskMeta& tm, uint32_t w, uint32_t lane, int grp,
                                              int nnz) {
  const int* __restrict__ col = reinterpret_cast<const int*>(a.col);
  const float* __restrict__ val = reinterpret_cast<const float*>(a.val);
  const float* __restrict__ xg = reinterpret_cast<const float*>(a.x);
  const int32_t wlo = tm.wlo;
  const uint32_t wlen = tm.wlen;
  auto xval = [&](int c) -> float {
    const uint32_t d = uint32_t(c - wlo);
    return d < wlen ? xw[d] : __ldg(xg + c);
  };
  const uint32_t nrows = min(tm.n * 32u, a.n_rows - tm.g * 32u);
  const int q = int(lane & 3);
  float acc[kU];
  int lo[kU], hi[kU];
  bool longrow = false;
#pragma unroll
  for (int u = 0; u < kU; ++u) {
    row_bounds(rps, nrows, task_row(w, lane, grp, u), lo[u], hi[u]);
    const int base = ((lo[u] >> 2) + q) * 4;
    acc[u] = spmvseg::fma_seg(0.f, G.s[u], base, lo[u], hi[u], xval);
    longrow |= ((lo[u] >> 2) + 4) * 4 < hi[u];   // the row has segments past its first four
  }
  if (__any_sync(0xffffffffu, longrow)) {
#pragma unroll
    for (int u = 0; u < kU; ++u) acc[u] = spmvseg::row_tail(acc[u], col, val, nnz, lo[u], hi[u], q, 1, xval);
  }
#pragma unroll
  for (int u = 0; u < kU; ++u) {
    const float v = spmvseg::reduce4(acc[u]);
    const uint32_t lr = task_row(w, lane, grp, u);
    if (q == 0 && lr < nrows) __stcs(reinterpret_cast<float*>(a.y) + tm.g * 32u + lr, v);
  }
}

// ------------------------------------------------------------------ the worker
__global__ void __launch_bounds__(kThreads, 1) spmv_worker(const __grid_constant__ WorkerParams<slate_args_spmv> p) {
  extern __shared__ __align__(128) char smem_raw[];
  Smem S;
  S.h = reinterpret_cast<Hdr*>(smem_raw);
  S.rpb = smem_raw + kHdrBytes;
  S.win = S.rpb + kRpBufs * kRpInts * 4;
  Hdr& H = *S.h;
  const slate_args_spmv& a = p.args;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (threadIdx.x == kTaskWarp * 32) {
    for (int i = 0; i < kRpBufs; ++i) {
      mbar_init(&H.rp_full[i], 32);               // every lane of the task warp (plain loads + stores)
      mbar_init(&H.rp_empty[i], kComputeWarps);   // every compute warp, after the task
      mbar_init(&H.rp_tx[i], 1);                  // the task warp's expect_tx arrive (+ the slice's bytes)
    }
    for (int i = 0; i < kWinBufs; ++i) {
      mbar_init(&H.win_full[i], 1);               // the task warp's expect_tx arrive (+ x bytes)
      mbar_init(&H.win_empty[i], kComputeWarps);
    }
    fence_mbar_init();
    // ---- Lst1: bind to the SM, standby while under-staffed
    const uint32_t r = p.rank_of[smid()];
    uint64_t c = 0;
    H.rank = r;
    H.retired = 0;
    H.blocks = 0;
    H.tasks = 0;
    H.nnz = __ldg(reinterpret_cast<const int*>(a.rowptr) + a.n_rows);
    H.go = prologue(p, r, c) ? 1u : 0u;
    H.ctrl = c;
  }
  __syncthreads();
  if (!H.go) {
    if (threadIdx.x == 0) leave_main(p);
    return;
  }
  pdl_wait();   // a PDL launch: the previous kernel on the stream has completed from here on
  const int nnz = H.nnz;

  if (warp == kTaskWarp) {
    // ===================== task warp: the slate task protocol, rp slices, x windows =====================
    uint64_t c = H.ctrl;
    const uint32_t rank = H.rank;
    __syncwarp();   // every lane has read H.ctrl before lane 0 may rewrite it (the stop sentinel)
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
      } else {
        g_next = atomicAdd(&p.tc->next, p.iters);                     // Lst2 (2)
        log_task(p, g_next, rank, c, !inr);
      }
      c_pre = ld_acquire_u64(p.ctrl);
    }
    for (uint32_t t = 0;; ++t) {
      const int b = int(t % kRpBufs), wb = int(t % kWinBufs);
      uint32_t g = 0xffffffffu, chg = 0;
      if (lane == 0) {
        // resolve the fetch taken at the previous boundary
        if (next_ret) {
          H.retired = 1;
        } else if (g_next < p.B) {
          g = g_next;
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
          if (!inr && try_retire(p.tc)) next_ret = true;
          else {
            g_next = atomicAdd(&p.tc->next, p.iters);                 // Lst2 (2); result used next round
            log_task(p, g_next, rank, c, !inr);
          }
          c_pre = ld_acquire_u64(p.ctrl);
        }
        mbar_wait(&H.rp_empty[b], ((t / kRpBufs) & 1) ^ 1);         // task t-4 fully consumed
      }
      g = __shfl_sync(0xffffffffu, g, 0);
      chg = __shfl_sync(0xffffffffu, chg, 0);
      c = __shfl_sync(0xffffffffu, c, 0);
      if (chg) check_shrink_done(p, c, lane);
      TaskMeta& tm = H.tmeta[b];
      if (g == 0xffffffffu) {
        if (lane == 0) {
          tm.g = 0; tm.n = 0; tm.wlo = 0; tm.wlen = 0;
          H.ctrl = c;                                 // the word the CTA acted on last
        }
        mbar_arrive(&H.rp_full[b]);                   // sentinel: publishes the stop
        break;
      }
      // rp[r0 .. r1]: whole 16-B granules by one bulk copy (r0 = 32 g is 128-B
      // aligned; no registers hold the slice), the last 1-3 entries by lanes
      const uint32_t n = min(p.iters, p.B - g);
      const uint32_t r0 = g * 32, r1 = min(r0 + n * 32, a.n_rows);
      const uint32_t cnt = r1 - r0 + 1, n4 = cnt / 4;
      const int32_t* rpg = reinterpret_cast<const int32_t*>(a.rowptr) + r0;
      int32_t* rps = S.rp(b);
      if (lane == 0) {
        mbar_expect_tx(&H.rp_tx[b], n4 * 16);
        bulk_g2s_keep(rps, rpg, n4 * 16, &H.rp_tx[b]);
      }
      if (lane < cnt - n4 * 4) rps[n4 * 4 + lane] = __ldg(rpg + n4 * 4 + lane);
      if (lane == 0) mbar_wait(&H.rp_tx[b], (t / kRpBufs) & 1);
      __syncwarp();
      if (lane == 0) {
        // the x window from the task's first and last nonzero
        const int32_t e0 = rps[0], e1 = rps[r1 - r0];
        int32_t wlo = 0;
        uint32_t wlen = 0;
        if (e1 > e0) {
          const int32_t* colg = reinterpret_cast<const int32_t*>(a.col);
          const int32_t cf = __ldg(colg + e0), cl = __ldg(colg + e1 - 1);
          const int32_t cmin = min(cf, cl), cmax = max(cf, cl);
          const int32_t ncols = int32_t(a.n_cols);
          const int32_t span = cmax - cmin + 1;
          int32_t lo = span >= kWin ? cmin : cmin - (kWin - span) / 2;
          lo = max(0, min(lo, ncols - kWin)) & ~3;
          wlo = lo;
          // whole granules inside x; columns past the window read global memory
          wlen = uint32_t(max(0, min(kWin, ncols - lo)) & ~3);
        }
        tm.g = g; tm.n = n; tm.wlo = wlo; tm.wlen = wlen;
        mbar_wait(&H.win_empty[wb], ((t / kWinBufs) & 1) ^ 1);     // task t-3 is done with the window
        mbar_expect_tx(&H.win_full[wb], wlen * 4);
        if (wlen) bulk_g2s_keep(S.xw(wb), reinterpret_cast<const float*>(a.x) + wlo, wlen * 4, &H.win_full[wb]);
      }
      __syncwarp();
      mbar_arrive(&H.rp_full[b]);                     // each lane after its stores (count 32)
    }
  } else {
    // ===================== compute warps: loads of the next group in flight during this one =====================
    // the groups of every task in order -- (t, 0), (t, 1), .., (t + 1, 0), ... --
    // with two register sets alternating statically (the loop body is two steps)
    uint32_t my_blocks = 0, my_tasks = 0;
    struct Item {
      uint32_t t;
      int grp;
      TaskMeta tm;
    };
    // the item after `it` (a new task's first group waits for its slice; n = 0: the stop)
    auto advance = [&](const Item& it) -> Item {
      if (it.grp + 1 < kGroups) return Item{it.t, it.grp + 1, it.tm};
      const uint32_t t1 = it.t + 1;
      mbar_wait(&H.rp_full[t1 % kRpBufs], (t1 / kRpBufs) & 1);
      return Item{t1, 0, H.tmeta[t1 % kRpBufs]};
    };
    auto finish = [&](const Item& it, const Group& G) {
      const int b = int(it.t % kRpBufs), wb = int(it.t % kWinBufs);
      if (it.grp == 0) mbar_wait(&H.win_full[wb], (it.t / kWinBufs) & 1);
      compute_group(G, a, S.rp(b), S.xw(wb), it.tm, warp, lane, it.grp, nnz);
      if (it.grp + 1 == kGroups) {   // the task's last group: its slice and window are free
        __syncwarp();
        if (lane == 0) {
          mbar_arrive(&H.rp_empty[b]);
          mbar_arrive(&H.win_empty[wb]);
          if (warp == 0 && p.cov)
            for (uint32_t i = 0; i < it.tm.n; ++i) atomicAdd(&p.cov[it.tm.g + i], 1u);
        }
        my_blocks += it.tm.n;
        my_tasks += 1;
      }
    };
    mbar_wait(&H.rp_full[0], 0);
    Item cur{0, 0, H.tmeta[0]};
    Group G0, G1;
    if (cur.tm.n) load_group(G0, a, S.rp(0), cur.tm, warp, lane, 0, nnz);
    while (cur.tm.n) {
      Item nx = advance(cur);
      if (nx.tm.n) load_group(G1, a, S.rp(nx.t % kRpBufs), nx.tm, warp, lane, nx.grp, nnz);
      finish(cur, G0);
      cur = nx;
      if (!cur.tm.n) break;
      nx = advance(cur);
      if (nx.tm.n) load_group(G0, a, S.rp(nx.t % kRpBufs), nx.tm, warp, lane, nx.grp, nnz);
      finish(cur, G1);
      cur = nx;
    }
    if (warp == 0 && lane == 0) {
      H.blocks = my_blocks;
      H.tasks = my_tasks;
    }
  }
  __syncthreads();   // every compute warp is done: the CTA's blocks are complete
  if (warp == kTaskWarp) {
    if (lane == 0 && H.blocks) count_done(p, H.blocks, H.tasks);
    if (lane == 0) atomicAdd(&p.tc->live_rank[H.rank], 0xffffffffu);   // live_rank -= 1
    if (H.retired) check_shrink_done(p, H.ctrl, lane);
    if (lane == 0) leave_main(p);   // after the shrink bookkeeping (see slate_device.cuh)
  }
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
  p.ctrl = w.ctrl; p.tc = w.tc; p.mirror = w.mirror; p.cov = w.cov; p.rank_of = w.rank_of;
  void* kargs[] = {&p};
  return launch_kernel(reinterpret_cast<const void*>(&spmv_worker), dim3(grid), dim3(kThreads), kargs, kSmemBytes, st,
                       w.pdl);
}

static cudaError_t launch_standalone(const void* args, dim3 grid, cudaStream_t st) {
  slate_args_spmv a;
  std::memcpy(&a, args, sizeof(a));
  void* kargs[] = {&a};
  return cudaLaunchKernel(reinterpret_cast<const void*>(&standalone<SpmvSeg>), grid, dim3(SpmvSeg::kThreads), kargs,
                          0, st);
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
  return o;
}

}  // namespace slate
