// slate_device.cuh -- the transformed kernel K*(B*,T) for sm_100a.
//
// Paper: Listing 1 (SM binding), Listing 2 (task queue + decode,
// P:L195-231), §III-C (dynamic resizing).
// Design: persistent worker CTAs read %smid -> dense
// rank (reading Q5), check it
// against the queue's resize word {epoch, lo, hi} (one acquire load), pull
// SLATE_ITERS consecutive original blocks from the task counter with ONE
// atomic issued by lane 0 and broadcast by __shfl_sync, decode the task start
// once (one div + one mod per task) and walk the blocks with x++ and
// x->y->z rollover, run the tenant body, and re-check the resize word at every
// task boundary.  Shrink = workers outside the new range
// retire; grow = waiting CTAs join / a top-up launch adds workers on the new
// ranks; progress lives only in the counter.  No relaunch (north star).
#pragma once
#include "rtc_types.h"
#include "kernels.h"

namespace slate {

// Optional per-tenant hooks default to off.
struct TenantBase {
  static constexpr bool kHasInit = false;   // cta_init(smem): once per CTA before the first block
  static constexpr bool kHasTask = false;   // cta_task(args, g, n, smem): task [g, g+n) of a 1-D grid at once
  static constexpr bool kHasFusedTask = false; // cta_task_fused(args, g, n, smem): the task body used inside a
                                               // fused co-run kernel (at the pair's lower occupancy) instead
  static constexpr bool kLookahead = false; // cta_task2(args, g, n, g2, n2, smem): run task [g, g+n) of a
                                            // 1-D grid knowing the CTA's next task [g2, g2+n2) (n2 = 0: none)
  static constexpr uint32_t kMaxIters = 10; // cap of the automatic task size (P:L303 default 10)
  static constexpr int kMinBlocks = 1;      // __launch_bounds__ min blocks per SM of the worker
  static constexpr bool kSpeculative = false; // fetch the next task while this one runs (+registers)
  static constexpr uint32_t kTasksPerWorker = 8; // auto task size aims at >= this many tasks per worker
  static constexpr bool kHasFini = false;   // cta_fini(smem): once per CTA before it exits
  static constexpr bool kLateCtrl = false;  // read the resize word at the boundary, not at task start
};

// ------------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t smid() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t r;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(r));
  return r;
}
__device__ __forceinline__ uint64_t ld_acquire_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_relaxed_u64(const unsigned long long* p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
// a store to mapped host memory, visible to the host without a fence (one 8-byte word)
__device__ __forceinline__ void st_sys_u64(volatile unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// Publish a packed (epoch, ns) event to the host mirror so that the mirror only
// ever moves forward in epoch: the device word takes the max, and a writer
// whose store may have overtaken a newer one re-reads and re-stores until the
// mirror holds the device word's value (two CTAs completing shrinks of
// consecutive epochs may otherwise store in the reverse order).
__device__ __forceinline__ void publish_mirror(unsigned long long* word, volatile unsigned long long* host,
                                               unsigned long long v) {
  unsigned long long cur = atomicMax(word, v);
  cur = cur > v ? cur : v;
  for (int i = 0; i < 4; ++i) {
    st_sys_u64(host, cur);
    const unsigned long long now = ld_relaxed_u64(word);
    if (now == cur) break;
    cur = now;
  }
}
__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

template <class Args>
struct WorkerParams {
  Args args;
  uint32_t gx, gy, gz;            // original grid (gridDim of K)
  uint32_t B;                     // slateMax = gx*gy*gz
  uint32_t iters;                 // SLATE_ITERS
  uint32_t occ;                   // resident CTAs per SM of this worker
  uint32_t bound_lo, bound_hi;    // launch bound (top-up launches), else [0, N-1]
  uint32_t n_ranks;
  uint32_t standby_timeout_ns;
  uint32_t base_epoch;            // resize-word epoch when the launch was issued: a join under a later epoch is a grow
  uint32_t is_topup;              // 1: a top-up grid (grow) sharing a running launch's TaskCtl
  uint32_t gate_first;            // top-up: join only once the launch has taken its first task
  uint32_t ranklog;               // 1: cov holds 2B words, cov[B + b] = the rank log entry of block b
  uint32_t pdl_early;             // 1: the previous grid (PDL) is this kernel with these args: inputs may be read
                                  // before griddepcontrol.wait (kinds that allow it, e.g. SpMV's producer warps)
  const uint64_t* ctrl;           // the queue's resize word
  TaskCtl* tc;
  HostMirror* mirror;             // device alias of the pinned mirror (may be null)
  uint32_t* cov;                  // coverage log u32[B] or null
  const uint16_t* rank_of;        // %smid -> rank
};

// programmatic dependent launch: wait for the previous kernel on the stream
// (no-op for a normal launch).  A worker CTA triggers its dependents
// (griddepcontrol.launch_dependents) once every task of the launch has been
// handed out -- the fetch that returned the last task start, a drained queue,
// or its retirement -- so the next grid of the batch is launched, and its CTAs
// run their prologue, while this grid's last tasks finish (the next grid reads
// no tenant data before griddepcontrol.wait).  Not earlier: round 1 triggered
// at entry, and the next grid's waiting CTAs took the SM slots a top-up of the
// running launch needed (one C4 run stalled 320 ms); once every task is handed
// out a top-up has nothing left to run.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
#ifndef SLATE_EARLY_TRIGGER
#define SLATE_EARLY_TRIGGER 1   // experiment switch: 0 = the next grid of a batch launches when this one completes (measured: C2 32.2-32.5 ms instead of 31.9, C4 shrink tail unchanged)
#endif
__device__ __forceinline__ void pdl_trigger() {
#if SLATE_EARLY_TRIGGER
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
#endif
}

// ------------------------------------------------------------------ decode (Lst2 (4))
struct BlockWalk {
  uint32_t x, y, z;
  __device__ __forceinline__ void start(uint32_t g, uint32_t gx, uint32_t gy) {
    // one division and one modulo per task; z for 3-D grids (Q18)
    const uint32_t yz = g / gx;
    x = g - yz * gx;
    y = yz % gy;
    z = yz / gy;
  }
  __device__ __forceinline__ void advance(uint32_t gx, uint32_t gy) {
    // ++blockID.x with rollover, extended y -> z
    if (++x == gx) {
      x = 0;
      if (++y == gy) { y = 0; ++z; }
    }
  }
};

// ------------------------------------------------------------------ rank log (debug, SLATE_KFLAG_RANKLOG)
// Who took each task: written by the fetching lane when it hands out task
// [g, g+n), one word per block at cov[B + b]: the worker's SM rank, the range
// [lo, hi] of the resize word it acted on (as the host published it; a top-up
// worker is further bound to the ranks it was launched for), and flags --
// bit 0: the worker was outside its range and kept the task only under the
// last-live-worker rule (Q22), bit 7: valid.  Tests check that every
// task ran on a rank inside the range in force ("ensures that the
// kernel only runs on these SMs") and that co-runners' rank sets are disjoint.
__device__ __forceinline__ uint32_t ranklog_entry(uint32_t rank, uint32_t lo, uint32_t hi, bool outside) {
  return (rank & 0xffu) | ((lo & 0xffu) << 8) | ((hi & 0xffu) << 16) | ((0x80u | (outside ? 1u : 0u)) << 24);
}
template <class P>
__device__ __forceinline__ void log_task(const P& p, uint32_t g, uint32_t rank, uint64_t c, bool outside) {
  if (!p.ranklog || !p.cov || g >= p.B) return;
  const uint32_t e = ranklog_entry(rank, ctrl_lo(c), ctrl_hi(c), outside), n = min(p.iters, p.B - g);
  for (uint32_t i = 0; i < n; ++i) p.cov[p.B + g + i] = e;
}

// ------------------------------------------------------------------ bookkeeping
// Latency discipline: every bookkeeping atomic whose result is not needed is a
// fire-and-forget reduction (RED), the resize word for a task boundary is
// loaded when the task STARTS (its latency hides behind the task) and only the
// task-counter atomic is a round trip on the boundary.
template <class P>
__device__ __forceinline__ bool in_range(const P& p, uint32_t rank, uint64_t c) {
  return rank >= ctrl_lo(c) && rank <= ctrl_hi(c) && rank >= p.bound_lo && rank <= p.bound_hi;
}

// Lst1 prologue, by ONE thread for its CTA: returns true if the CTA works.
// An out-of-range CTA waits (standby) while the tenant is under-staffed, so a
// launch cannot burn its grid on SMs it does not own; it leaves once the
// tenant has occ*|range| workers or the queue is drained, and after a timeout
// with zero live workers it runs anyway (liveness).
template <class P>
__device__ bool prologue(const P& p, uint32_t rank, uint64_t& c_out) {
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
    // the counter load first: a relaxed load issued after the acquire would wait
    // for it; this way both round trips (and the caller's rank lookup) overlap
    const uint32_t nxt = ld_relaxed_u32(&tc->next);
    const uint64_t c = ld_acquire_u64(p.ctrl);
    if (nxt >= p.B) return false;                                       // exit (2)
    bool join = in_range(p, rank, c);
    if (!join) {
      const uint32_t live = uint32_t(ld_relaxed_u64(&tc->live_pending));
      const uint32_t target = p.occ * (ctrl_hi(c) - ctrl_lo(c) + 1);
      if (live >= target) return false;                                  // exit (1)
      if (t0 == 0) t0 = globaltimer();
      if (live == 0 && globaltimer() - t0 > p.standby_timeout_ns) join = true;
    }
    if (join) {
      atomicAdd(&tc->live_pending, 1ull);    // results unused: RED, no round trip
      atomicAdd(&tc->live_rank[rank], 1u);
      atomicAdd(&tc->started, 1u);
      const uint32_t e = ctrl_epoch(c);
      if (e > p.base_epoch && ld_relaxed_u32(&tc->join_epoch) < e && atomicMax(&tc->join_epoch, e) < e && p.mirror) {
        publish_mirror(&tc->join_word, &p.mirror->join, mirror_pack(e, globaltimer()));   // grow observed under epoch e
      }
      c_out = c;
      return true;
    }
    __nanosleep(backoff);
    if (backoff < 4096) backoff <<= 1;
  }
}

// Whole warp: after the epoch changed, signal the host when no worker is live
// on a rank outside the new range (end of a shrink).  Called by retiring
// workers and by the first boundary of each worker after an epoch change.
template <class P>
__device__ void check_shrink_done(const P& p, uint64_t c, uint32_t lane) {
  TaskCtl* tc = p.tc;
  __syncwarp();      // lane 0's live_rank decrement happens-before the other lanes' scan
  __threadfence();   // fence.sc: order our live_rank decrement before the scan
  bool busy = false;
  for (uint32_t r = lane; r < p.n_ranks; r += 32)
    if ((r < ctrl_lo(c) || r > ctrl_hi(c)) && ld_relaxed_u32(&tc->live_rank[r]) != 0) busy = true;
  busy = __any_sync(0xffffffffu, busy);
  const uint32_t e = ctrl_epoch(c);
  if (!busy && lane == 0 && atomicMax(&tc->shrink_epoch, e) < e && p.mirror) {
    publish_mirror(&tc->shrink_word, &p.mirror->shrink, mirror_pack(e, globaltimer()));
  }
}

// Retire unless this is the last live worker (liveness rule).  Without a
// give-back this is one fetch-and-add: live -= 1, and if that took the count
// from 1 to 0 the worker was the last and puts its unit back (the transient 0
// is visible only to standby CTAs, which may then join -- a transition the
// protocol allows anyway).  A CAS loop here serialises a mass retirement: with
// N workers leaving at once only one CAS per L2 round trip succeeds, and a
// shrink of half the SMs of a 4-CTA/SM tenant took ~90 us (tools/storm_tenant.py).
// With `give_back` (Q28: retiring and returning the task must be one atomic
// step, so a returned task is never orphaned) it is one fetch-and-add too
// (reading Q50): live -1 and returned +1 in the same word.  A worker that was
// not the last has retired and returned its task (true: the caller publishes
// the task in the ring).  The last one takes the unit back -- returned -1,
// live +1, by CAS, and keeps its task (false) -- unless the returned count is
// already 0: a taker has claimed the unit and waits for its publication, and
// that taker is live, so the worker publishes and leaves (true).  Only the
// last worker ever loops.  Round 2 kept a CAS loop for every give-back, and a
// GEMM shrink of ~60 CTA pairs serialised on it (storm shrink p50 34-42 us
// against 13 us for grows).  Modelled in oracle/protocol.py (Config.faa_abort).
__device__ __forceinline__ bool try_retire(TaskCtl* tc, bool give_back = false) {
  if (!give_back) {
    const unsigned long long old = atomicAdd(&tc->live_pending, ~0ull);   // live -= 1
    if (uint32_t(old) > 1u) return true;
    atomicAdd(&tc->live_pending, 1ull);                                    // the last one stays
    return false;
  }
  const unsigned long long delta = (1ull << 32) - 1ull;                    // live -1, returned +1
  const unsigned long long old = atomicAdd(&tc->live_pending, delta);
  if (uint32_t(old) > 1u) return true;
  unsigned long long v = old + delta;
  while ((v >> 32) != 0) {
    const unsigned long long w = atomicCAS(&tc->live_pending, v, v - delta);   // take it back: live +1, returned -1
    if (w == v) return false;   // the last live worker stays, with its task
    v = w;
  }
  return true;                  // claimed by a live taker: publish it and leave
}

// Q28 returned-task ring (long-task tenants only).  A retiring worker that
// abandons its task first wins try_retire(give_back) and then publishes the
// task start; a fetcher first claims a returned task in the same word and then
// takes the next ring slot, waiting for its publication.
__device__ __forceinline__ void give_back_task(TaskCtl* tc, uint32_t g) {
  const uint32_t t = atomicAdd(&tc->ret_tail, 1u) % kMaxRanks;
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(&tc->ret[t]), "r"(g + 1u) : "memory");
}
// one lane: a returned task if any (0xffffffff if none), or, when the queue is
// drained and none is returned, leave (live -= 1) -- atomically with respect to
// returns, so a returned task can never be orphaned.
__device__ __forceinline__ uint32_t take_returned(TaskCtl* tc, bool drained, bool& leave) {
  leave = false;
  unsigned long long v = ld_relaxed_u64(&tc->live_pending);
  for (;;) {
    if ((v >> 32) != 0) {
      const unsigned long long w = atomicCAS(&tc->live_pending, v, v - (1ull << 32));
      if (w != v) { v = w; continue; }
      const uint32_t h = atomicAdd(&tc->ret_head, 1u) % kMaxRanks;
      uint32_t g1;
      do {
        asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(g1) : "l"(&tc->ret[h]) : "memory");
      } while (g1 == 0);
      tc->ret[h] = 0;
      return g1 - 1u;
    }
    if (!drained) return 0xffffffffu;
    const unsigned long long w = atomicCAS(&tc->live_pending, v, v - 1ull);
    if (w == v) {
      leave = true;
      return 0xffffffffu;
    }
    v = w;
  }
}

// Task boundary, by ONE lane: given the resize word c2 (loaded
// when the finished task started) and the finished task (g_done, n_done; n_done
// = 0 for none), count it done and decide the next task.  Returns the next task
// start or 0xffffffff to leave (retired, or the queue is drained).
template <class P>
__device__ __forceinline__ uint32_t boundary(const P& p, uint32_t rank, uint64_t c2, uint64_t& c, uint32_t g_done,
                                             uint32_t n_done, bool& retired, bool& epoch_changed) {
  TaskCtl* tc = p.tc;
  epoch_changed = ctrl_epoch(c2) != ctrl_epoch(c);
  if (epoch_changed) asm volatile("fence.acq_rel.gpu;" ::: "memory");   // completes the acquire of c2
  c = c2;
  retired = false;
  unsigned long long old = 0;
  // task_done: one 64-bit atomic; its result is needed only to spot the last block
  if (n_done) old = atomicAdd(&tc->done, (1ull << 32) | n_done);
  uint32_t g = 0xffffffffu;
  const bool inr = in_range(p, rank, c2);
  if (!inr && try_retire(tc)) {
    retired = true;
    pdl_trigger();                                                      // this CTA fetches no more
  } else {
    g = atomicAdd(&tc->next, p.iters);                                  // Lst2 (2)
    if (g + p.iters >= p.B) pdl_trigger();                              // every task is handed out
    if (g >= p.B) {                                                     // Q3: nothing to run
      atomicAdd(&tc->live_pending, ~0ull);                               // live -= 1 (RED)
      g = 0xffffffffu;
    } else {
      if (g == 0) tc->t_first = globaltimer();
      log_task(p, g, rank, c2, !inr);
    }
  }
  if (n_done && uint32_t(old) + n_done == p.B) {                        // last block of the launch
    const uint64_t t = globaltimer();
    tc->t_last = t;
    if (p.mirror) st_sys_u64(&p.mirror->done, t);
  }
  return g;
}

// A CTA of the launch's own grid leaves -- every one, worker or not (a CTA
// that finds the queue drained in its prologue too).  The one whose exit
// completes the grid waits until every block of the launch is done: top-up
// CTAs (another stream, grow) may still hold some, and the queue's next
// launch starts when this grid completes (stream order).  Without top-ups the
// blocks are all counted by then and it does not wait.  Modelled in
// oracle/protocol.py (Config.leave_main; counting only joined CTAs was not
// enough: a grid whose CTAs all arrived after a top-up took the last tasks
// completed early).
template <class P>
__device__ __forceinline__ void leave_main(const P& p) {
  if (p.is_topup) return;
  if (atomicAdd(&p.tc->main_exited, 1u) + 1u != gridDim.x) return;
  uint32_t ns = 128;
  while (uint32_t(ld_relaxed_u64(&p.tc->done)) < p.B) {
    __nanosleep(ns);
    if (ns < 2048) ns <<= 1;
  }
}

// one finished task: blocks_done += n, tasks_done += 1; the CTA that
// completes the last block stamps the end and tells the host
template <class P>
__device__ __forceinline__ void count_done(const P& p, uint32_t n, uint32_t tasks = 1) {
  const unsigned long long old = atomicAdd(&p.tc->done, (uint64_t(tasks) << 32) | n);
  if (uint32_t(old) + n == p.B) {
    const uint64_t t = globaltimer();
    p.tc->t_last = t;
    if (p.mirror) st_sys_u64(&p.mirror->done, t);
  }
}

// ------------------------------------------------------------------ the worker
// Tn (tenant) provides: using Args; kThreads; kSmem; optional hooks (TenantBase)
//   __device__ static void cta_block(const Args&, uint32_t x, uint32_t y, uint32_t z, char* smem)
// executed by all kThreads threads of the CTA (may use __syncthreads).
//
// Per task (Lst2): lane 0 of warp 0 makes the boundary decision; warp 0 gets
// the task start by __shfl_sync, the other warps through shared memory and the
// barrier that ends the task (reading Q19).
template <class Tn>
__device__ __forceinline__ void worker_body(const WorkerParams<typename Tn::Args>& p) {
  extern __shared__ __align__(128) char dyn_smem[];
  __shared__ uint32_t s_go;
  __shared__ uint32_t s_g[3];
  __shared__ uint32_t s_retired;
  __shared__ uint32_t s_rank;
  const uint32_t lane = threadIdx.x & 31;
  uint64_t c = 0;    // the resize word last acted on (warp 0)
  uint64_t c2 = 0;   // the resize word for the next boundary, loaded at task start (lane 0 of warp 0)

  // ---- Lst1: the block leader binds the CTA to its SM
  if (threadIdx.x == 0) {
    if (blockIdx.x == 0) atomicCAS(&p.tc->t_enter, 0ull, globaltimer());   // result unused
    const uint32_t r = p.rank_of[smid()];   // in flight together with the prologue's loads
    s_retired = 0;
    s_go = prologue(p, r, c) ? 1u : 0u;
    s_rank = r;
  }
  __syncthreads();
  if (!s_go) {
    if (threadIdx.x == 0) leave_main(p);
    return;
  }
  const uint32_t rank = s_rank;
  c = __shfl_sync(0xffffffffu, c, 0);
  if constexpr (Tn::kHasInit) {
    Tn::cta_init(dyn_smem);
    __syncthreads();
  }

  // boundary by warp 0; ends with the barrier; every thread gets the same start
  auto fetch = [&](int slot, uint32_t g_done, uint32_t n_done) -> uint32_t {
    if (threadIdx.x < 32) {
      uint32_t g = 0, ret = 0, chg = 0;
      if (lane == 0) {
        bool retired, changed;
        g = boundary(p, rank, c2, c, g_done, n_done, retired, changed);
        ret = retired;
        chg = changed;
      }
      g = __shfl_sync(0xffffffffu, g, 0);
      chg = __shfl_sync(0xffffffffu, chg, 0);
      c = __shfl_sync(0xffffffffu, c, 0);
      if (lane == 0) {
        s_g[slot] = g;
        if (ret) s_retired = 1;
      }
      if (chg && g != 0xffffffffu) check_shrink_done(p, c, lane);
    }
    __syncthreads();
    return s_g[slot];
  };
  auto prefetch_ctrl = [&]() {   // the next boundary's resize word, in flight during the task
    // relaxed: an acquire load here would hold back warp 0's body loads for an
    // L2 round trip every task; the acquire is a fence at the boundary instead,
    // taken only when the epoch changed (relaxed load + fence = acquire pattern)
    if (threadIdx.x == 0) c2 = ld_relaxed_u64(reinterpret_cast<const unsigned long long*>(p.ctrl));
  };

  pdl_wait();   // a PDL launch: the previous kernel on the stream has completed from here on
  c2 = c;
  uint32_t g = fetch(0, 0, 0);
  int slot = 0;
  // finished work is counted once per CTA at exit (one atomic per worker, not
  // per task); the CTA whose count completes B stamps the end of the launch
  uint32_t my_blocks = 0, my_tasks = 0;
  while (g != 0xffffffffu) {                      // Lst2 (1): until retreat or an empty queue
    const uint32_t n = min(p.iters, p.B - g);     // clamp the last task
    if constexpr (Tn::kLookahead) {
      // the next task is fetched before this one runs, so the tenant can
      // stream its data in while this task computes
      prefetch_ctrl();
      const uint32_t g2 = fetch(slot ^ 1, 0, 0);
      const uint32_t n2 = g2 == 0xffffffffu ? 0u : min(p.iters, p.B - g2);
      Tn::cta_task2(p.args, g, n, g2, n2, dyn_smem);
      if (p.cov && threadIdx.x == 0)
        for (uint32_t i = 0; i < n; ++i) atomicAdd(&p.cov[g + i], 1u);
      __syncthreads();
      my_blocks += n;
      my_tasks += 1;
      g = g2;
      slot ^= 1;
    } else if constexpr (!Tn::kSpeculative) {
      // the boundary's resize word is in flight during the task; the counter
      // atomic is one round trip at the boundary (fewer live registers than
      // the speculative form below).  Long-task tenants (kLateCtrl) load the
      // word at the boundary instead: one more round trip per task, but a
      // resize is honoured after the running task rather than the next one.
      if constexpr (!Tn::kLateCtrl) prefetch_ctrl();
      if constexpr (Tn::kHasTask) {
        Tn::cta_task(p.args, g, n, dyn_smem);
        if (p.cov && threadIdx.x == 0)
          for (uint32_t i = 0; i < n; ++i) atomicAdd(&p.cov[g + i], 1u);
      } else {
        BlockWalk w;
        w.start(g, p.gx, p.gy);
        for (uint32_t i = 0; i < n; ++i) {
          Tn::cta_block(p.args, w.x, w.y, w.z, dyn_smem);
          if (p.cov && threadIdx.x == 0) atomicAdd(&p.cov[g + i], 1u);
          w.advance(p.gx, p.gy);
        }
      }
      if constexpr (Tn::kLateCtrl) prefetch_ctrl();
      __syncthreads();
      my_blocks += n;
      my_tasks += 1;
      g = fetch(slot ^= 1, 0, 0);
    } else {
      // speculative boundary: the decision for the NEXT task is taken now, from
      // the resize word loaded when the previous task started, and the counter
      // atomic is in flight while this task runs (its result is read at the
      // end).  A resize is therefore honoured within at most two tasks.
      uint32_t fut = 0xffffffffu;
      bool spec_retired = false, spec_changed = false;
      if (threadIdx.x == 0) {
        spec_changed = ctrl_epoch(c2) != ctrl_epoch(c);
        if (spec_changed) asm volatile("fence.acq_rel.gpu;" ::: "memory");
        c = c2;
        const bool inr = in_range(p, rank, c);
        if (!inr && try_retire(p.tc)) {
          spec_retired = true;
          pdl_trigger();
        } else {
          fut = atomicAdd(&p.tc->next, p.iters);                       // Lst2 (2), result used below
          if (fut + p.iters >= p.B) pdl_trigger();
          log_task(p, fut, rank, c, !inr);
        }
        c2 = ld_relaxed_u64(reinterpret_cast<const unsigned long long*>(p.ctrl));   // next boundary
      }
      if constexpr (Tn::kHasTask) {
        Tn::cta_task(p.args, g, n, dyn_smem);     // Lst2 (3)-(5) for a 1-D grid, blocks in flight together
        if (p.cov && threadIdx.x == 0)
          for (uint32_t i = 0; i < n; ++i) atomicAdd(&p.cov[g + i], 1u);
      } else {
        BlockWalk w;
        w.start(g, p.gx, p.gy);
        for (uint32_t i = 0; i < n; ++i) {        // Lst2 (3): the task's blocks, in order
          Tn::cta_block(p.args, w.x, w.y, w.z, dyn_smem);   // Lst2 (5): the user code
          if (p.cov && threadIdx.x == 0) atomicAdd(&p.cov[g + i], 1u);
          w.advance(p.gx, p.gy);                  // Lst2 (4)
        }
      }
      if (threadIdx.x == 0) {
        uint32_t g2 = 0xffffffffu;
        if (!spec_retired) {
          if (fut >= p.B) atomicAdd(&p.tc->live_pending, ~0ull);      // queue drained: live -= 1
          else g2 = fut;
          if (fut == 0) p.tc->t_first = globaltimer();
        } else {
          s_retired = 1;
        }
        s_g[slot ^ 1] = g2;
        s_g[2] = spec_changed ? 1u : 0u;
      }
      __syncthreads();                            // every thread is done with the task
      my_blocks += n;
      my_tasks += 1;
      slot ^= 1;
      g = s_g[slot];
      if (s_g[2] && threadIdx.x < 32) {           // epoch changed: maybe the end of a shrink
        c = __shfl_sync(0xffffffffu, c, 0);
        if (g != 0xffffffffu) check_shrink_done(p, c, lane);
      }
    }
  }
  if constexpr (Tn::kHasFini) Tn::cta_fini(dyn_smem);
  if (threadIdx.x == 0 && my_blocks) {
    count_done(p, my_blocks, my_tasks);
#ifdef SLATE_DIAG_EXIT   // diagnostic only: one more same-line atomic per CTA in the kernel's tail
    atomicMax(&p.tc->t_exit, globaltimer());
#endif
  }
  if (threadIdx.x < 32) {
    c = __shfl_sync(0xffffffffu, c, 0);
    if (lane == 0) atomicAdd(&p.tc->live_rank[rank], 0xffffffffu);   // live_rank -= 1
    if (s_retired) check_shrink_done(p, c, lane);
  }
  // after the shrink bookkeeping: a retired CTA that ends up waiting here for
  // the launch's blocks must not hold up the end of the shrink it retired for
  if (threadIdx.x == 0) leave_main(p);
}

template <class Tn>
__global__ void __launch_bounds__(Tn::kThreads, Tn::kMinBlocks) slate_worker(const __grid_constant__ WorkerParams<typename Tn::Args> p) {
  worker_body<Tn>(p);
}

// The original kernel K(B,T) on the hardware block scheduler: the same body
// code, blockIdx from hardware.  Used for the bit-exact comparison (north
// star) and as the "vanilla CUDA" schedule.
template <class Tn>
__global__ void __launch_bounds__(Tn::kThreads) standalone(const __grid_constant__ typename Tn::Args a) {
  extern __shared__ __align__(128) char dyn_smem[];
  if constexpr (Tn::kHasInit) {
    Tn::cta_init(dyn_smem);
    __syncthreads();
  }
  Tn::cta_block(a, blockIdx.x, blockIdx.y, blockIdx.z, dyn_smem);
  if constexpr (Tn::kHasFini) Tn::cta_fini(dyn_smem);
}

// SM-id calibration probe (K13): every CTA records its %smid.
__global__ void calibrate_kernel(uint32_t* out, uint32_t spin_ns);

}  // namespace slate
