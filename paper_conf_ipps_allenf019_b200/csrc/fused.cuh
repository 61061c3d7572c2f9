// fused.cuh -- NEXT-1: the fused co-run worker.
//
// Paper: §III-C -- a running kernel shrinks when another
// arrives and "a completed kernel releases its SMs without delay, and the
// remaining kernel seamlessly claims" them; §IV-C -- the three
// exit conditions of a worker.  The separate-kernel build (slate_device.cuh)
// grows a tenant with standby CTAs or a top-up launch; here ONE persistent
// kernel runs both tenants of a co-running pair, so a CTA changes tenant at a
// task boundary and a resize in either direction -- or the grow when one
// tenant drains -- needs no launch and no standby CTA.
//
// Per SM rank the "tenant map" is the two queues' resize words {epoch, lo, hi}
// (the host resizes a fused pair exactly as two separate launches).  At every
// task boundary thread 0 of a CTA reads both words and picks:
//   * the tenant whose range holds its rank and that still has tasks;
//   * else (grow on completion) the other tenant if the first is
//     drained;
//   * else, if both are drained, the CTA exits (exit condition (2));
//   * else it waits (standby) -- ranks outside both ranges.
// The CTA shape is uniform (both tenants' bodies run with the same block of
// kThreads threads; dynamic shared memory is the larger of the two).  Each
// tenant keeps its own TaskCtl (task counter, done counters, live workers per
// rank), so coverage, counters, the rank log and the resize-latency stamps
// are the separate-kernel build's: a switch away from a tenant counts its
// blocks, decrements its live count on this rank and checks whether its
// shrink is complete; a switch to a tenant under a newer epoch publishes the
// grow.
#pragma once
#include "slate_device.cuh"

namespace slate {

template <class TA, class TB>
struct FusedParams {
  WorkerParams<typename TA::Args> a;
  WorkerParams<typename TB::Args> b;
  uint32_t grow_on_drain;   // a drained tenant's SMs go to the other at once
  uint32_t speculative;     // fetch the same tenant's next task during this one (see fused_body)
};

// whole-CTA-free (thread 0) version of check_shrink_done for the fused worker
template <class P>
__device__ __forceinline__ void fused_shrink_check(const P& p, uint64_t c) {
  TaskCtl* tc = p.tc;
  __threadfence();   // our live_rank decrement before the scan
  for (uint32_t r = 0; r < p.n_ranks; ++r)
    if ((r < ctrl_lo(c) || r > ctrl_hi(c)) && ld_relaxed_u32(&tc->live_rank[r]) != 0) return;
  const uint32_t e = ctrl_epoch(c);
  if (atomicMax(&tc->shrink_epoch, e) < e && p.mirror)
    publish_mirror(&tc->shrink_word, &p.mirror->shrink, mirror_pack(e, globaltimer()));
}

template <class P>
__device__ __forceinline__ void fused_join(const P& p, uint32_t rank, uint64_t c) {
  TaskCtl* tc = p.tc;
  atomicAdd(&tc->live_rank[rank], 1u);
  atomicAdd(&tc->started, 1u);
  const uint32_t e = ctrl_epoch(c);
  if (e > p.base_epoch && ld_relaxed_u32(&tc->join_epoch) < e && atomicMax(&tc->join_epoch, e) < e && p.mirror)
    publish_mirror(&tc->join_word, &p.mirror->join, mirror_pack(e, globaltimer()));   // grow observed under e
}

// kRegs: the register budget of the pair's kernel (the fused task body needs >= 64)
template <class Tn, int kRegs, class P>
__device__ __forceinline__ void fused_run_task(const P& p, uint32_t g, char* smem) {
  const uint32_t n = min(p.iters, p.B - g);
  constexpr bool kFusedBody = Tn::kHasFusedTask && kRegs >= 64;
  if constexpr (kFusedBody || Tn::kHasTask) {
    if constexpr (kFusedBody)
      Tn::cta_task_fused(p.args, g, n, smem);
    else
      Tn::cta_task(p.args, g, n, smem);
    if (p.cov && threadIdx.x == 0)
      for (uint32_t i = 0; i < n; ++i) atomicAdd(&p.cov[g + i], 1u);
  } else {
    BlockWalk w;
    w.start(g, p.gx, p.gy);
    for (uint32_t i = 0; i < n; ++i) {
      Tn::cta_block(p.args, w.x, w.y, w.z, smem);
      if (p.cov && threadIdx.x == 0) atomicAdd(&p.cov[g + i], 1u);
      w.advance(p.gx, p.gy);
    }
  }
}

template <class TA, class TB>
__device__ __forceinline__ void fused_body(const FusedParams<TA, TB>& fp) {
  static_assert(TA::kThreads == TB::kThreads, "a fused pair runs both bodies on one CTA shape");
  static_assert(!TA::kHasInit && !TB::kHasInit && !TA::kHasFini && !TB::kHasFini && !TA::kLookahead &&
                    !TB::kLookahead,
                "tenants with per-CTA state (init/fini/lookahead) cannot share a CTA");
  extern __shared__ __align__(128) char dyn_smem[];
  __shared__ uint32_t s_ten, s_g;
  const auto& pa = fp.a;
  const auto& pb = fp.b;
  uint32_t rank = 0;
  int cur = -1;                                  // tenant this CTA works for (thread 0)
  uint64_t c_cur = 0;                            // the resize word it acted on (thread 0)
  uint32_t blocks_a = 0, tasks_a = 0, blocks_b = 0, tasks_b = 0;   // done since the CTA joined the tenant
  if (threadIdx.x == 0) {
    rank = pa.rank_of[smid()];
    if (blockIdx.x == 0) {
      const uint64_t t = globaltimer();
      atomicCAS(&pa.tc->t_enter, 0ull, t);
      atomicCAS(&pb.tc->t_enter, 0ull, t);
    }
  }
  // leave tenant `cur` (its blocks are counted now, so its end is stamped when
  // its last block finishes, not when this CTA exits)
  auto leave = [&]() {
    if (cur < 0) return;
    if (cur == 0) {
      if (blocks_a) count_done(pa, blocks_a, tasks_a);
      atomicAdd(&pa.tc->live_rank[rank], 0xffffffffu);
      fused_shrink_check(pa, ld_acquire_u64(pa.ctrl));
      blocks_a = tasks_a = 0;
    } else {
      if (blocks_b) count_done(pb, blocks_b, tasks_b);
      atomicAdd(&pb.tc->live_rank[rank], 0xffffffffu);
      fused_shrink_check(pb, ld_acquire_u64(pb.ctrl));
      blocks_b = tasks_b = 0;
    }
    cur = -1;
  };
  // the next boundary's inputs -- both resize words and both task counters --
  // are loaded (relaxed) when a task starts, so their round trips overlap the
  // task; a word whose epoch changed is made an acquire by a fence (the
  // generic worker's discipline, slate_device.cuh)
  uint64_t pre_ca = 0, pre_cb = 0;
  uint32_t pre_na = 0, pre_nb = 0, seen_ea = 0, seen_eb = 0;
  auto prefetch = [&]() {
    pre_ca = ld_relaxed_u64(reinterpret_cast<const unsigned long long*>(pa.ctrl));
    pre_cb = ld_relaxed_u64(reinterpret_cast<const unsigned long long*>(pb.ctrl));
    pre_na = ld_relaxed_u32(&pa.tc->next);
    pre_nb = ld_relaxed_u32(&pb.tc->next);
  };
  if (threadIdx.x == 0) {
    pre_ca = ld_acquire_u64(pa.ctrl);
    pre_cb = ld_acquire_u64(pb.ctrl);
    seen_ea = ctrl_epoch(pre_ca);
    seen_eb = ctrl_epoch(pre_cb);
    pre_na = ld_relaxed_u32(&pa.tc->next);
    pre_nb = ld_relaxed_u32(&pb.tc->next);
  }
  uint32_t backoff = 128;
  // speculative boundary (optional): once a task is decided, the counter
  // atomic for the same tenant's next task is issued and its result read at
  // the next boundary, so the round trip overlaps the task (the generic
  // worker's kSpeculative mode); a task fetched that way is always run --
  // fetched means owned -- so a resize is then honoured within two tasks, not
  // one.  Measured (tools/fused_bench.py): no throughput gain on the pairs
  // tried, twice the grow latency; off by default.
  uint32_t spec_g = 0xffffffffu;
  int spec_t = -1;
  uint64_t spec_c = 0;
  // the tenant this CTA should work for now, from the prefetched words and
  // counters: 0 / 1, -1 standby (outside both ranges), -2 exit (both drained);
  // *c the range in force (the tenant's word, or the whole chip when it works
  // for a tenant because the partner drained)
  auto choose = [&](uint64_t* c) -> int {
    const uint64_t ca = pre_ca, cb = pre_cb;
    if (ctrl_epoch(ca) != seen_ea || ctrl_epoch(cb) != seen_eb) {
      asm volatile("fence.acq_rel.gpu;" ::: "memory");   // completes the acquire of the new word
      seen_ea = ctrl_epoch(ca);
      seen_eb = ctrl_epoch(cb);
    }
    const bool da = pre_na >= pa.B, db = pre_nb >= pb.B;
    if (da && db) return -2;                                           // exit (2): both queues drained
    const bool ina = in_range(pa, rank, ca), inb = in_range(pb, rank, cb);
    const uint64_t all_a = pack_ctrl(ctrl_epoch(ca), 0, pa.n_ranks - 1);
    const uint64_t all_b = pack_ctrl(ctrl_epoch(cb), 0, pb.n_ranks - 1);
    if (ina && !da) { *c = ca; return 0; }
    if (inb && !db) { *c = cb; return 1; }
    if (fp.grow_on_drain && da && !db) { *c = all_b; return 1; }       // the drained tenant's SMs
    if (fp.grow_on_drain && db && !da) { *c = all_a; return 0; }
    return -1;
  };
  for (;;) {
    if (threadIdx.x == 0) {
      uint32_t ten = 2, g = 0xffffffffu;
      bool keep = false;
      if (spec_t >= 0 && spec_g < (spec_t == 0 ? pa.B : pb.B)) {
        // a task fetched at the previous boundary: owned, so run it; keep
        // speculating only if this CTA would still choose the same tenant
        ten = uint32_t(spec_t);
        g = spec_g;
        c_cur = spec_c;
        if (ten == 0) log_task(pa, g, rank, c_cur, false);
        else log_task(pb, g, rank, c_cur, false);
        uint64_t c = 0;
        keep = choose(&c) == int(ten);
        if (keep) c_cur = c;
      } else {
        if (spec_t == 0) pre_na = pa.B;   // the speculative fetch found the tenant drained
        if (spec_t == 1) pre_nb = pb.B;
        for (;;) {
          uint64_t c = 0;
          const int want = choose(&c);
          if (want == -2) break;
          if (want == -1) {                                               // outside both ranges: standby
            leave();
            __nanosleep(backoff);
            if (backoff < 2048) backoff <<= 1;
            prefetch();
            continue;
          }
          backoff = 128;
          if (want != cur) {
            leave();
            cur = want;
            if (cur == 0) fused_join(pa, rank, c);
            else fused_join(pb, rank, c);
          }
          c_cur = c;
          // Lst2 (2): the task counter of the chosen tenant
          g = cur == 0 ? atomicAdd(&pa.tc->next, pa.iters) : atomicAdd(&pb.tc->next, pb.iters);
          if (cur == 0 ? g >= pa.B : g >= pb.B) {                        // drained meanwhile: decide again
            prefetch();
            if (cur == 0) pre_na = pa.B;
            else pre_nb = pb.B;
            continue;
          }
          if (cur == 0) log_task(pa, g, rank, c_cur, false);
          else log_task(pb, g, rank, c_cur, false);
          ten = uint32_t(cur);
          keep = true;
          break;
        }
      }
      spec_t = -1;
      if (ten != 2) {
        if (g == 0) (ten == 0 ? pa.tc : pb.tc)->t_first = globaltimer();
        prefetch();                              // the next boundary's words, in flight during the task
        if (keep && fp.speculative) {            // the same tenant's next task, in flight during this one
          spec_t = int(ten);
          spec_c = c_cur;
          spec_g = ten == 0 ? atomicAdd(&pa.tc->next, pa.iters) : atomicAdd(&pb.tc->next, pb.iters);
        }
      }
      s_ten = ten;
      s_g = g;
    }
    __syncthreads();
    const uint32_t ten = s_ten, g = s_g;
    if (ten == 2) break;
    constexpr int kMinB = TA::kMinBlocks < TB::kMinBlocks ? TA::kMinBlocks : TB::kMinBlocks;
    constexpr int kRegs = 65536 / (TA::kThreads * (kMinB > 0 ? kMinB : 1));
    if (ten == 0) fused_run_task<TA, kRegs>(pa, g, dyn_smem);
    else fused_run_task<TB, kRegs>(pb, g, dyn_smem);
    __syncthreads();                             // the task's blocks are done; s_ten / s_g may be rewritten
    if (threadIdx.x == 0) {
      if (ten == 0) {
        blocks_a += min(pa.iters, pa.B - g);
        tasks_a += 1;
      } else {
        blocks_b += min(pb.iters, pb.B - g);
        tasks_b += 1;
      }
    }
  }
  if (threadIdx.x == 0) leave();
}

// the uniform CTA shape's occupancy is the lower of the two tenants' (the
// register budget of the hungrier body): a memory tenant paired with a
// register-heavy compute tenant runs with fewer CTAs -- less memory in flight
// -- than on its own (tools/fused_bench.py)
template <class TA, class TB>
__global__ void __launch_bounds__(TA::kThreads, (TA::kMinBlocks < TB::kMinBlocks ? TA::kMinBlocks : TB::kMinBlocks))
    slate_fused(const __grid_constant__ FusedParams<TA, TB> p) {
  fused_body<TA, TB>(p);
}

}  // namespace slate
