// kernels.h -- host/device shared layout of the slate control structures and
// the host-side dispatch table over tenant kinds.  No torch types anywhere.
#pragma once
#include <cstddef>
#include <cstdint>
#include <cuda_runtime.h>
#include "../../include/slate.h"

namespace slate {

constexpr int kMaxRanks = 256;   // B200 has 148 SMs; calibration checks the bound

// resize word: epoch in the high 32 bits, lo in bits 16..31, hi in bits 0..15
__host__ __device__ __forceinline__ uint64_t pack_ctrl(uint32_t epoch, uint32_t lo, uint32_t hi) {
  return (uint64_t(epoch) << 32) | (uint64_t(lo & 0xffff) << 16) | uint64_t(hi & 0xffff);
}
__host__ __device__ __forceinline__ uint32_t ctrl_epoch(uint64_t c) { return uint32_t(c >> 32); }
__host__ __device__ __forceinline__ uint32_t ctrl_lo(uint64_t c) { return uint32_t(c >> 16) & 0xffff; }
__host__ __device__ __forceinline__ uint32_t ctrl_hi(uint64_t c) { return uint32_t(c) & 0xffff; }

// Per launch, in device memory.  Line 0 holds the task counter alone (the hot
// atomic, slateIdx of Lst2); line 1 the completion counters; then per-rank
// live counts used to detect the end of a shrink.
struct alignas(128) TaskCtl {
  uint32_t next;                  // slateIdx: next original block to hand out
  uint32_t pad0[31];
  unsigned long long done;        // (tasks_done << 32) | blocks_done
  unsigned long long live_pending;// (returned tasks << 32) | live worker CTAs: one word, so that
                                  // abandoning a task and retiring is one atomic step (Q28)
  uint32_t started;               // workers that joined
  uint32_t pad_s;
  unsigned long long t_first;     // %globaltimer at the start of the task at block 0
  unsigned long long t_last;      // %globaltimer when blocks_done reached B
  uint32_t shrink_epoch;          // last epoch whose shrink was observed complete
  uint32_t join_epoch;            // last epoch in which a worker joined (grow)
  uint32_t pad1[20];
  uint32_t live_rank[kMaxRanks];  // live workers per SM rank
  uint32_t ret_head, ret_tail;    // ring of abandoned task starts (+1; 0 = slot empty)
  uint32_t pad2[30];
  uint32_t ret[kMaxRanks];
};
static_assert(offsetof(TaskCtl, live_rank) == 256, "TaskCtl header must stay 256 B (the query snapshot)");
constexpr size_t kTaskCtlHeader = 256;   // the part snapshotted to the host at the end

// Per launch, in mapped pinned host memory: what the host poller watches.
struct HostMirror {
  volatile uint32_t complete;     // 1 once every block has run
  volatile uint32_t shrink_epoch; // epoch whose shrink completed (no live worker outside)
  volatile uint32_t join_epoch;   // epoch in which a worker first joined
  volatile uint32_t pad;
  volatile unsigned long long t_last;
  volatile unsigned long long shrink_ns;
  volatile unsigned long long join_ns;
  uint64_t pad2[3];
};

// Everything a worker launch needs besides the tenant's own arguments.
struct WorkerCommon {
  uint32_t gx, gy, gz, B, iters, occ;
  uint32_t bound_lo, bound_hi, n_ranks, standby_timeout_ns;
  const uint64_t* ctrl;
  TaskCtl* tc;
  HostMirror* mirror;
  uint32_t* cov;
  const uint16_t* rank_of;
};

struct KindOps {
  const void* worker_fn = nullptr;
  const void* standalone_fn = nullptr;
  int threads = 0;
  int smem = 0;              // dynamic smem of the worker
  int smem_standalone = 0;   // dynamic smem of the standalone kernel
  size_t args_size = 0;
  uint32_t default_iters = 0;   // 0: auto (reading Q11)
  uint32_t max_auto_iters = 10; // per-tenant cap of the automatic task size
  uint32_t max_iters = 0;       // largest task size the worker supports (0: any)
  uint32_t tasks_per_worker = 8; // the automatic task size aims at >= this many tasks per worker
  uint32_t tile_m = 0;           // GEMM: output rows per original block
  uint32_t tile_n = 0;           // GEMM: output columns per original block
  cudaError_t (*launch_worker)(const WorkerCommon&, const void* args, uint32_t grid, cudaStream_t) = nullptr;
  cudaError_t (*launch_standalone)(const void* args, dim3 grid, cudaStream_t) = nullptr;
};

const KindOps* kind_ops(uint32_t kind);   // nullptr if the kind is not built
cudaError_t launch_calibrate(uint32_t* out, uint32_t blocks, uint32_t spin_ns, cudaStream_t st);
cudaError_t launch_clock_probe(volatile uint32_t* flag, volatile unsigned long long* stamp, int rounds,
                               cudaStream_t st);

}  // namespace slate
