// kernels.h -- host/device shared layout of the slate control structures and
// the host-side dispatch table over tenant kinds.  No torch types anywhere.
#pragma once
#include "rtc_types.h"
#ifndef __CUDACC_RTC__
#include <string>
#include <vector>
#include "../../include/slate.h"
#endif

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
// Each counter every worker CTA updates has a 128-B line of its own: same-line
// atomics serialise in one L2 slice (tools/probe/launch_cost.cu: ~1 us per
// launch of 1184 CTAs).
struct alignas(128) TaskCtl {
  uint32_t next;                  // slateIdx: next original block to hand out
  uint32_t pad0[31];
  unsigned long long done;        // (tasks_done << 32) | blocks_done
  unsigned long long t_first;     // %globaltimer at the start of the task at block 0
  unsigned long long t_last;      // %globaltimer when blocks_done reached B
  uint32_t shrink_epoch;          // last epoch whose shrink was observed complete
  uint32_t join_epoch;            // last epoch in which a worker joined (grow)
  unsigned long long t_enter;     // %globaltimer at the first worker CTA's entry (launch overhead split)
  unsigned long long t_exit;      // %globaltimer at the last working CTA's exit
  unsigned long long shrink_word; // max mirror_pack(epoch, ns) of completed shrinks (the mirror's source)
  unsigned long long join_word;   // max mirror_pack(epoch, ns) of grow joins
  uint32_t pad1[16];
  unsigned long long live_pending;// (returned tasks << 32) | live worker CTAs: one word, so that
                                  // abandoning a task and retiring is one atomic step (Q28)
  uint32_t pad_l[30];
  uint32_t started;               // workers that joined
  uint32_t main_exited;           // CTAs of the launch's own grid (not top-ups) that left, joined or not
  uint32_t pad_s[30];
  uint32_t live_rank[kMaxRanks];  // live workers per SM rank
  uint32_t ret_head, ret_tail;    // ring of abandoned task starts (+1; 0 = slot empty)
  uint32_t pad2[30];
  uint32_t ret[kMaxRanks];
};
#ifndef __CUDACC_RTC__
static_assert(offsetof(TaskCtl, live_pending) == 256 && offsetof(TaskCtl, started) == 384 &&
              offsetof(TaskCtl, live_rank) == 512, "TaskCtl header lines: next | done.. | live_pending | started");
#endif
constexpr size_t kTaskCtlHeader = 512;   // the part snapshotted to the host at the end

// Per launch, in mapped pinned host memory: what the host poller watches.
// Every event is ONE 8-byte store with no fence: a __threadfence_system()
// before a flag store cost ~4 us per launch (tools/probe/launch_cost.cu),
// paid by the CTA whose exit ends the kernel.  An epoch and its device time
// share one word (mirror_pack); the host restores the time's upper bits.
constexpr int kMirrorNsBits = 44;   // 2^44 ns = 17.6 s of device clock
__host__ __device__ __forceinline__ unsigned long long mirror_pack(uint32_t epoch, unsigned long long ns) {
  return (static_cast<unsigned long long>(epoch) << kMirrorNsBits) | (ns & ((1ull << kMirrorNsBits) - 1));
}
__host__ __device__ __forceinline__ uint32_t mirror_epoch(unsigned long long w) { return uint32_t(w >> kMirrorNsBits); }
struct HostMirror {
  volatile unsigned long long done;   // %globaltimer when every block had run (0: not yet)
  volatile unsigned long long shrink; // mirror_pack(epoch, ns): the last epoch whose shrink completed
  volatile unsigned long long join;   // mirror_pack(epoch, ns): the last epoch in which a worker joined
  uint64_t pad[5];
};

// The second kernel parameter of a runtime-compiled user worker (NEXT-3): every
// WorkerParams field but the user's arguments (the first parameter), in a
// layout both nvcc (host) and NVRTC (the worker) see.
struct UserWorkerCommon {
  uint32_t gx, gy, gz, B, iters, occ;
  uint32_t bound_lo, bound_hi, n_ranks, standby_timeout_ns;
  uint32_t base_epoch, is_topup, gate_first, ranklog;
  const uint64_t* ctrl;
  TaskCtl* tc;
  HostMirror* mirror;
  uint32_t* cov;
  const uint16_t* rank_of;
};

#ifndef __CUDACC_RTC__   // host side (not needed by runtime-compiled user workers)
// Everything a worker launch needs besides the tenant's own arguments.
struct WorkerCommon {
  uint32_t gx, gy, gz, B, iters, occ;
  uint32_t bound_lo, bound_hi, n_ranks, standby_timeout_ns;
  uint32_t base_epoch;   // the queue's epoch at issue (0 for top-ups: every join of theirs is a grow)
  uint32_t is_topup;     // 1: a top-up grid sharing a running launch's counter
  uint32_t gate_first;   // top-up of a launch with no start event: wait until the launch took its first task
  uint32_t ranklog = 0;  // cov holds 2B words: the rank log follows the coverage counts (SLATE_KFLAG_RANKLOG)
  uint32_t pdl_early = 0; // the previous grid of the PDL chain is this kernel with the same args (pdl_early_ok kinds)
  bool pdl = false;      // launch with programmatic stream serialization (the previous op on the stream is
                         // the previous worker of the same batch; the worker waits in griddepcontrol.wait)
  const uint64_t* ctrl;
  TaskCtl* tc;
  HostMirror* mirror;
  uint32_t* cov;
  const uint16_t* rank_of;
  const struct KindOps* ops = nullptr;   // the kind being launched (runtime-compiled kinds read their kernels here)
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
  bool pdl_ok = false;           // the worker calls griddepcontrol.wait before its first task
  // the worker may read its inputs before griddepcontrol.wait when the previous
  // grid is the same kernel with the same arguments and the output overlaps no
  // input (it then writes only what this launch rewrites with the same values)
  bool pdl_early_ok = false;
  bool (*outputs_disjoint)(const void* args) = nullptr;
  bool topup_anytime = false;    // the worker's last main CTA waits for every block (leave_main), so a
                                 // running launch may get a top-up while later launches are queued
  cudaError_t (*launch_worker)(const WorkerCommon&, const void* args, uint32_t grid, cudaStream_t) = nullptr;
  cudaError_t (*launch_standalone)(const void* args, dim3 grid, cudaStream_t) = nullptr;
  // runtime-compiled user kernels (NEXT-3): the original kernel needs its kind
  cudaError_t (*launch_standalone_ops)(const KindOps*, const void* args, dim3 grid, cudaStream_t) = nullptr;
  uint32_t user_threads = 0;     // T of a user kernel
  void* user_ctx = nullptr;      // the loaded user kernels (user_kernels.cu)
  double user_bytes_per_block = 0, user_flops_per_block = 0;
  std::vector<size_t> user_ptr_offsets;   // pointer parameters of a user kernel's argument struct
};

// NEXT-3 (the paper's runtime kernel transformation): scan a user's
// CUDA source for its __global__ kernel and generate the slate worker around it
// (and an original-kernel wrapper over the same body); compile it with NVRTC
// for sm_100a and load it.  Returns false with *err set on failure.
bool transform_user_kernel(const char* src, const char* name, uint32_t bx, uint32_t by, uint32_t bz, uint32_t smem,
                           std::string* out, std::string* err);
// compiled images are cached: *compiled says whether NVRTC ran
bool build_user_kind(const char* src, const char* name, uint32_t bx, uint32_t by, uint32_t bz, uint32_t smem,
                     uint32_t args_size, KindOps* ops, std::string* err, bool* compiled = nullptr);

const KindOps* kind_ops(uint32_t kind);   // nullptr if the kind is not built

// NEXT-1 (fused.cu): one persistent kernel running two tenants (kind_a, kind_b)
bool fused_supported(uint32_t kind_a, uint32_t kind_b);
cudaError_t fused_shape(uint32_t kind_a, uint32_t kind_b, const void** fn, int* threads, int* smem);
cudaError_t launch_fused(uint32_t kind_a, uint32_t kind_b, const WorkerCommon& wa, const void* args_a,
                         const WorkerCommon& wb, const void* args_b, uint32_t grow_on_drain, uint32_t grid,
                         cudaStream_t st);

// cudaLaunchKernel, or with programmatic dependent launch (PDL): the kernel may
// start while the previous kernel on the stream drains, and waits for it in
// griddepcontrol.wait (tools/probe/pdl_cost.cu: ~2 us per back-to-back launch)
inline cudaError_t launch_kernel(const void* fn, dim3 grid, dim3 block, void** args, size_t smem, cudaStream_t st,
                                 bool pdl) {
  if (!pdl) return cudaLaunchKernel(fn, grid, block, args, smem, st);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelExC(&cfg, fn, args);
}
cudaError_t launch_calibrate(uint32_t* out, uint32_t blocks, uint32_t spin_ns, cudaStream_t st);
cudaError_t launch_clock_probe(volatile uint32_t* flag, volatile unsigned long long* stamp, int rounds,
                               cudaStream_t st);

#endif  // __CUDACC_RTC__

}  // namespace slate
