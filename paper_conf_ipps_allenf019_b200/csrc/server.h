// server.h -- the single-context Slate server (§IV-A): kernel
// registry, per-session queues with SM ranges, the workload-aware scheduler
// (Tab I selector + split), the resize controller, the completion poller and
// the kernel profile table.  Used in-process by libslate and by the `slated`
// daemon; no torch types, no Python.
#pragma once
#include <atomic>
#include <condition_variable>
#include <cstdint>
#include <deque>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include <cuda_runtime.h>
#include "kernels.h"

namespace slate {

struct KernelEntry {
  uint64_t id;
  slate_kernel_desc desc;
  const KindOps* ops;
  int occ;                      // resident worker CTAs per SM
  std::unique_ptr<KindOps> own_ops;   // a runtime-compiled user kernel's kind (NEXT-3)
};

struct Launch {
  uint64_t id;
  uint32_t queue;
  const KernelEntry* k;
  slate_launch_desc desc;       // args pointer rewritten to `args`
  std::vector<unsigned char> args;
  uint32_t B = 0, iters = 1;
  int state = 0;                // 0 queued, 1 issued, 2 complete
  int slot = -1;                // TaskCtl / mirror slot
  cudaEvent_t ev_start = nullptr;     // recorded before the kernel, or null when chained:
  cudaEvent_t start_after = nullptr;  // the predecessor's end (same stream): this launch starts there
  // batch issue (no events between the kernels of a batch): the batch's first
  // launch (times of members come from device stamps relative to it), the
  // member's index, and the event that ends the batch
  uint64_t batch_first = 0;
  uint32_t batch_idx = 0, batch_n = 0;
  cudaEvent_t batch_end = nullptr;
  std::vector<cudaEvent_t> ev_end;    // kernel ends (main + top-ups), for timing
  std::vector<cudaEvent_t> ev_done;   // all must complete (main + top-ups, after snapshots)
  int error = 0;                      // cudaError_t seen on completion
  bool mirror_complete_seen = false;
  uint32_t n_resizes = 0, n_topups = 0, n_superseded = 0;
  std::vector<double> resize_us;
  std::vector<uint8_t> resize_kind;   // 1 shrink, 2 grow
  unsigned char snapshot[kTaskCtlHeader];   // final TaskCtl header copy
  bool has_snapshot = false;
  bool fused = false;           // one tenant of a fused co-run kernel (NEXT-1): no top-ups; times from device stamps
  double t_issue_us = 0;        // host time of the issue (the watchdog's clock)
  bool watchdog_fired = false;  // ran longer than the watchdog limit: its syncs report an error
};

struct Queue {
  uint32_t id;
  cudaStream_t stream = nullptr;
  // the queue's own stream for its control-block snapshot copies (each waits
  // for a launch's or batch's end): per queue, so one queue's long batch never
  // holds back the completion of another's (a shared copy stream serialised
  // them in issue order: a co-runner's end was observed only after the other
  // job's whole batch, delaying its release and the survivor's grow)
  cudaStream_t snap = nullptr;
  static constexpr int kAux = 8;
  cudaStream_t aux[kAux] = {};  // top-up launches (round robin: a top-up whose workers joined runs
                                // until the launch drains, so top-ups must not queue behind each other)
  uint32_t aux_next = 0;
  cudaEvent_t ev_ctrl = nullptr;  // recorded on the control stream after each write of this queue's word
                                  // (reused: a grow's critical path makes no event create/destroy calls)
  bool ctrl_wait_pending = false; // the queue's stream has not waited for ev_ctrl yet (settle_ctrl)
  uint64_t* d_ctrl = nullptr;   // the resize word {epoch, lo, hi}
  uint32_t epoch = 0, lo = 0, hi = 0;
  bool active = false;          // holds an SM range
  bool explicit_range = false;  // set by a CORUN placement
  bool auto_split = false;      // co-running on a split the selector took (re-taken as work arrives)
  bool low_side = true;         // co-running: this queue holds the low ranks [0, k)
  // ranks the running (front) launch has workers on: its range when it started,
  // widened by top-ups, narrowed by shrinks (workers outside retire).  A queue
  // is never shrunk onto ranks its running launch has no workers on (where a
  // lone last worker would then carry the whole launch).
  uint32_t cov_lo = 1, cov_hi = 0;
  std::deque<uint64_t> pending; // launches waiting for SMs (AUTO/SOLO)
  std::deque<uint64_t> deferred;  // granted SMs but waiting for a control block (stream order)
  std::deque<uint64_t> issued;  // issued, not complete (stream order)
  uint32_t n_fused = 0;         // fused co-run launches (NEXT-1) among `issued`
  std::vector<cudaEvent_t> topup_ends;  // top-ups of the last issued launch: successors wait for all
  std::vector<uint64_t> open_batch;     // issued launches of the current batch, no end event yet
  bool last_op_kernel = false;          // the last op on `stream` is the last issued worker kernel (PDL)
  // resize latencies being measured (Q30): epoch, kind (1 shrink, 2 grow), host
  // t0, and where the result goes (launch id, index in its resize_us)
  // lid: the launch the latency is recorded on; run: the queue's running launch at the call
  struct PendingResize { uint32_t epoch; int kind; double t0_us; uint64_t lid; int idx; uint64_t run = 0; };
  std::vector<PendingResize> pending_resize;
  bool closed = false;
  int first_error = 0;          // the first cudaError_t a launch of this queue completed with
  bool watchdog = false;        // a launch of this queue outlived the watchdog limit
};

struct ProfileEntry {
  slate_profile_t p;
};

class Server {
 public:
  explicit Server(int device);
  ~Server();
  int init(std::string* err);
  // Stops and joins the poller and clock threads (idempotent).  In-process
  // servers live until process exit; this runs from an atexit handler, before
  // the CUDA runtime's own teardown, so no server thread is inside a CUDA call
  // (or has a clock probe kernel waiting on it) while the context is destroyed.
  void stop_threads();
  // Development aid (SLATE_EXIT_TRACE): which of the server's streams still
  // has work after up to `wait_ms` (stderr).
  void report_busy_streams(double wait_ms);

  int num_sms() const { return n_sms_; }
  slate_info info() const;

  uint32_t open_queue();
  int close_queue(uint32_t q, int64_t timeout_us, std::string* err);
  bool busy();   // any queue has launches pending, deferred or issued and not complete

  int register_kernel(const slate_kernel_desc* d, uint64_t* out, std::string* err);
  int register_source(const slate_source_desc* d, uint64_t* out, std::string* err);
  int launch(uint32_t q, uint64_t k, const slate_launch_desc* d, uint64_t* out, std::string* err);
  int launch_n(uint32_t q, uint64_t k, const slate_launch_desc* d, uint32_t n, uint64_t* first, std::string* err);
  int launch_many(uint32_t q, uint32_t n, const uint64_t* ks, const slate_launch_desc* ds, uint64_t* first,
                  std::string* err);
  int resize(uint32_t q, uint64_t l, uint32_t lo, uint32_t hi, std::string* err);
  // NEXT-1: launches da (queue qa) and db (queue qb) as ONE fused worker kernel,
  // B on the top sm_b ranks, A on the rest; both queues must be idle
  int launch_fused(uint32_t qa, uint64_t ka, const slate_launch_desc* da, uint32_t qb, uint64_t kb,
                   const slate_launch_desc* db, uint32_t sm_b, uint64_t* la, uint64_t* lb, std::string* err);
  int set_policy(uint32_t policy, std::string* err);
  int set_split_objective(uint32_t objective, double slack, std::string* err);
  // through_watchdog: wait for the launches to really finish (detach), not only until the watchdog reported
  int sync(uint32_t q, uint64_t l, int64_t timeout_us, std::string* err, bool through_watchdog = false);
  int profile(uint64_t k, const slate_launch_desc* d, uint32_t flags, slate_profile_t* out, std::string* err);
  int query(uint64_t l, slate_launch_info* out, std::string* err);
  bool kernel_kind(uint64_t k, uint32_t* kind) const;
  bool kernel_ptr_fields(uint64_t k, std::vector<size_t>* offs) const;   // a user kernel's pointer parameters

 private:
  // all private helpers are called with mu_ held
  int launch_locked(uint32_t q, uint64_t k, const slate_launch_desc* d, uint64_t* out, std::string* err, bool defer);
  int issue(Launch& L, Queue& Q, std::string* err);
  int issue_now(Launch& L, Queue& Q, std::string* err);
  void drain_deferred(Queue& Q);
  void fail_launch(Launch& L, int code);
  int write_ctrl(Queue& Q, uint32_t lo, uint32_t hi, bool immediate, std::string* err);
  void settle_ctrl(Queue& Q);   // the queue's stream waits for its latest resize-word write
  size_t first_running(const Queue& Q) const;   // index in Q.issued of the first launch not done
  int grow_running(Queue& Q, uint32_t old_lo, uint32_t old_hi, std::string* err);
  int topup(Queue& Q, Launch& R, std::string* err);
  void drop_idle_grow(Queue& Q);
  void close_batch(Queue& Q, cudaEvent_t end, bool closed_by_launch = false);
  void launch_times(const Launch& L, double* start, double* end) const;
  bool batch_more_ = false;
  bool pdl_enabled_ = true;   // SLATE_PDL=0 turns programmatic dependent launch off   // set by the issuing loops: another launch of this queue is issued right after
  void schedule();
  void release(Queue& Q);
  bool curve_of(const Launch& L, std::vector<uint32_t>* sms, std::vector<double>* ms) const;
  uint32_t pair_split(const Launch& LA, const Queue& A, const Launch& LB, const Queue& B, int catA, int catB,
                      double* gain) const;
  // NEXT-4 (Q49): job curve of a queue's head kernel (x its queued launches),
  // a third co-runner's admission, and contiguous SM shares for a group
  bool job_curve(const Queue& Q, std::vector<uint32_t>* sms, std::vector<double>* ms) const;
  bool try_admit_kway();
  void apply_shares(const std::vector<uint32_t>& qids, const std::vector<uint32_t>& shares);
  void resplit();
  void poll_once();
  void poller_main();
  int category_of(const Launch& L) const;
  std::string profile_key(const KernelEntry& k, const slate_launch_desc* d) const;
  int run_timed(const KernelEntry& k, const slate_launch_desc* d, uint32_t lo, uint32_t hi, int reps, double* ms,
                std::string* err);
  double now_us() const;
  // host steady clock <-> device %globaltimer (they drift apart ~30 ppm, linearly)
  int clock_anchor(double* th, double* off);
  void clock_main();
  bool host_to_dev_us(double t_host_us, double* t_dev_us) const;   // t_dev relative to clk_base_ns_
  volatile uint32_t* clk_flag_ = nullptr;
  volatile unsigned long long* clk_stamp_ = nullptr;
  uint32_t* clk_dflag_ = nullptr;
  unsigned long long* clk_dstamp_ = nullptr;
  cudaStream_t clk_stream_ = nullptr;
  unsigned long long clk_base_ns_ = 0;
  mutable std::mutex clk_mu_;
  std::deque<std::pair<double, double>> clk_anchors_;   // (host us, device - host us)
  double clk_a_ = 0, clk_b_ = 0, clk_tref_ = 0;
  std::atomic<bool> clk_stop_{false};
  std::thread clock_;
  bool launch_done_events(Launch& L);
  void track_resize(Launch& R, uint32_t epoch, int kind, double t0);
  unsigned long long unwrap_mirror_ns(unsigned long long w, double t) const;
  void resolve_resizes(Queue& Q, double t_host, const Launch* ended);
  void record_resize(const Queue::PendingResize& pr, unsigned long long done_ns, double t_host);
  int alloc_slot();
  void free_slot(int slot);
  uint32_t auto_iters(uint32_t B, int occ, uint32_t cap, uint32_t per_worker) const;
  uint32_t worker_grid(int occ, uint32_t B, uint32_t iters, bool full_range) const;
  uint32_t choose_iters(const KernelEntry& k, const slate_launch_desc* d, uint32_t B) const;
  double task_budget_us_ = 20.0;
  bool validate(const KernelEntry& k, const slate_launch_desc* d, uint32_t* B, std::string* err) const;
  void work(const KernelEntry& k, const slate_launch_desc* d, double* bytes, double* fp32, double* tc) const;

  int device_;
  int n_sms_ = 0;
  uint32_t max_smid_ = 0;
  uint16_t* d_rank_of_ = nullptr;
  cudaStream_t ctrl_stream_ = nullptr;
  cudaStream_t copy_stream_ = nullptr;
  cudaEvent_t epoch_ev_ = nullptr;
  void* write_value64_ = nullptr;   // cuStreamWriteValue64 (driver entry point)

  // pools
  static constexpr int kSlots = 16384;   // control blocks: a Gaussian elimination at n = 4096 is 8190 launches in one batch
  TaskCtl* d_tc_ = nullptr;
  HostMirror* h_mirror_ = nullptr;
  HostMirror* d_mirror_ = nullptr;
  unsigned char* h_snap_ = nullptr;   // pinned, kSlots * kTaskCtlHeader
  void* h_zero_ = nullptr;            // pinned zeros (TaskCtl reset by DMA, no SM), kZeroRun blocks
  static constexpr int kZeroRun = 256;   // control blocks zeroed by one copy
  static constexpr int kZeroEv = 1024;   // events marking zeroing copies (round robin)
  std::vector<cudaEvent_t> zero_ev_;
  uint32_t zero_ev_next_ = 0;
  std::vector<int> pending_free_;     // freed this poll, zeroed together by flush_free()
  void flush_free();
  std::deque<int> free_slots_;     // FIFO: a freed block is reused as late as possible
  std::vector<cudaEvent_t> slot_zeroed_;   // DMA zeroing of a freed slot, off the critical path
  static constexpr int kQueues = 64;
  uint64_t* d_ctrl_pool_ = nullptr;
  std::vector<int> free_ctrl_;

  double peak_hbm_ = 6650.0, peak_fp32_ = 74400.0, peak_tc_ = 1590.0;
  uint32_t standby_timeout_ns_ = 200000;
  double saturation_frac_ = 0.95;
  uint32_t policy_ = SLATE_POLICY_HYBRID;
  double min_gain_ = 1.05;
  uint32_t split_objective_ = SLATE_SPLIT_MAKESPAN;   // reading Q41 (ANTT opt-in)
  uint32_t max_corun_ = 3;                         // SLATE_MAX_CORUN: co-runners per group (NEXT-4, Q49)
  double split_slack_ = 0.05;

  mutable std::mutex mu_;
  std::condition_variable cv_;       // state changes (completion, activation)
  std::map<uint64_t, std::unique_ptr<KernelEntry>> kernels_;
  std::map<uint32_t, std::unique_ptr<Queue>> queues_;
  std::map<uint64_t, std::unique_ptr<Launch>> launches_;
  // completed launches in completion order: records (and their CUDA events)
  // are kept for slate_query until kKeepFinished newer ones completed, then
  // dropped in bulk (retire_finished), so a long-running slated stays bounded
  std::deque<uint64_t> finished_;
  size_t keep_finished_ = 65536;   // SLATE_KEEP_FINISHED (tests use a small window)
  double watchdog_us_ = 120e6;
  bool pdl_early_enabled_ = true;  // SLATE_PDL_EARLY=0: every worker waits for the previous grid first     // SLATE_WATCHDOG_S: a launch issued longer ago is reported (0: off)
  void retire_finished();
  std::deque<uint32_t> waiting_;     // queues waiting for SMs, FIFO
  std::map<uint32_t, uint32_t> bypassed_;
  std::vector<uint32_t> active_;     // queues holding SMs
  std::map<std::string, ProfileEntry> profiles_;
  uint64_t next_kernel_id_ = 1, next_launch_id_ = 1;
  uint32_t next_queue_id_ = 1;
  bool profiling_ = false;
  bool stop_ = false;
  std::thread poller_;
};

}  // namespace slate
