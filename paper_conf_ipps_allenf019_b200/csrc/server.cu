// server.cu -- the single-context Slate server (see server.h).
//
// Paper map: context funnelling and sessions (§IV-A), the profiler
// and profile table, the scheduler triggered by arrival and
// completion of kernels, selection (Tab I), dynamic resizing
// (P:L123-127).  B200 design in DESIGN.md §Runtime.
#include <algorithm>
#include <unordered_set>
#include <chrono>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <sstream>

#include <cuda.h>
#include "server.h"

namespace slate {

typedef CUresult (*WriteValue64Fn)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);

#define CK(call)                                                                   \
  do {                                                                             \
    cudaError_t e_ = (call);                                                       \
    if (e_ != cudaSuccess) {                                                       \
      if (err) *err = std::string(#call) + ": " + cudaGetErrorString(e_);          \
      return SLATE_ECUDA;                                                          \
    }                                                                              \
  } while (0)

static double env_double(const char* name, double dflt) {
  const char* v = std::getenv(name);
  return v && *v ? std::atof(v) : dflt;
}

static uint64_t cdiv(uint64_t a, uint64_t b) { return (a + b - 1) / b; }

// ranks in [a_lo, a_hi] ∩ [b_lo, b_hi] (empty ranges have lo > hi)
static uint32_t overlap(uint32_t a_lo, uint32_t a_hi, uint32_t b_lo, uint32_t b_hi) {
  const uint32_t lo = std::max(a_lo, b_lo), hi = std::min(a_hi, b_hi);
  return lo > hi ? 0u : hi - lo + 1;
}

Server::Server(int device) : device_(device) {}

Server::~Server() { stop_threads(); }

void Server::stop_threads() {
  clk_stop_.store(true);                       // a clock probe in flight is released (clock_anchor)
  if (clock_.joinable()) clock_.join();
  {
    std::lock_guard<std::mutex> g(mu_);
    stop_ = true;
  }
  cv_.notify_all();
  if (poller_.joinable()) poller_.join();
}

void Server::report_busy_streams(double wait_ms) {
  std::vector<std::pair<std::string, cudaStream_t>> ss = {{"ctrl", ctrl_stream_}, {"copy", copy_stream_},
                                                           {"clk", clk_stream_}};
  {
    std::lock_guard<std::mutex> g(mu_);
    for (auto& kv : queues_) {
      const Queue& Q = *kv.second;
      if (Q.closed) continue;
      const std::string q = "q" + std::to_string(Q.id);
      ss.push_back({q + ".stream", Q.stream});
      ss.push_back({q + ".snap", Q.snap});
      for (int i = 0; i < Queue::kAux; ++i) ss.push_back({q + ".aux" + std::to_string(i), Q.aux[i]});
    }
  }
  const double t0 = now_us();
  for (auto& x : ss) {
    if (!x.second) continue;
    cudaError_t e;
    while ((e = cudaStreamQuery(x.second)) == cudaErrorNotReady && now_us() - t0 < wait_ms * 1e3)
      std::this_thread::sleep_for(std::chrono::milliseconds(1));
    if (e != cudaSuccess) fprintf(stderr, "[slate] exit: stream %s busy (%s)\n", x.first.c_str(), cudaGetErrorString(e));
  }
  fprintf(stderr, "[slate] exit: streams checked (%zu)\n", ss.size());
}

double Server::now_us() const {
  return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int Server::init(std::string* err) {
  CK(cudaSetDevice(device_));
  CK(cudaFree(nullptr));
  cudaDeviceProp prop;
  CK(cudaGetDeviceProperties(&prop, device_));
  if (prop.major < 10) {
    if (err) *err = "libslate is built for sm_100a (B200); device is sm_" + std::to_string(prop.major * 10 + prop.minor);
    return SLATE_ECUDA;
  }
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuStreamWriteValue64", &write_value64_, cudaEnableDefault, &q));
  if (!write_value64_) {
    if (err) *err = "cuStreamWriteValue64 not available";
    return SLATE_ECUDA;
  }
  int lo_prio, hi_prio;
  CK(cudaDeviceGetStreamPriorityRange(&lo_prio, &hi_prio));
  CK(cudaStreamCreateWithPriority(&ctrl_stream_, cudaStreamNonBlocking, hi_prio));
  CK(cudaStreamCreateWithPriority(&copy_stream_, cudaStreamNonBlocking, hi_prio));
  CK(cudaEventCreate(&epoch_ev_));
  CK(cudaEventRecord(epoch_ev_, copy_stream_));

  // ---- SM calibration (K13): %smid is a virtual id on sm_100a; rank = order in the sorted set
  {
    const uint32_t blocks = 32u * uint32_t(prop.multiProcessorCount);
    uint32_t* d_ids = nullptr;
    CK(cudaMalloc(&d_ids, blocks * 4));
    if (launch_calibrate(d_ids, blocks, 20000, copy_stream_) != cudaSuccess) {
      if (err) *err = "calibration launch failed";
      return SLATE_ECUDA;
    }
    std::vector<uint32_t> ids(blocks);
    CK(cudaMemcpyAsync(ids.data(), d_ids, blocks * 4, cudaMemcpyDeviceToHost, copy_stream_));
    CK(cudaStreamSynchronize(copy_stream_));
    CK(cudaFree(d_ids));
    std::sort(ids.begin(), ids.end());
    ids.erase(std::unique(ids.begin(), ids.end()), ids.end());
    if (ids.empty() || ids.back() >= 1024 || ids.size() > size_t(kMaxRanks)) {
      if (err) *err = "SM calibration out of bounds";
      return SLATE_ECUDA;
    }
    n_sms_ = int(ids.size());
    max_smid_ = ids.back();
    std::vector<uint16_t> lut(1024, uint16_t(n_sms_ - 1));   // unseen ids: clamp (never expected)
    for (size_t r = 0; r < ids.size(); ++r) lut[ids[r]] = uint16_t(r);
    CK(cudaMalloc(&d_rank_of_, 1024 * sizeof(uint16_t)));
    CK(cudaMemcpy(d_rank_of_, lut.data(), 1024 * sizeof(uint16_t), cudaMemcpyHostToDevice));
  }
  // ---- pools
  CK(cudaMalloc(&d_tc_, sizeof(TaskCtl) * kSlots));
  CK(cudaMemset(d_tc_, 0, sizeof(TaskCtl) * kSlots));
  CK(cudaHostAlloc(reinterpret_cast<void**>(&h_mirror_), sizeof(HostMirror) * kSlots, cudaHostAllocMapped));
  std::memset(reinterpret_cast<void*>(h_mirror_), 0, sizeof(HostMirror) * kSlots);
  CK(cudaHostGetDevicePointer(reinterpret_cast<void**>(&d_mirror_), h_mirror_, 0));
  CK(cudaHostAlloc(reinterpret_cast<void**>(&h_snap_), kTaskCtlHeader * kSlots, cudaHostAllocDefault));
  CK(cudaHostAlloc(&h_zero_, sizeof(TaskCtl) * kZeroRun, cudaHostAllocDefault));
  std::memset(h_zero_, 0, sizeof(TaskCtl) * kZeroRun);
  zero_ev_.resize(kZeroEv);
  for (auto& e : zero_ev_) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  for (int i = 0; i < kSlots; ++i) free_slots_.push_back(i);
  slot_zeroed_.assign(kSlots, nullptr);
  CK(cudaMalloc(&d_ctrl_pool_, 128 * kQueues));
  CK(cudaMemset(d_ctrl_pool_, 0, 128 * kQueues));
  for (int i = kQueues - 1; i >= 0; --i) free_ctrl_.push_back(i);

  {
    CK(cudaHostAlloc((void**)&clk_flag_, 64 * sizeof(uint32_t), cudaHostAllocMapped));
    CK(cudaHostAlloc((void**)&clk_stamp_, 32 * sizeof(unsigned long long), cudaHostAllocMapped));
    CK(cudaHostGetDevicePointer((void**)&clk_dflag_, (void*)clk_flag_, 0));
    CK(cudaHostGetDevicePointer((void**)&clk_dstamp_, (void*)clk_stamp_, 0));
    int lo_prio, hi_prio;
    CK(cudaDeviceGetStreamPriorityRange(&lo_prio, &hi_prio));
    CK(cudaStreamCreateWithPriority(&clk_stream_, cudaStreamNonBlocking, lo_prio));
    // resize latencies use host observation until anchored (and for good with SLATE_CLOCK_SYNC=0)
    if (env_double("SLATE_CLOCK_SYNC", 1.0) != 0.0) clock_ = std::thread([this] { clock_main(); });
  }
  peak_hbm_ = env_double("SLATE_PEAK_HBM_GBPS", 6650.0);
  peak_fp32_ = env_double("SLATE_PEAK_FP32_GFLOPS", 2.0 * 128 * prop.multiProcessorCount * (prop.clockRate / 1e6));
  peak_tc_ = env_double("SLATE_PEAK_TC_TFLOPS", 1590.0);
  standby_timeout_ns_ = uint32_t(env_double("SLATE_STANDBY_TIMEOUT_US", 200.0) * 1000.0);
  keep_finished_ = size_t(std::max(16.0, env_double("SLATE_KEEP_FINISHED", 65536.0)));
  pdl_early_enabled_ = env_double("SLATE_PDL_EARLY", 1.0) != 0.0;
  watchdog_us_ = env_double("SLATE_WATCHDOG_S", 120.0) * 1e6;
  saturation_frac_ = env_double("SLATE_SATURATION_FRAC", 0.95);   // reading Q29 (1.0: no cap)
  if (const char* pol = std::getenv("SLATE_POLICY")) {              // reading Q31
    const std::string v(pol);
    policy_ = v == "table" ? SLATE_POLICY_TABLE : v == "literal" ? SLATE_POLICY_LITERAL : SLATE_POLICY_HYBRID;
  }
  {
    pdl_enabled_ = env_double("SLATE_PDL", 1.0) != 0.0;
    task_budget_us_ = env_double("SLATE_TASK_BUDGET_US", 20.0);
  }
  min_gain_ = env_double("SLATE_MIN_GAIN", 1.05);
  if (const char* o = std::getenv("SLATE_SPLIT_OBJECTIVE"))
    split_objective_ = std::string(o) == "antt" ? SLATE_SPLIT_ANTT : SLATE_SPLIT_MAKESPAN;
  split_slack_ = env_double("SLATE_SPLIT_SLACK", 0.05);
  max_corun_ = uint32_t(std::max(2.0, std::min(4.0, env_double("SLATE_MAX_CORUN", 3.0))));
  poller_ = std::thread([this] { poller_main(); });
  return SLATE_OK;
}

// host <-> device clock: a mapped-memory ping-pong gives one
// anchor -- the smallest (device stamp - host raise time) over 32 rounds, i.e.
// the offset plus the one-way host->device latency (< 1 us).  %globaltimer
// drifts against the host's steady clock at a constant rate (measured ~ -33 ppm,
// tools/probe/clock_drift.cu), so a background thread keeps re-anchoring and the
// mapping is a least-squares line through the recent anchors.  Resize latencies
// are device completion stamps minus the host's resize call mapped through it.
int Server::clock_anchor(double* th_out, double* off_out) {
  const int rounds = 32;
  for (int i = 0; i < 2 * rounds; ++i) clk_flag_[i] = 0;
  for (int i = 0; i < rounds; ++i) clk_stamp_[i] = 0;
  if (launch_clock_probe(clk_dflag_, clk_dstamp_, rounds, clk_stream_) != cudaSuccess) return SLATE_ECUDA;
  double best = 1e300, th_best = 0;
  bool ok = true;
  for (int i = 0; i < rounds && ok; ++i) {
    // the probe may wait behind persistent workers for a free CTA slot
    const double t_wait = now_us();
    uint32_t spins = 0;
    while (clk_flag_[2 * i + 1] == 0 && clk_stamp_[i] == 0) {
      if (clk_stop_.load() || now_us() - t_wait > 200e3) { ok = false; break; }
      if (++spins > 1000) std::this_thread::sleep_for(std::chrono::microseconds(20));
    }
    if (!ok) break;
    const double th = now_us();
    clk_flag_[2 * i] = 1;
    while (clk_stamp_[i] == 0) {
      if (now_us() - th > 50e3) { ok = false; break; }
    }
    if (!ok || clk_stamp_[i] == 1ull) { ok = false; break; }   // the probe timed out
    if (!clk_base_ns_) clk_base_ns_ = clk_stamp_[i];
    const double off = double(int64_t(clk_stamp_[i] - clk_base_ns_)) * 1e-3 - th;
    if (off < best) {
      best = off;
      th_best = th;
    }
  }
  if (!ok)
    for (int j = 0; j < 2 * rounds; ++j) clk_flag_[j] = 1;   // let the probe finish
  if (cudaStreamSynchronize(clk_stream_) != cudaSuccess || !ok) return SLATE_ECUDA;
  *th_out = th_best;
  *off_out = best;
  return SLATE_OK;
}

bool Server::host_to_dev_us(double t, double* out) const {
  std::lock_guard<std::mutex> g(clk_mu_);
  if (clk_anchors_.empty()) return false;
  *out = t + clk_a_ + clk_b_ * (t - clk_tref_);
  return true;
}

void Server::clock_main() {
  cudaSetDevice(device_);
  int n = 0, fails = 0;
  while (!clk_stop_.load()) {
    double th, off;
    if (clock_anchor(&th, &off) != SLATE_OK) {
      if (++fails > 8) return;   // e.g. under a kernel-replaying profiler: keep host-observed latencies
    } else {
      std::lock_guard<std::mutex> g(clk_mu_);
      clk_anchors_.emplace_back(th, off);
      if (clk_anchors_.size() > 24) clk_anchors_.pop_front();
      double mt = 0, mo = 0;
      for (auto& a : clk_anchors_) {
        mt += a.first;
        mo += a.second;
      }
      mt /= clk_anchors_.size();
      mo /= clk_anchors_.size();
      double sxx = 0, sxy = 0;
      for (auto& a : clk_anchors_) {
        sxx += (a.first - mt) * (a.first - mt);
        sxy += (a.first - mt) * (a.second - mo);
      }
      clk_tref_ = mt;
      clk_a_ = mo;
      clk_b_ = sxx > 0 ? sxy / sxx : 0.0;
      if (std::getenv("SLATE_DEBUG"))
        fprintf(stderr, "[slate] clock anchor %d: off %.3f us, drift %.2f ppm\n", n, off, clk_b_ * 1e6);
    }
    ++n;
    // dense anchors first (the drift rate), then a slow refresh
    const int wait_ms = n < 8 ? 50 : 250;
    for (int i = 0; i < wait_ms && !clk_stop_.load(); i += 10)
      std::this_thread::sleep_for(std::chrono::milliseconds(10));
  }
}

slate_info Server::info() const {
  slate_info i{};
  i.abi_version = SLATE_ABI_VERSION;
  i.num_sms = uint32_t(n_sms_);
  i.max_smid = max_smid_;
  i.device = uint32_t(device_);
  i.peak_hbm_gbps = peak_hbm_;
  i.peak_fp32_gflops = peak_fp32_;
  i.peak_tc_tflops = peak_tc_;
  return i;
}

// ------------------------------------------------------------------ queues
uint32_t Server::open_queue() {
  std::lock_guard<std::mutex> g(mu_);
  if (free_ctrl_.empty()) return 0;
  auto Q = std::make_unique<Queue>();
  Q->id = next_queue_id_++;
  const int slot = free_ctrl_.back();
  free_ctrl_.pop_back();
  Q->d_ctrl = d_ctrl_pool_ + slot * 16;
  Q->lo = 0;
  Q->hi = uint32_t(n_sms_ - 1);
  cudaStreamCreateWithFlags(&Q->stream, cudaStreamNonBlocking);
  {
    int lo_prio = 0, hi_prio = 0;
    cudaDeviceGetStreamPriorityRange(&lo_prio, &hi_prio);
    cudaStreamCreateWithPriority(&Q->snap, cudaStreamNonBlocking, hi_prio);
  }
  for (cudaStream_t& a : Q->aux) cudaStreamCreateWithFlags(&a, cudaStreamNonBlocking);   // not on the resize path
  cudaEventCreateWithFlags(&Q->ev_ctrl, cudaEventDisableTiming);
  const uint32_t id = Q->id;
  queues_[id] = std::move(Q);
  return id;
}

bool Server::busy() {
  std::lock_guard<std::mutex> g(mu_);
  for (const auto& kv : queues_) {
    const Queue& Q = *kv.second;
    if (!Q.issued.empty() || !Q.pending.empty() || !Q.deferred.empty()) return true;
  }
  return false;
}

int Server::close_queue(uint32_t q, int64_t timeout_us, std::string* err) {
  const int rc = sync(q, 0, timeout_us, err, true);   // until every launch really finished
  std::lock_guard<std::mutex> g(mu_);
  auto it = queues_.find(q);
  if (it == queues_.end()) return SLATE_ENOTFOUND;
  Queue& Q = *it->second;
  Q.closed = true;
  if (rc == SLATE_OK) {
    cudaStreamSynchronize(Q.stream);
    for (cudaStream_t a : Q.aux)
      if (a) cudaStreamSynchronize(a);
    cudaStreamSynchronize(Q.snap);
    const int slot = int((Q.d_ctrl - d_ctrl_pool_) / 16);
    free_ctrl_.push_back(slot);
    cudaStreamDestroy(Q.stream);
    cudaStreamDestroy(Q.snap);
    if (Q.ev_ctrl) cudaEventDestroy(Q.ev_ctrl);
    for (cudaStream_t a : Q.aux)
      if (a) cudaStreamDestroy(a);
    // a queue can still hold SMs with nothing issued (a resize after its last
    // launch completed activates it): give them back before it goes away, and
    // leave no reference to it in the scheduler's lists
    if (Q.active) release(Q);
    waiting_.erase(std::remove(waiting_.begin(), waiting_.end(), q), waiting_.end());
    active_.erase(std::remove(active_.begin(), active_.end(), q), active_.end());
    bypassed_.erase(q);
    queues_.erase(it);
  }
  return rc;
}

// ------------------------------------------------------------------ kernels
bool Server::kernel_ptr_fields(uint64_t k, std::vector<size_t>* offs) const {
  std::lock_guard<std::mutex> g(mu_);
  auto it = kernels_.find(k);
  if (it == kernels_.end()) return false;
  *offs = it->second->ops->user_ptr_offsets;
  return true;
}

bool Server::kernel_kind(uint64_t k, uint32_t* kind) const {
  std::lock_guard<std::mutex> g(mu_);
  auto it = kernels_.find(k);
  if (it == kernels_.end()) return false;
  *kind = it->second->desc.kind;
  return true;
}

int Server::register_kernel(const slate_kernel_desc* d, uint64_t* out, std::string* err) {
  if (!d || !out || d->abi_version != SLATE_ABI_VERSION) {
    if (err) *err = "bad kernel descriptor";
    return SLATE_EINVAL;
  }
  if (d->kind == 0 || d->kind >= SLATE_KIND_MAX_ || (d->flags & ~(SLATE_KFLAG_COVERAGE | SLATE_KFLAG_RANKLOG)) ||
      ((d->flags & SLATE_KFLAG_RANKLOG) && !(d->flags & SLATE_KFLAG_COVERAGE))) {
    if (err) *err = "bad kind or flags";
    return SLATE_EINVAL;
  }
  const KindOps* ops = kind_ops(d->kind);
  if (!ops) {
    if (err) *err = "kind not built into this library";
    return SLATE_EUNSUPPORTED;
  }
  if (ops->max_iters && d->iters > ops->max_iters) {
    if (err) *err = "iters exceeds the kind's maximum task size";
    return SLATE_EINVAL;
  }
  std::lock_guard<std::mutex> g(mu_);
  const uint32_t iters = d->iters ? d->iters : ops->default_iters;   // 0 = auto per launch
  for (auto& kv : kernels_) {
    const KernelEntry& k = *kv.second;
    if (k.desc.kind == d->kind && k.desc.iters == iters && k.desc.flags == d->flags) {
      *out = k.id;
      return SLATE_OK;
    }
  }
  auto k = std::make_unique<KernelEntry>();
  k->id = next_kernel_id_++;
  k->desc = *d;
  k->desc.iters = iters;
  k->ops = ops;
  if (ops->smem > 48 * 1024)
    CK(cudaFuncSetAttribute(ops->worker_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, ops->smem));
  if (ops->smem_standalone > 48 * 1024)
    CK(cudaFuncSetAttribute(ops->standalone_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, ops->smem_standalone));
  int occ = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ops->worker_fn, ops->threads, ops->smem));
  if (occ < 1) {
    if (err) *err = "worker does not fit on an SM";
    return SLATE_ECUDA;
  }
  static const int occ_cap = int(env_double("SLATE_OCC_CAP", 0));   // experiments: fewer workers per SM
  if (occ_cap > 0 && occ > occ_cap) occ = occ_cap;
  k->occ = occ;
  *out = k->id;
  kernels_[k->id] = std::move(k);
  return SLATE_OK;
}

// NEXT-3: a user kernel from source (user_kernels.cu), a kind of its own
int Server::register_source(const slate_source_desc* d, uint64_t* out, std::string* err) {
  const uint64_t threads = d ? uint64_t(d->block_threads) * (d->block_y ? d->block_y : 1) * (d->block_z ? d->block_z : 1)
                             : 0;
  if (!d || !out || d->abi_version != SLATE_ABI_VERSION || !d->source || !d->kernel_name || d->args_size == 0 ||
      d->args_size > 4096 || threads == 0 || threads > 1024) {
    if (err) *err = "bad source descriptor";
    return SLATE_EINVAL;
  }
  auto ops = std::make_unique<KindOps>();
  std::string e;
  if (!build_user_kind(d->source, d->kernel_name, d->block_threads, d->block_y, d->block_z, d->smem_bytes,
                       d->args_size, ops.get(), &e)) {
    if (err) *err = e;
    return e.find("not found") != std::string::npos ? SLATE_EUNSUPPORTED
           : (e.find("no `__global__") != std::string::npos || e.find("args_size") == 0) ? SLATE_EINVAL : SLATE_ECUDA;
  }
  ops->user_bytes_per_block = d->bytes_per_block;
  ops->user_flops_per_block = d->flops_per_block;
  if (ops->smem > 48 * 1024) {
    CK(cudaFuncSetAttribute(ops->worker_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, ops->smem));
    CK(cudaFuncSetAttribute(ops->standalone_fn, cudaFuncAttributeMaxDynamicSharedMemorySize, ops->smem));
  }
  int occ = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ops->worker_fn, ops->threads, ops->smem));
  if (occ < 1) {
    if (err) *err = "the user worker does not fit on an SM";
    return SLATE_ECUDA;
  }
  std::lock_guard<std::mutex> g(mu_);
  auto k = std::make_unique<KernelEntry>();
  k->id = next_kernel_id_++;
  k->desc = slate_kernel_desc{};
  k->desc.abi_version = SLATE_ABI_VERSION;
  k->desc.kind = SLATE_KIND_USER;
  k->desc.iters = d->iters;
  k->desc.flags = d->flags & (SLATE_KFLAG_COVERAGE | SLATE_KFLAG_RANKLOG);
  if ((k->desc.flags & SLATE_KFLAG_RANKLOG) && !(k->desc.flags & SLATE_KFLAG_COVERAGE)) {
    if (err) *err = "SLATE_KFLAG_RANKLOG needs SLATE_KFLAG_COVERAGE";
    return SLATE_EINVAL;
  }
  k->occ = occ;
  k->ops = ops.get();
  k->own_ops = std::move(ops);
  *out = k->id;
  kernels_[k->id] = std::move(k);
  return SLATE_OK;
}

bool Server::validate(const KernelEntry& k, const slate_launch_desc* d, uint32_t* B, std::string* err) const {
  auto fail = [&](const char* m) {
    if (err) *err = m;
    return false;
  };
  if (!d || !d->args || d->args_size != k.ops->args_size) return fail("args missing or args_size mismatch");
  uint64_t g[3] = {0, 1, 1};
  auto al = [](uint64_t p) { return (p & 15) == 0; };
  switch (k.desc.kind) {
    case SLATE_KIND_TRIAD: {
      auto a = static_cast<const slate_args_triad*>(d->args);
      if (!al(a->a) || !al(a->b) || !al(a->c)) return fail("triad arrays must be 16-byte aligned");
      g[0] = cdiv(a->n, 1024);
      break;
    }
    case SLATE_KIND_COPY: {
      auto a = static_cast<const slate_args_copy*>(d->args);
      if (!al(a->a) || !al(a->b)) return fail("copy arrays must be 16-byte aligned");
      g[0] = cdiv(a->n, 4096);
      break;
    }
    case SLATE_KIND_SGEMM_NAIVE: {
      auto a = static_cast<const slate_args_sgemm*>(d->args);
      g[0] = cdiv(a->n, 16);
      g[1] = cdiv(a->m, 16);
      if (a->k == 0) return fail("k == 0");
      break;
    }
    case SLATE_KIND_SPMV_CSR: {
      auto a = static_cast<const slate_args_spmv*>(d->args);
      if (!al(a->rowptr) || !al(a->col) || !al(a->val) || !al(a->x))
        return fail("spmv rowptr/col/val/x must be 16-byte aligned");
      g[0] = cdiv(a->n_rows, 32);
      break;
    }
    case SLATE_KIND_BLACKSCHOLES: {
      auto a = static_cast<const slate_args_bs*>(d->args);
      if (!al(a->S) || !al(a->X) || !al(a->T) || !al(a->call) || !al(a->put)) return fail("bs arrays must be 16-byte aligned");
      if (a->n_scen == 0) return fail("n_scen == 0");
      g[0] = cdiv(a->n, 1024);
      break;
    }
    case SLATE_KIND_STENCIL2D: {
      auto a = static_cast<const slate_args_stencil*>(d->args);
      g[0] = cdiv(a->w, 128);
      g[1] = cdiv(a->h, 8);
      break;
    }
    case SLATE_KIND_GEMM_BF16: {
      auto a = static_cast<const slate_args_gemm*>(d->args);
      const uint32_t tn = k.ops->tile_n ? k.ops->tile_n : 128, tm = k.ops->tile_m ? k.ops->tile_m : 128;
      // any m; tensor-map row strides must be 16-byte multiples: k % 8, n % 4.
      // Ragged tiles: the TMA loads zero-fill past m, n and k (zero products),
      // the TMA stores of C clip past m and n
      if (a->m == 0 || a->n == 0 || a->k == 0 || a->k % 8 || a->n % 4)
        return fail("gemm_bf16 needs m, n, k > 0, k % 8 == 0 and n % 4 == 0 (16-byte row strides)");
      if (!al(a->A) || !al(a->B) || !al(a->C)) return fail("gemm arrays must be 16-byte aligned");
      g[0] = cdiv(a->n, tn);
      g[1] = cdiv(a->m, tm);
      break;
    }
    case SLATE_KIND_TRANSPOSE: {
      auto a = static_cast<const slate_args_transpose*>(d->args);
      g[0] = cdiv(a->w, 32);
      g[1] = cdiv(a->h, 32);
      break;
    }
    case SLATE_KIND_SGEMM_TILED: {
      auto a = static_cast<const slate_args_sgemm*>(d->args);
      g[0] = cdiv(a->n, 32);
      g[1] = cdiv(a->m, 32);
      if (a->k == 0) return fail("k == 0");
      break;
    }
    case SLATE_KIND_QRNG: {
      auto a = static_cast<const slate_args_qrng*>(d->args);
      if (!al(a->out)) return fail("qrng output must be 16-byte aligned");
      if (a->dims == 0 || a->dims > 65535) return fail("qrng dims must be in [1, 65535]");
      g[0] = cdiv(a->n, 1024);
      g[1] = a->dims;
      break;
    }
    case SLATE_KIND_GAUSS_FAN1:
    case SLATE_KIND_GAUSS_FAN2: {
      auto a = static_cast<const slate_args_gauss*>(d->args);
      if (a->n < 2 || a->t + 1 >= a->n) return fail("gauss step needs t < n - 1");
      if (k.desc.kind == SLATE_KIND_GAUSS_FAN1) {
        g[0] = cdiv(a->n - 1 - a->t, 256);
      } else {
        g[0] = cdiv(a->n - a->t, 128);
        g[1] = cdiv(a->n - 1 - a->t, 16);
      }
      break;
    }
    case SLATE_KIND_USER:        // the caller's grid is the original grid
      g[0] = d->grid[0];
      g[1] = d->grid[1];
      g[2] = d->grid[2];
      break;
    default:
      return fail("unknown kind");
  }
  if (d->grid[0] != g[0] || d->grid[1] != g[1] || d->grid[2] != g[2]) return fail("grid does not match the kind's args");
  const uint64_t total = g[0] * g[1] * g[2];
  if (total == 0) return fail("empty grid");
  if (total >= (1ull << 31)) return fail("grid too large (B >= 2^31)");
  *B = uint32_t(total);
  return true;
}

// algorithmic work per launch: bytes moved, fp32 flops, tensor-core flops
void Server::work(const KernelEntry& k, const slate_launch_desc* d, double* bytes, double* fp32, double* tc) const {
  *bytes = *fp32 = *tc = 0;
  switch (k.desc.kind) {
    case SLATE_KIND_TRIAD: {
      auto a = static_cast<const slate_args_triad*>(d->args);
      *bytes = 12.0 * a->n;
      *fp32 = 2.0 * a->n;
      break;
    }
    case SLATE_KIND_COPY: {
      auto a = static_cast<const slate_args_copy*>(d->args);
      *bytes = 8.0 * a->n;
      break;
    }
    case SLATE_KIND_SGEMM_NAIVE: {
      auto a = static_cast<const slate_args_sgemm*>(d->args);
      *bytes = 4.0 * (double(a->m) * a->k + double(a->k) * a->n + double(a->m) * a->n);
      *fp32 = 2.0 * a->m * double(a->n) * a->k;
      break;
    }
    case SLATE_KIND_SPMV_CSR: {
      auto a = static_cast<const slate_args_spmv*>(d->args);
      int nnz = 0;
      cudaMemcpy(&nnz, reinterpret_cast<const int*>(a->rowptr) + a->n_rows, 4, cudaMemcpyDeviceToHost);
      *bytes = 8.0 * nnz + 4.0 * (a->n_rows + 1) + 4.0 * a->n_rows + 4.0 * a->n_cols;
      *fp32 = 2.0 * nnz;
      break;
    }
    case SLATE_KIND_BLACKSCHOLES: {
      auto a = static_cast<const slate_args_bs*>(d->args);
      *bytes = 20.0 * a->n + 4.0 * a->n_scen;
      *fp32 = 36.0 * a->n * a->n_scen;   // 36 flops per option-scenario
      break;
    }
    case SLATE_KIND_STENCIL2D: {
      auto a = static_cast<const slate_args_stencil*>(d->args);
      *bytes = 8.0 * a->h * double(a->w);
      *fp32 = 4.0 * a->h * double(a->w);
      break;
    }
    case SLATE_KIND_GEMM_BF16: {
      auto a = static_cast<const slate_args_gemm*>(d->args);
      *bytes = 2.0 * (double(a->m) * a->k + double(a->n) * a->k) + 4.0 * double(a->m) * a->n;
      *tc = 2.0 * a->m * double(a->n) * a->k;
      break;
    }
    case SLATE_KIND_TRANSPOSE: {
      auto a = static_cast<const slate_args_transpose*>(d->args);
      *bytes = 8.0 * a->h * double(a->w);
      break;
    }
    case SLATE_KIND_SGEMM_TILED: {
      auto a = static_cast<const slate_args_sgemm*>(d->args);
      *bytes = 4.0 * (double(a->m) * a->k + double(a->k) * a->n + double(a->m) * a->n);
      *fp32 = 2.0 * a->m * double(a->n) * a->k;
      break;
    }
    case SLATE_KIND_QRNG: {
      auto a = static_cast<const slate_args_qrng*>(d->args);
      *bytes = 4.0 * double(a->n) * a->dims + 124.0 * a->dims;
      *fp32 = double(a->n) * a->dims;           // the 2^-31 scaling (the XOR walk is integer work)
      break;
    }
    case SLATE_KIND_GAUSS_FAN1: {
      auto a = static_cast<const slate_args_gauss*>(d->args);
      const double r = a->n - 1.0 - a->t;
      *bytes = 8.0 * r + 4.0;
      *fp32 = r;
      break;
    }
    case SLATE_KIND_USER: {      // declared at registration, per block
      const double B = double(d->grid[0]) * d->grid[1] * d->grid[2];
      *bytes = k.ops->user_bytes_per_block * B;
      *fp32 = k.ops->user_flops_per_block * B;
      break;
    }
    case SLATE_KIND_GAUSS_FAN2: {
      auto a = static_cast<const slate_args_gauss*>(d->args);
      const double r = a->n - 1.0 - a->t, c = double(a->n) - a->t;
      *bytes = 8.0 * r * c + 4.0 * c + 4.0 * r + 8.0 * r + 4.0;   // trailing block r/w, pivot row, m column, b
      *fp32 = 2.0 * r * c + 2.0 * r;
      break;
    }
  }
}

int Server::alloc_slot() {
  if (free_slots_.empty()) return -1;
  const int s = free_slots_.front();
  free_slots_.pop_front();
  return s;
}

// a freed control block is zeroed by DMA on the copy stream right away, so the
// next launch that takes the slot only waits on an (already complete) event
void Server::free_slot(int slot) { pending_free_.push_back(slot); }

// Zero the control blocks freed since the last flush by DMA, one copy per run
// of consecutive slots (a batch's launches hold consecutive slots: a job of
// 8190 launches is ~32 copies, not 8190).  A slot's event is its run's, from
// a round-robin pool: an event re-recorded later only makes a waiter wait
// longer (the copy stream is in order).
void Server::flush_free() {
  if (pending_free_.empty()) return;
  std::sort(pending_free_.begin(), pending_free_.end());
  size_t i = 0;
  while (i < pending_free_.size()) {
    size_t j = i + 1;
    while (j < pending_free_.size() && pending_free_[j] == pending_free_[j - 1] + 1 && int(j - i) < kZeroRun) ++j;
    const int s0 = pending_free_[i], len = int(j - i);
    cudaMemcpyAsync(d_tc_ + s0, h_zero_, sizeof(TaskCtl) * len, cudaMemcpyHostToDevice, copy_stream_);
    cudaEvent_t e = zero_ev_[zero_ev_next_++ % kZeroEv];
    cudaEventRecord(e, copy_stream_);
    for (size_t k = i; k < j; ++k) {
      slot_zeroed_[pending_free_[k]] = e;
      free_slots_.push_back(pending_free_[k]);
    }
    i = j;
  }
  pending_free_.clear();
}

// one wave of workers (Q12) -- but no more CTAs than there are tasks,
// and at least one per SM (so any SM range gets workers): every worker CTA
// costs its launch a prologue and a fetch (tools/probe/launch_cost.cu)
uint32_t Server::worker_grid(int occ, uint32_t B, uint32_t iters, bool full_range) const {
  const uint64_t wave = uint64_t(occ) * uint64_t(n_sms_);
  const uint64_t tasks = (uint64_t(B) + iters - 1) / iters;
  // on the whole chip any SM will do: one CTA per task suffices (a 6-block
  // Gaussian-elimination step gets 6 CTAs, not 148)
  return uint32_t(std::min<uint64_t>(wave, full_range ? tasks : std::max<uint64_t>(uint64_t(n_sms_), tasks)));
}

// reading Q11: the paper's default task of 10 blocks, reduced so every
// worker gets at least ~8 tasks (a fixed 10 mis-fits small grids: the last
// tasks leave workers idle)
uint32_t Server::auto_iters(uint32_t B, int occ, uint32_t cap, uint32_t per_worker) const {
  const uint64_t workers = uint64_t(occ) * uint64_t(n_sms_);
  const uint64_t it = B / (uint64_t(per_worker ? per_worker : 8) * workers);
  return uint32_t(it < 1 ? 1 : (it > cap ? cap : it));
}

// ------------------------------------------------------------------ control word
int Server::write_ctrl(Queue& Q, uint32_t lo, uint32_t hi, bool, std::string* err) {
  Q.epoch += 1;
  Q.lo = lo;
  Q.hi = hi;
  Q.cov_lo = std::max(Q.cov_lo, lo);   // workers outside the new range retire
  Q.cov_hi = std::min(Q.cov_hi, hi);
  const uint64_t v = pack_ctrl(Q.epoch, lo, hi);
  // a stream memory write needs no SM: it lands even while persistent workers fill every SM
  const CUresult r = reinterpret_cast<WriteValue64Fn>(write_value64_)(
      reinterpret_cast<CUstream>(ctrl_stream_), reinterpret_cast<CUdeviceptr>(Q.d_ctrl), v, 0);
  if (r != CUDA_SUCCESS) {
    if (err) *err = "cuStreamWriteValue64 failed: " + std::to_string(int(r));
    return SLATE_ECUDA;
  }
  // later launches of this queue start after the write: the event is recorded
  // now (a top-up waits for it on its own stream), and the queue's stream waits
  // for it just before its next kernel (settle_ctrl) -- one wait for several
  // writes between two kernels of the queue
  CK(cudaEventRecord(Q.ev_ctrl, ctrl_stream_));
  Q.ctrl_wait_pending = true;
  return SLATE_OK;
}

// The first issued launch of the queue that has not finished its blocks, by
// binary search: launches of a queue run in stream order, so the done ones are
// a prefix of `issued`.  A batch's members stay in `issued` until the batch's
// end event (no events between them), so the prefix can hold hundreds of
// launches: the linear scans this replaces cost ~120 us of the server lock per
// grow in C2 (640-launch SpMV jobs), delaying the top-up by as much.
size_t Server::first_running(const Queue& Q) const {
  size_t lo = 0, hi = Q.issued.size();
  while (lo < hi) {
    const size_t mid = (lo + hi) / 2;
    const Launch& E = *launches_.at(Q.issued[mid]);
    const bool done = E.slot < 0 || h_mirror_[E.slot].done != 0;
    if (done) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

void Server::settle_ctrl(Queue& Q) {
  if (!Q.ctrl_wait_pending) return;
  cudaStreamWaitEvent(Q.stream, Q.ev_ctrl, 0);   // the latest record: the queue's latest word (a failure
                                                 // here is sticky and surfaces at the next launch's CK)
  Q.last_op_kernel = false;
  Q.ctrl_wait_pending = false;
}

// ------------------------------------------------------------------ issue
// Launches of a queue reach its stream in submission order; one that finds no
// free control block waits in Q.deferred (and so do all later ones) until the
// poller frees blocks.
int Server::issue(Launch& L, Queue& Q, std::string* err) {
  const bool needs_slot = L.desc.mode != SLATE_MODE_STANDALONE;
  if (!Q.deferred.empty() || (needs_slot && free_slots_.empty())) {
    if (!Q.open_batch.empty()) close_batch(Q, nullptr);
    Q.deferred.push_back(L.id);
    return SLATE_OK;
  }
  return issue_now(L, Q, err);
}

// End the queue's open batch: every member completes with the batch's end
// event `end` (recorded here on the queue's stream if null); the workers'
// control-block snapshots are copied after it.
void Server::close_batch(Queue& Q, cudaEvent_t end, bool closed_by_launch) {
  if (Q.open_batch.empty()) return;
  if (!end) {
    cudaEventCreate(&end);
    cudaEventRecord(end, Q.stream);
    Q.last_op_kernel = false;
  }
  std::vector<Launch*> ws;
  for (uint64_t id : Q.open_batch) {
    Launch& M = *launches_[id];
    M.batch_end = end;
    M.batch_n = uint32_t(Q.open_batch.size()) + (closed_by_launch ? 1u : 0u);
    if (M.slot >= 0) ws.push_back(&M);
    else M.ev_done.push_back(end);
  }
  if (!ws.empty()) {
    cudaEvent_t snap;
    cudaEventCreateWithFlags(&snap, cudaEventDisableTiming);
    cudaStreamWaitEvent(Q.snap, end, 0);
    // one strided copy per run of consecutive slots (headers out of 2.5-KB blocks)
    for (size_t i = 0; i < ws.size();) {
      size_t j = i + 1;
      while (j < ws.size() && ws[j]->slot == ws[j - 1]->slot + 1) ++j;
      const int s0 = ws[i]->slot;
      cudaMemcpy2DAsync(h_snap_ + size_t(s0) * kTaskCtlHeader, kTaskCtlHeader, d_tc_ + s0, sizeof(TaskCtl),
                        kTaskCtlHeader, j - i, cudaMemcpyDeviceToHost, Q.snap);
      i = j;
    }
    cudaEventRecord(snap, Q.snap);
    for (Launch* M : ws) M->ev_done.push_back(snap);
  }
  Q.open_batch.clear();
}

void Server::fail_launch(Launch& L, int code) {
  L.error = code;
  L.state = 2;
  finished_.push_back(L.id);
  auto qi = queues_.find(L.queue);
  if (qi != queues_.end() && !qi->second->first_error) qi->second->first_error = code;
  cv_.notify_all();
}

// Drop the oldest completed launch records beyond the retention window, with
// the CUDA events only they reference.  Events are shared between launches (a
// batch's end and snapshot events, a chained launch's start = its
// predecessor's end, top-up ends), so an event is destroyed only when no
// retained launch or queue names it.  Bulk: one scan per keep_finished_
// evictions.
void Server::retire_finished() {
  if (finished_.size() <= keep_finished_) return;
  std::unordered_set<cudaEvent_t> cand;
  const size_t n = finished_.size() - keep_finished_;
  for (size_t i = 0; i < n; ++i) {
    const uint64_t id = finished_.front();
    finished_.pop_front();
    auto it = launches_.find(id);
    if (it == launches_.end()) continue;
    const Launch& L = *it->second;
    cand.insert(L.ev_start);
    cand.insert(L.batch_end);
    for (cudaEvent_t e : L.ev_end) cand.insert(e);
    for (cudaEvent_t e : L.ev_done) cand.insert(e);
    launches_.erase(it);
  }
  for (const auto& kv : launches_) {
    const Launch& L = *kv.second;
    cand.erase(L.ev_start);
    cand.erase(L.start_after);
    cand.erase(L.batch_end);
    for (cudaEvent_t e : L.ev_end) cand.erase(e);
    for (cudaEvent_t e : L.ev_done) cand.erase(e);
  }
  for (const auto& kv : queues_)
    for (cudaEvent_t e : kv.second->topup_ends) cand.erase(e);
  for (cudaEvent_t e : cand)
    if (e) cudaEventDestroy(e);
}

void Server::drain_deferred(Queue& Q) {
  std::string err;
  while (!Q.deferred.empty()) {
    Launch& L = *launches_[Q.deferred.front()];
    if (L.desc.mode != SLATE_MODE_STANDALONE && free_slots_.empty()) break;
    Q.deferred.pop_front();
    const Launch* nx = Q.deferred.empty() ? nullptr : launches_[Q.deferred.front()].get();
    batch_more_ = nx && (nx->desc.mode == SLATE_MODE_STANDALONE || free_slots_.size() > 1);
    if (issue_now(L, Q, &err) != SLATE_OK) fail_launch(L, int(cudaErrorLaunchFailure));
    batch_more_ = false;
  }
  close_batch(Q, nullptr);
}

int Server::issue_now(Launch& L, Queue& Q, std::string* err) {
  const KindOps* ops = L.k->ops;
  settle_ctrl(Q);
  for (cudaEvent_t e : Q.topup_ends) {   // stream semantics: the predecessor's top-up workers finish first
    CK(cudaStreamWaitEvent(Q.stream, e, 0));
    Q.last_op_kernel = false;
  }
  Q.topup_ends.clear();
  // a batch holds launches of one mode
  if (!Q.open_batch.empty() && launches_[Q.open_batch.front()]->desc.mode != L.desc.mode) close_batch(Q, nullptr);
  // Events between kernels cost ~3 us of stream time each and stop programmatic
  // dependent launch (tools/probe/pdl_cost.cu).  A launch queued right behind
  // another of its queue starts where that one ends (stream order), so it
  // records no start event; inside a batch (launches issued back to back by one
  // loop) only the last records an end event.
  const bool in_batch = !Q.open_batch.empty();
  if (in_batch) {
    L.batch_first = Q.open_batch.front();
    L.batch_idx = uint32_t(Q.open_batch.size());
  } else if (!Q.issued.empty() && !launches_[Q.issued.back()]->ev_end.empty()) {
    L.start_after = launches_[Q.issued.back()]->ev_end.front();
  } else {
    CK(cudaEventCreate(&L.ev_start));
  }
  const bool batch_member = batch_more_;   // no end event: the batch's end completes it
  cudaEvent_t ev_end = nullptr;
  if (!batch_member) CK(cudaEventCreate(&ev_end));
  const auto& g = L.desc.grid;
  if (L.desc.mode == SLATE_MODE_STANDALONE) {
    if (L.ev_start) CK(cudaEventRecord(L.ev_start, Q.stream));
    if (ops->launch_standalone_ops)
      CK(ops->launch_standalone_ops(ops, L.args.data(), dim3(g[0], g[1], g[2]), Q.stream));
    else
      CK(ops->launch_standalone(L.args.data(), dim3(g[0], g[1], g[2]), Q.stream));
    Q.last_op_kernel = false;   // standalone kernels do not wait in griddepcontrol.wait: no PDL after them
    if (ev_end) {
      CK(cudaEventRecord(ev_end, Q.stream));
      L.ev_end.push_back(ev_end);
      L.ev_done.push_back(ev_end);
    }
  } else {
    const int slot = alloc_slot();
    if (slot < 0) {
      if (err) *err = "control-block pool exhausted";
      return SLATE_ENOMEM;
    }
    L.slot = slot;
    std::memset(reinterpret_cast<void*>(h_mirror_ + slot), 0, sizeof(HostMirror));
    // the control block was zeroed by DMA when it was freed (no SM needed); only
    // wait (a cross-stream dependency) if that copy has not finished yet
    if (slot_zeroed_[slot] && cudaEventQuery(slot_zeroed_[slot]) != cudaSuccess) {
      CK(cudaStreamWaitEvent(Q.stream, slot_zeroed_[slot], 0));
      Q.last_op_kernel = false;
    }
    if (L.ev_start) {
      CK(cudaEventRecord(L.ev_start, Q.stream));
      Q.last_op_kernel = false;
    }
    WorkerCommon w{};
    w.gx = g[0]; w.gy = g[1]; w.gz = g[2]; w.B = L.B; w.iters = L.iters; w.occ = uint32_t(L.k->occ);
    w.bound_lo = 0; w.bound_hi = uint32_t(n_sms_ - 1); w.n_ranks = uint32_t(n_sms_);
    w.standby_timeout_ns = standby_timeout_ns_;
    w.base_epoch = Q.epoch;
    w.ctrl = Q.d_ctrl; w.tc = d_tc_ + slot; w.mirror = d_mirror_ + slot;
    w.cov = reinterpret_cast<uint32_t*>(L.desc.coverage);
    w.ranklog = (L.k->desc.flags & SLATE_KFLAG_RANKLOG) && w.cov ? 1u : 0u;
    w.rank_of = d_rank_of_;
    w.ops = ops;
    // PDL: the previous op on the stream is the previous worker of this batch
    w.pdl = in_batch && Q.last_op_kernel && ops->pdl_ok && pdl_enabled_;
    if (w.pdl && ops->pdl_early_ok && pdl_early_enabled_) {   // the previous grid: the same kernel, the same args?
      const Launch& P = *launches_[Q.open_batch.back()];
      w.pdl_early = P.k == L.k && P.args == L.args && P.slot >= 0 &&
                    (!ops->outputs_disjoint || ops->outputs_disjoint(L.args.data())) ? 1u : 0u;
    }
    const bool full = Q.lo == 0 && Q.hi == uint32_t(n_sms_ - 1);
    CK(ops->launch_worker(w, L.args.data(), worker_grid(L.k->occ, L.B, L.iters, full), Q.stream));
    Q.last_op_kernel = ops->pdl_ok;
    if (ev_end) {
      CK(cudaEventRecord(ev_end, Q.stream));
      Q.last_op_kernel = false;
      L.ev_end.push_back(ev_end);
      cudaEvent_t ev_snap;
      CK(cudaEventCreateWithFlags(&ev_snap, cudaEventDisableTiming));
      CK(cudaStreamWaitEvent(Q.snap, ev_end, 0));
      CK(cudaMemcpyAsync(h_snap_ + size_t(slot) * kTaskCtlHeader, d_tc_ + slot, kTaskCtlHeader,
                         cudaMemcpyDeviceToHost, Q.snap));
      CK(cudaEventRecord(ev_snap, Q.snap));
      L.ev_done.push_back(ev_snap);
    }
  }
  if (batch_member) {
    Q.open_batch.push_back(L.id);
  } else if (!Q.open_batch.empty()) {
    L.batch_n = uint32_t(Q.open_batch.size()) + 1;
    close_batch(Q, ev_end, true);   // this launch ends the batch
  }
  L.state = 1;
  L.t_issue_us = now_us();
  if (Q.issued.empty()) {
    Q.cov_lo = Q.lo;
    Q.cov_hi = Q.hi;
  }
  Q.issued.push_back(L.id);
  cv_.notify_all();
  return SLATE_OK;
}

// grow: workers for the ranks newly in range of the queue's running launch.
// Only the LAST issued launch of the queue gets a top-up (a launch already
// queued behind it on the stream picks up the new range by itself); later
// launches wait for the top-up's end (stream semantics).
int Server::grow_running(Queue& Q, uint32_t, uint32_t, std::string* err) {
  // only the last issued launch can get a top-up (later launches must stay behind
  // it in stream order); launches before it that finished all their blocks but
  // are not yet retired by the poller do not count
  static const bool dbg = std::getenv("SLATE_DEBUG") != nullptr;
  if (Q.n_fused) return SLATE_OK;   // a fused co-run kernel (NEXT-1): its CTAs switch tenant, no launch
  if (!Q.issued.empty()) {
    // kinds whose last main CTA waits for all blocks (leave_main): top up the
    // RUNNING launch -- the first issued one that has not finished its blocks --
    // whatever is queued behind it (a grow then lands within a task, not a launch)
    const size_t i = first_running(Q);
    if (i < Q.issued.size()) {
      Launch& E = *launches_[Q.issued[i]];
      if (E.slot >= 0 && E.desc.mode != SLATE_MODE_STANDALONE && E.k->ops->topup_anytime) return topup(Q, E, err);
    }
  }
  if (Q.issued.empty() || !Q.pending.empty() || !Q.deferred.empty()) {
    if (dbg) fprintf(stderr, "[slate] grow: no top-up (issued %zu pending %zu deferred %zu)\n", Q.issued.size(),
                     Q.pending.size(), Q.deferred.size());
    if (Q.pending.empty() && Q.deferred.empty()) drop_idle_grow(Q);
    return SLATE_OK;
  }
  for (size_t i = 0; i + 1 < Q.issued.size(); ++i) {
    const Launch& E = *launches_[Q.issued[i]];
    if (E.slot < 0 || !h_mirror_[E.slot].done) {
      if (dbg) fprintf(stderr, "[slate] grow: no top-up (an earlier launch is still running)\n");
      return SLATE_OK;
    }
  }
  Launch& R = *launches_[Q.issued.back()];
  if (R.state != 1 || R.slot < 0 || R.desc.mode == SLATE_MODE_STANDALONE) return SLATE_OK;
  if (h_mirror_[R.slot].done) {
    if (dbg) fprintf(stderr, "[slate] grow: no top-up (the launch finished its blocks)\n");
    drop_idle_grow(Q);
    return SLATE_OK;
  }
  return topup(Q, R, err);
}

// A grow when the queue has no block left to run (its launches finished their
// blocks, nothing queued): no worker can join until the client's next launch,
// so the grow has no completion of its own to time -- counted with the
// superseded resizes (n_superseded), not as a latency.
void Server::drop_idle_grow(Queue& Q) {
  for (auto it = Q.pending_resize.rbegin(); it != Q.pending_resize.rend(); ++it) {
    if (it->kind == 2 && it->epoch == Q.epoch) {
      auto li = launches_.find(it->lid);
      if (li != launches_.end()) li->second->n_superseded += 1;
      Q.pending_resize.erase(std::next(it).base());
      return;
    }
  }
}

// a top-up grid for launch R on the queue's current range, sharing R's counter
int Server::topup(Queue& Q, Launch& R, std::string* err) {
  static const bool dbg = std::getenv("SLATE_DEBUG") != nullptr;
  if (dbg) {
    double since = -1;   // host time since the queue's latest grow call (us)
    for (auto it = Q.pending_resize.rbegin(); it != Q.pending_resize.rend(); ++it)
      if (it->kind == 2) { since = now_us() - it->t0_us; break; }
    fprintf(stderr, "[slate] grow: top-up for launch %llu on [%u, %u], %.1f us after the grow call\n",
            (unsigned long long)R.id, Q.lo, Q.hi, since);
  }
  const auto& g = R.desc.grid;
  cudaStream_t aux = Q.aux[Q.aux_next++ % Queue::kAux];
  // the top-up starts after the resize word it must see (recorded by write_ctrl
  // right after the queue's latest write) and after R started
  CK(cudaStreamWaitEvent(aux, Q.ev_ctrl, 0));
  cudaEvent_t r_start = R.ev_start ? R.ev_start : R.start_after;
  if (r_start) CK(cudaStreamWaitEvent(aux, r_start, 0));
  WorkerCommon w{};
  w.gate_first = r_start ? 0u : 1u;   // a batch member has no start event: its top-up waits on the device
  w.gx = g[0]; w.gy = g[1]; w.gz = g[2]; w.B = R.B; w.iters = R.iters; w.occ = uint32_t(R.k->occ);
  w.bound_lo = Q.lo; w.bound_hi = Q.hi; w.n_ranks = uint32_t(n_sms_);
  w.standby_timeout_ns = standby_timeout_ns_;
  w.is_topup = 1;
  w.ops = R.k->ops;
  w.ctrl = Q.d_ctrl; w.tc = d_tc_ + R.slot; w.mirror = d_mirror_ + R.slot;
  w.cov = reinterpret_cast<uint32_t*>(R.desc.coverage);
  w.ranklog = (R.k->desc.flags & SLATE_KFLAG_RANKLOG) && w.cov ? 1u : 0u;
  w.rank_of = d_rank_of_;
  CK(R.k->ops->launch_worker(w, R.args.data(), uint32_t(R.k->occ) * uint32_t(n_sms_), aux));
  cudaEvent_t ev_end, ev_snap;
  CK(cudaEventCreate(&ev_end));
  CK(cudaEventRecord(ev_end, aux));
  R.ev_end.push_back(ev_end);
  CK(cudaEventCreateWithFlags(&ev_snap, cudaEventDisableTiming));
  CK(cudaStreamWaitEvent(Q.snap, ev_end, 0));
  CK(cudaMemcpyAsync(h_snap_ + size_t(R.slot) * kTaskCtlHeader, d_tc_ + R.slot, kTaskCtlHeader,
                     cudaMemcpyDeviceToHost, Q.snap));
  CK(cudaEventRecord(ev_snap, Q.snap));
  R.ev_done.push_back(ev_snap);
  Q.topup_ends.push_back(ev_end);
  R.n_topups += 1;
  if (Q.cov_lo > Q.cov_hi) {
    Q.cov_lo = Q.lo;
    Q.cov_hi = Q.hi;
  } else {
    Q.cov_lo = std::min(Q.cov_lo, Q.lo);
    Q.cov_hi = std::max(Q.cov_hi, Q.hi);
  }
  return SLATE_OK;
}

// ------------------------------------------------------------------ launch
int Server::launch(uint32_t q, uint64_t kid, const slate_launch_desc* d, uint64_t* out, std::string* err) {
  std::unique_lock<std::mutex> g(mu_);
  return launch_locked(q, kid, d, out, err, false);
}

// n launches of one kernel in one call (a job): all are queued before the
// selector looks at them, so a co-run decision sees the whole job
int Server::launch_n(uint32_t q, uint64_t kid, const slate_launch_desc* d, uint32_t n, uint64_t* first,
                     std::string* err) {
  if (n == 0) {
    if (err) *err = "n == 0";
    return SLATE_EINVAL;
  }
  std::unique_lock<std::mutex> g(mu_);
  int rc = SLATE_OK;
  for (uint32_t i = 0; i < n && rc == SLATE_OK; ++i) {
    uint64_t id = 0;
    batch_more_ = i + 1 < n;   // the job's launches go out as one batch if the queue can take them now
    rc = launch_locked(q, kid, d, &id, err, i + 1 < n);
    if (i == 0) *first = id;
  }
  batch_more_ = false;
  auto qi = queues_.find(q);
  if (qi != queues_.end()) close_batch(*qi->second, nullptr);
  return rc;
}

// n launches of different kernels/descriptors in one call, issued as one batch
int Server::launch_many(uint32_t q, uint32_t n, const uint64_t* ks, const slate_launch_desc* ds, uint64_t* first,
                        std::string* err) {
  if (n == 0) {
    if (err) *err = "n == 0";
    return SLATE_EINVAL;
  }
  std::unique_lock<std::mutex> g(mu_);
  int rc = SLATE_OK;
  for (uint32_t i = 0; i < n && rc == SLATE_OK; ++i) {
    uint64_t id = 0;
    batch_more_ = i + 1 < n;
    rc = launch_locked(q, ks[i], &ds[i], &id, err, i + 1 < n);
    if (i == 0) *first = id;
  }
  batch_more_ = false;
  auto qi = queues_.find(q);
  if (qi != queues_.end()) close_batch(*qi->second, nullptr);
  return rc;
}

// NEXT-1 (fused.cuh): one persistent kernel runs both launches; each keeps its
// own control block, resize word (its queue's) and records, so sync, query
// and resize work as for separate launches, but a resize -- and the grow when
// one tenant drains -- needs no top-up launch: the CTAs switch tenant
// at their next task boundary.
int Server::launch_fused(uint32_t qa, uint64_t ka, const slate_launch_desc* da, uint32_t qb, uint64_t kb,
                         const slate_launch_desc* db, uint32_t sm_b, uint64_t* la, uint64_t* lb, std::string* err) {
  std::unique_lock<std::mutex> g(mu_);
  auto fail = [&](int rc, const char* m) {
    if (err) *err = m;
    return rc;
  };
  if (qa == qb) return fail(SLATE_EINVAL, "a fused pair needs two sessions (queues)");
  auto qia = queues_.find(qa), qib = queues_.find(qb);
  auto kia = kernels_.find(ka), kib = kernels_.find(kb);
  if (qia == queues_.end() || qib == queues_.end() || kia == kernels_.end() || kib == kernels_.end())
    return fail(SLATE_ENOTFOUND, "unknown session or kernel");
  const KernelEntry& KA = *kia->second;
  const KernelEntry& KB = *kib->second;
  if (!fused_supported(KA.desc.kind, KB.desc.kind))
    return fail(SLATE_EUNSUPPORTED, "no fused worker for this pair of kinds");
  if (da->mode != SLATE_MODE_SLATE || db->mode != SLATE_MODE_SLATE) return fail(SLATE_EINVAL, "fused launches are slate mode");
  if (sm_b == 0 || sm_b >= uint32_t(n_sms_)) return fail(SLATE_EINVAL, "sm_b must be in [1, N-1]");
  if ((da->coverage && !(KA.desc.flags & SLATE_KFLAG_COVERAGE)) || (db->coverage && !(KB.desc.flags & SLATE_KFLAG_COVERAGE)))
    return fail(SLATE_EINVAL, "coverage log given but the kernel was not registered with SLATE_KFLAG_COVERAGE");
  Queue& A = *qia->second;
  Queue& B = *qib->second;
  auto idle = [](const Queue& Q) { return Q.issued.empty() && Q.pending.empty() && Q.deferred.empty(); };
  if (!idle(A) || !idle(B)) return fail(SLATE_ESTATE, "both sessions must have no launch queued or running");
  uint32_t BA = 0, BB = 0;
  if (!validate(KA, da, &BA, err) || !validate(KB, db, &BB, err)) return SLATE_EINVAL;
  if (free_slots_.size() < 2) return fail(SLATE_ENOMEM, "control-block pool exhausted");
  const uint32_t n = uint32_t(n_sms_);
  // the ranges: A [0, n - sm_b - 1], B [n - sm_b, n - 1]; both queues hold SMs
  for (Queue* Q : {&A, &B}) {
    if (!Q->active) {
      Q->active = true;
      active_.push_back(Q->id);
    }
    Q->explicit_range = true;
    Q->auto_split = false;
  }
  int rc = write_ctrl(A, 0, n - sm_b - 1, false, err);
  if (rc == SLATE_OK) rc = write_ctrl(B, n - sm_b, n - 1, false, err);
  if (rc != SLATE_OK) return rc;
  Launch* Ls[2];
  WorkerCommon w[2];
  const KernelEntry* Ks[2] = {&KA, &KB};
  const slate_launch_desc* Ds[2] = {da, db};
  Queue* Qs[2] = {&A, &B};
  const uint32_t Bs[2] = {BA, BB};
  cudaEvent_t ev_start = nullptr, ev_end = nullptr, ev_snap = nullptr;
  CK(cudaEventCreate(&ev_start));
  CK(cudaEventCreate(&ev_end));
  CK(cudaEventCreateWithFlags(&ev_snap, cudaEventDisableTiming));
  // the kernel goes on A's stream after B's stream is ready (its resize word written)
  settle_ctrl(A);
  settle_ctrl(B);
  cudaEvent_t ev_b;
  CK(cudaEventCreateWithFlags(&ev_b, cudaEventDisableTiming));
  CK(cudaEventRecord(ev_b, B.stream));
  CK(cudaStreamWaitEvent(A.stream, ev_b, 0));
  cudaEventDestroy(ev_b);
  for (int i = 0; i < 2; ++i) {
    auto L = std::make_unique<Launch>();
    L->id = next_launch_id_++;
    L->queue = Qs[i]->id;
    L->k = Ks[i];
    L->desc = *Ds[i];
    L->args.assign(static_cast<const unsigned char*>(Ds[i]->args),
                   static_cast<const unsigned char*>(Ds[i]->args) + Ds[i]->args_size);
    L->desc.args = nullptr;
    L->B = Bs[i];
    L->iters = Ks[i]->desc.iters ? Ks[i]->desc.iters : choose_iters(*Ks[i], Ds[i], Bs[i]);
    L->fused = true;
    Qs[i]->n_fused += 1;
    L->slot = alloc_slot();
    std::memset(reinterpret_cast<void*>(h_mirror_ + L->slot), 0, sizeof(HostMirror));
    if (slot_zeroed_[L->slot] && cudaEventQuery(slot_zeroed_[L->slot]) != cudaSuccess)
      CK(cudaStreamWaitEvent(A.stream, slot_zeroed_[L->slot], 0));
    L->ev_start = ev_start;
    L->ev_end.push_back(ev_end);
    L->ev_done.push_back(ev_snap);
    L->state = 1;
    const auto& gd = L->desc.grid;
    WorkerCommon& c = w[i];
    c.gx = gd[0]; c.gy = gd[1]; c.gz = gd[2]; c.B = L->B; c.iters = L->iters; c.occ = 1;
    c.bound_lo = 0; c.bound_hi = n - 1; c.n_ranks = n;
    c.standby_timeout_ns = standby_timeout_ns_;
    c.base_epoch = Qs[i]->epoch;
    c.is_topup = 0;
    c.gate_first = 0;
    c.ctrl = Qs[i]->d_ctrl; c.tc = d_tc_ + L->slot; c.mirror = d_mirror_ + L->slot;
    c.cov = reinterpret_cast<uint32_t*>(L->desc.coverage);
    c.ranklog = (Ks[i]->desc.flags & SLATE_KFLAG_RANKLOG) && c.cov ? 1u : 0u;
    c.rank_of = d_rank_of_;
    Ls[i] = L.get();
    launches_[L->id] = std::move(L);
  }
  const void* fn = nullptr;
  int threads = 0, smem = 0, occ = 0;
  CK(fused_shape(KA.desc.kind, KB.desc.kind, &fn, &threads, &smem));
  if (smem > 48 * 1024) CK(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, threads, smem));
  if (occ < 1) return fail(SLATE_ECUDA, "the fused worker does not fit on an SM");
  w[0].occ = w[1].occ = uint32_t(occ);
  CK(cudaEventRecord(ev_start, A.stream));
  CK(slate::launch_fused(KA.desc.kind, KB.desc.kind, w[0], Ls[0]->args.data(), w[1], Ls[1]->args.data(), 1u,
                  uint32_t(occ) * n, A.stream));
  CK(cudaEventRecord(ev_end, A.stream));
  CK(cudaStreamWaitEvent(B.stream, ev_end, 0));   // B's later launches follow the fused kernel
  A.last_op_kernel = B.last_op_kernel = false;
  CK(cudaStreamWaitEvent(A.snap, ev_end, 0));
  for (Launch* L : Ls)
    CK(cudaMemcpyAsync(h_snap_ + size_t(L->slot) * kTaskCtlHeader, d_tc_ + L->slot, kTaskCtlHeader,
                       cudaMemcpyDeviceToHost, A.snap));
  CK(cudaEventRecord(ev_snap, A.snap));
  for (int i = 0; i < 2; ++i) {
    Ls[i]->t_issue_us = now_us();
    Qs[i]->issued.push_back(Ls[i]->id);
    Qs[i]->cov_lo = 0;
    Qs[i]->cov_hi = n - 1;
  }
  *la = Ls[0]->id;
  *lb = Ls[1]->id;
  cv_.notify_all();
  return SLATE_OK;
}

int Server::launch_locked(uint32_t q, uint64_t kid, const slate_launch_desc* d, uint64_t* out, std::string* err,
                          bool defer) {
  auto qi = queues_.find(q);
  if (qi == queues_.end()) return SLATE_ENOTFOUND;
  auto ki = kernels_.find(kid);
  if (ki == kernels_.end()) {
    if (err) *err = "unknown kernel";
    return SLATE_ENOTFOUND;
  }
  const KernelEntry& k = *ki->second;
  uint32_t B = 0;
  if (!validate(k, d, &B, err)) return SLATE_EINVAL;
  if (d->placement > SLATE_PLACE_CORUN || d->mode > SLATE_MODE_STANDALONE) {
    if (err) *err = "bad placement or mode";
    return SLATE_EINVAL;
  }
  if (d->placement == SLATE_PLACE_CORUN && (d->sm_lo > d->sm_hi || d->sm_hi >= uint32_t(n_sms_))) {
    if (err) *err = "bad SM range";
    return SLATE_EINVAL;
  }
  if (d->coverage && !(k.desc.flags & SLATE_KFLAG_COVERAGE)) {
    if (err) *err = "coverage log given but the kernel was not registered with SLATE_KFLAG_COVERAGE";
    return SLATE_EINVAL;
  }
  auto L = std::make_unique<Launch>();
  L->id = next_launch_id_++;
  L->queue = q;
  L->k = &k;
  L->desc = *d;
  L->args.assign(static_cast<const unsigned char*>(d->args), static_cast<const unsigned char*>(d->args) + d->args_size);
  L->desc.args = nullptr;
  L->B = B;
  L->iters = k.desc.iters ? k.desc.iters : choose_iters(k, d, B);
  Launch& LL = *L;
  launches_[L->id] = std::move(L);
  *out = LL.id;
  Queue& Q = *qi->second;
  int rc = SLATE_OK;
  if (d->mode == SLATE_MODE_STANDALONE) {
    rc = issue(LL, Q, err);
  } else if (d->placement == SLATE_PLACE_CORUN) {
    const uint32_t old_lo = Q.lo, old_hi = Q.hi;
    if (!Q.active) {
      Q.active = true;
      active_.push_back(Q.id);
      rc = write_ctrl(Q, d->sm_lo, d->sm_hi, false, err);
      // co-runners yield the requested SMs (shrink on arrival)
      for (uint32_t other : active_) {
        if (other == Q.id) continue;
        Queue& A = *queues_[other];
        if (A.hi < d->sm_lo || A.lo > d->sm_hi) continue;
        const uint32_t left = d->sm_lo > A.lo ? d->sm_lo - A.lo : 0;     // [A.lo, sm_lo - 1]
        const uint32_t right = A.hi > d->sm_hi ? A.hi - d->sm_hi : 0;    // [sm_hi + 1, A.hi]
        if (!left && !right) continue;                                     // nothing left to keep: overlap
        const uint32_t nlo = left >= right ? A.lo : d->sm_hi + 1;
        const uint32_t nhi = left >= right ? d->sm_lo - 1 : A.hi;
        const double t0 = now_us();
        if (write_ctrl(A, nlo, nhi, true, err) == SLATE_OK && !A.issued.empty()) {
          Launch& R = *launches_[A.issued.front()];
          R.n_resizes += 1;
          track_resize(R, A.epoch, 1, t0);
        }
      }
    } else if (Q.lo != d->sm_lo || Q.hi != d->sm_hi) {
      rc = write_ctrl(Q, d->sm_lo, d->sm_hi, true, err);
      if (rc == SLATE_OK && (d->sm_lo < old_lo || d->sm_hi > old_hi)) rc = grow_running(Q, old_lo, old_hi, err);
    }
    Q.explicit_range = true;
    if (rc == SLATE_OK) rc = issue(LL, Q, err);
  } else if (Q.active) {
    rc = issue(LL, Q, err);
    if (rc == SLATE_OK && Q.auto_split && !defer) resplit();
  } else {
    Q.pending.push_back(LL.id);
    if (std::find(waiting_.begin(), waiting_.end(), Q.id) == waiting_.end()) waiting_.push_back(Q.id);
    if (!defer) schedule();
  }
  if (rc != SLATE_OK) fail_launch(LL, int(cudaErrorLaunchFailure));
  return rc;
}

// ------------------------------------------------------------------ scheduler
std::string Server::profile_key(const KernelEntry& k, const slate_launch_desc* d) const {
  std::ostringstream s;
  s << k.desc.kind << ':' << k.desc.iters << ':';
  const void* a = d->args;
  switch (k.desc.kind) {
    case SLATE_KIND_TRIAD: s << static_cast<const slate_args_triad*>(a)->n; break;
    case SLATE_KIND_COPY: s << static_cast<const slate_args_copy*>(a)->n; break;
    case SLATE_KIND_SGEMM_NAIVE: { auto x = static_cast<const slate_args_sgemm*>(a); s << x->m << 'x' << x->n << 'x' << x->k; break; }
    case SLATE_KIND_SPMV_CSR: { auto x = static_cast<const slate_args_spmv*>(a); s << x->n_rows << 'x' << x->n_cols; break; }
    case SLATE_KIND_BLACKSCHOLES: { auto x = static_cast<const slate_args_bs*>(a); s << x->n << 'p' << x->n_scen; break; }
    case SLATE_KIND_STENCIL2D: { auto x = static_cast<const slate_args_stencil*>(a); s << x->h << 'x' << x->w; break; }
    case SLATE_KIND_GEMM_BF16: { auto x = static_cast<const slate_args_gemm*>(a); s << x->m << 'x' << x->n << 'x' << x->k; break; }
    case SLATE_KIND_TRANSPOSE: { auto x = static_cast<const slate_args_transpose*>(a); s << x->h << 'x' << x->w; break; }
    case SLATE_KIND_SGEMM_TILED: { auto x = static_cast<const slate_args_sgemm*>(a); s << x->m << 'x' << x->n << 'x' << x->k; break; }
    case SLATE_KIND_QRNG: { auto x = static_cast<const slate_args_qrng*>(a); s << x->n << 'd' << x->dims; break; }
    // one profile per system size: the steps of one elimination share it
    case SLATE_KIND_GAUSS_FAN1:
    case SLATE_KIND_GAUSS_FAN2: s << static_cast<const slate_args_gauss*>(a)->n; break;
    case SLATE_KIND_USER: s << k.id << ':' << d->grid[0] << 'x' << d->grid[1] << 'x' << d->grid[2]; break;
  }
  return s.str();
}

int Server::category_of(const Launch& L) const {
  slate_launch_desc d = L.desc;
  d.args = L.args.data();
  auto it = profiles_.find(profile_key(*L.k, &d));
  return it == profiles_.end() ? -1 : int(it->second.p.category);
}

static const slate_profile_t* find_profile(const std::map<std::string, ProfileEntry>& t, const std::string& key) {
  auto it = t.find(key);
  return it == t.end() ? nullptr : &it->second.p;
}

// NEXT-4 (the task size trades scheduling overhead
// against imbalance and reaction time).  With a solo profile of the launch's
// kernel and shape, a worker's time per block is t = T_solo * workers / B;
// the task takes as many blocks as fit a budget (SLATE_TASK_BUDGET_US, default
// 20 us: a resize is honoured within two tasks, reading Q23, inside the 50-us
// target), at least one, at most the kind's cap, and leaves every worker at
// least two tasks.  Without a profile: the occupancy rule (auto_iters, Q11).
uint32_t Server::choose_iters(const KernelEntry& k, const slate_launch_desc* d, uint32_t B) const {
  const uint32_t cap = k.ops->max_auto_iters;
  const slate_profile_t* p = find_profile(profiles_, profile_key(k, d));
  if (!p || p->solo_ms <= 0) return auto_iters(B, k.occ, cap, k.ops->tasks_per_worker);
  return slate_choose_iters(p->solo_ms, uint32_t(k.occ), uint32_t(n_sms_), B, cap, task_budget_us_);
}

int Server::set_policy(uint32_t policy, std::string* err) {
  if (policy > SLATE_POLICY_HYBRID) {
    if (err) *err = "unknown policy";
    return SLATE_EINVAL;
  }
  std::lock_guard<std::mutex> g(mu_);
  policy_ = policy;
  return SLATE_OK;
}

int Server::set_split_objective(uint32_t objective, double slack, std::string* err) {
  if (objective > SLATE_SPLIT_ANTT || !(slack >= 0.0 && slack <= 1.0)) {
    if (err) *err = "unknown split objective or slack outside [0, 1]";
    return SLATE_EINVAL;
  }
  std::lock_guard<std::mutex> g(mu_);
  split_objective_ = objective;
  split_slack_ = slack;
  return SLATE_OK;
}

// the launch's solo curve from the profile table, ascending in SMs
bool Server::curve_of(const Launch& L, std::vector<uint32_t>* sms, std::vector<double>* ms) const {
  slate_launch_desc d = L.desc;
  d.args = L.args.data();
  const slate_profile_t* p = find_profile(profiles_, profile_key(*L.k, &d));
  if (!p || p->n_curve < 2) return false;
  sms->clear();
  ms->clear();
  for (int i = int(p->n_curve) - 1; i >= 0; --i) {   // stored in descending SM order
    sms->push_back(p->curve_sms[i]);
    ms->push_back(p->curve_ms[i]);
  }
  return true;
}

// SMs for B's queue (A keeps the rest) from the job curves of both queues:
// each queue's remaining launches (running + waiting) of its head kernel back
// to back (reading Q10 over jobs, Q31), with the Q29 saturation cap; n/2 when
// a curve is missing.  *gain = the predicted T_seq / T_corun.
uint32_t Server::pair_split(const Launch& LA, const Queue& A, const Launch& LB, const Queue& B, int catA, int catB,
                            double* gain) const {
  *gain = 0;
  std::vector<uint32_t> sa, sb;
  std::vector<double> ta, tb;
  if (!curve_of(LA, &sa, &ta) || !curve_of(LB, &sb, &tb)) return uint32_t(n_sms_ / 2);
  const bool memA = catA >= 3, memB = catB >= 3;
  uint32_t lo_b = 0, hi_b = 0;
  if (saturation_frac_ < 1.0 && memB && !memA)
    hi_b = slate_saturation_sms(sb.data(), tb.data(), uint32_t(sb.size()), uint32_t(n_sms_), saturation_frac_);
  if (saturation_frac_ < 1.0 && memA && !memB)
    lo_b = uint32_t(n_sms_) - slate_saturation_sms(sa.data(), ta.data(), uint32_t(sa.size()), uint32_t(n_sms_),
                                                   saturation_frac_);
  const double wa = double(std::max<size_t>(1, A.issued.size() + A.pending.size()));
  const double wb = double(std::max<size_t>(1, B.issued.size() + B.pending.size()));
  uint32_t s = uint32_t(n_sms_ / 2);
  slate_fluid_corun_obj(sa.data(), ta.data(), uint32_t(sa.size()), wa, sb.data(), tb.data(), uint32_t(sb.size()), wb,
                        uint32_t(n_sms_), 2, lo_b, hi_b, min_gain_, split_objective_, split_slack_, &s, gain);
  return s;
}

// ------------------------------------------------------------------ k-way co-runs (NEXT-4, reading Q49)
bool Server::job_curve(const Queue& Q, std::vector<uint32_t>* sms, std::vector<double>* ms) const {
  const uint64_t lid = !Q.pending.empty() ? Q.pending.front() : (!Q.issued.empty() ? Q.issued.back() : 0);
  if (!lid) return false;
  auto it = launches_.find(lid);
  if (it == launches_.end() || !curve_of(*it->second, sms, ms)) return false;
  const double work = double(std::max<size_t>(1, Q.issued.size() + Q.pending.size()));
  for (double& v : *ms) v *= work;
  return true;
}

// Contiguous ranges in `qids` order (the first queue on the low ranks).  Queues
// that only shrink are written first, so SMs are given up before they are
// granted; growing queues get top-ups for their running launch.
void Server::apply_shares(const std::vector<uint32_t>& qids, const std::vector<uint32_t>& shares) {
  std::string err;
  const double t0 = now_us();
  std::vector<uint32_t> lo(qids.size()), hi(qids.size());
  uint32_t at = 0;
  for (size_t i = 0; i < qids.size(); ++i) {
    lo[i] = at;
    hi[i] = at + shares[i] - 1;
    at += shares[i];
  }
  hi.back() = uint32_t(n_sms_ - 1);
  for (int pass = 0; pass < 2; ++pass) {
    for (size_t i = 0; i < qids.size(); ++i) {
      Queue& Q = *queues_[qids[i]];
      const bool grows = lo[i] < Q.lo || hi[i] > Q.hi || !Q.active;
      if ((pass == 0) == grows || (Q.lo == lo[i] && Q.hi == hi[i])) continue;
      const uint32_t old_lo = Q.lo, old_hi = Q.hi;
      write_ctrl(Q, lo[i], hi[i], true, &err);
      if (!Q.issued.empty()) {
        Launch& R = *launches_[grows ? Q.issued.back() : Q.issued.front()];
        R.n_resizes += 1;
        track_resize(R, Q.epoch, grows ? 2 : 1, t0);
      }
      if (grows) grow_running(Q, old_lo, old_hi, &err);
    }
  }
  if (qids.size() == 2) {   // the pair's re-split (resplit) keeps each on its side
    queues_[qids[0]]->low_side = true;
    queues_[qids[1]]->low_side = false;
  }
}

// A third co-runner (the selection "examines other kernels in the
// queue"): the head of the waiting queue joins a co-running group if the group
// keeps at most one memory-intensive job (Q37) and the fluid model predicts a
// gain against running it after the group (slate_kway_admit).
bool Server::try_admit_kway() {
  if (waiting_.empty() || active_.size() < 2 || active_.size() >= max_corun_) return false;
  std::vector<std::vector<uint32_t>> sms;
  std::vector<std::vector<double>> ms;
  std::vector<uint32_t> cats, shares_cur;
  for (uint32_t qid : active_) {
    const Queue& Q = *queues_[qid];
    if (!Q.auto_split || Q.explicit_range || Q.issued.empty()) return false;
    std::vector<uint32_t> s;
    std::vector<double> t;
    if (!job_curve(Q, &s, &t)) return false;
    const int c = category_of(*launches_[Q.issued.back()]);
    if (c < 0) return false;
    sms.push_back(s);
    ms.push_back(t);
    cats.push_back(uint32_t(c));
    shares_cur.push_back(Q.hi - Q.lo + 1);
  }
  const uint32_t cand = waiting_.front();
  Queue& C = *queues_[cand];
  if (C.pending.empty()) return false;
  const Launch& H = *launches_[C.pending.front()];
  if (H.desc.placement == SLATE_PLACE_SOLO) return false;
  const int cc = category_of(H);
  std::vector<uint32_t> s;
  std::vector<double> t;
  if (cc < 0 || !job_curve(C, &s, &t)) return false;
  sms.push_back(s);
  ms.push_back(t);
  cats.push_back(uint32_t(cc));
  std::vector<const uint32_t*> sp;
  std::vector<const double*> mp;
  std::vector<uint32_t> np;
  for (size_t i = 0; i < sms.size(); ++i) {
    sp.push_back(sms[i].data());
    mp.push_back(ms[i].data());
    np.push_back(uint32_t(sms[i].size()));
  }
  std::vector<uint32_t> shares(sms.size());
  double g = 0;
  const int admit = slate_kway_admit(sp.data(), mp.data(), np.data(), cats.data(), uint32_t(active_.size()),
                                     shares_cur.data(), uint32_t(n_sms_), 2, min_gain_, shares.data(), &g);
  if (std::getenv("SLATE_DEBUG"))
    fprintf(stderr, "[slate] k-way: candidate queue %u (cat %d) into a group of %zu: gain %.3f -> %s\n", cand, cc,
            active_.size(), g, admit ? "admit" : "wait");
  if (!admit) return false;
  waiting_.erase(std::find(waiting_.begin(), waiting_.end(), cand));
  bypassed_.erase(cand);
  std::vector<uint32_t> group(active_.begin(), active_.end());
  group.push_back(cand);
  apply_shares(group, shares);
  C.active = true;
  C.explicit_range = false;
  C.auto_split = true;
  active_.push_back(cand);
  std::string err;
  while (!C.pending.empty()) {
    Launch& L = *launches_[C.pending.front()];
    C.pending.pop_front();
    batch_more_ = !C.pending.empty();
    if (issue(L, C, &err) != SLATE_OK) fail_launch(L, int(cudaErrorLaunchFailure));
  }
  batch_more_ = false;
  close_batch(C, nullptr);
  return true;
}

// A co-running pair on the selector's split: as launches arrive the jobs
// grow, so the split is re-taken from the job curves; a change of >= 6 SMs
// resizes both queues (shrink one, grow the other).
void Server::resplit() {
  if (active_.size() > 2) {   // a k-way group: re-take the shares from the job curves (NEXT-4)
    std::vector<std::vector<uint32_t>> sms;
    std::vector<std::vector<double>> ms;
    std::vector<uint32_t> cur;
    for (uint32_t qid : active_) {
      const Queue& Q = *queues_[qid];
      if (!Q.auto_split || Q.explicit_range) return;
      std::vector<uint32_t> s;
      std::vector<double> t;
      if (!job_curve(Q, &s, &t)) return;
      sms.push_back(s);
      ms.push_back(t);
      cur.push_back(Q.hi - Q.lo + 1);
    }
    std::vector<const uint32_t*> sp;
    std::vector<const double*> mp;
    std::vector<uint32_t> np;
    for (size_t i = 0; i < sms.size(); ++i) {
      sp.push_back(sms[i].data());
      mp.push_back(ms[i].data());
      np.push_back(uint32_t(sms[i].size()));
    }
    std::vector<uint32_t> shares(sms.size());
    if (slate_choose_split_k(sp.data(), mp.data(), np.data(), uint32_t(sms.size()), uint32_t(n_sms_), 2,
                             shares.data()) <= 0)
      return;
    bool big = false;
    for (size_t i = 0; i < shares.size(); ++i) big = big || (shares[i] > cur[i] ? shares[i] - cur[i] : cur[i] - shares[i]) >= 6;
    if (big) apply_shares(active_, shares);
    return;
  }
  if (active_.size() != 2) return;
  Queue& A = *queues_[active_[0]];
  Queue& B = *queues_[active_[1]];
  if (!A.auto_split || !B.auto_split || A.explicit_range || B.explicit_range) return;
  const uint64_t la = !A.pending.empty() ? A.pending.front() : (!A.issued.empty() ? A.issued.back() : 0);
  const uint64_t lb = !B.pending.empty() ? B.pending.front() : (!B.issued.empty() ? B.issued.back() : 0);
  if (!la || !lb) return;
  const Launch& LA = *launches_[la];
  const Launch& LB = *launches_[lb];
  const int catA = category_of(LA), catB = category_of(LB);
  if (catA < 0 || catB < 0) return;
  double g = 0;
  const uint32_t s = pair_split(LA, A, LB, B, catA, catB, &g);
  const uint32_t cur = B.hi - B.lo + 1;   // B's SMs
  if ((s > cur ? s - cur : cur - s) < 6) return;
  if (std::getenv("SLATE_DEBUG"))
    fprintf(stderr, "[slate] resplit: B %u -> %u SMs (A work %zu, B work %zu, gain %.3f)\n", cur, s,
            A.issued.size() + A.pending.size(), B.issued.size() + B.pending.size(), g);
  std::string err;
  const uint32_t n = uint32_t(n_sms_);
  Queue& shrink = s > cur ? A : B;
  Queue& grow = s > cur ? B : A;
  const uint32_t g_lo = grow.lo, g_hi = grow.hi;
  const double t0 = now_us();
  // ranges for B holding s SMs on its side, A the rest
  const uint32_t b_lo = B.low_side ? 0 : n - s, b_hi = B.low_side ? s - 1 : n - 1;
  const uint32_t a_lo = B.low_side ? s : 0, a_hi = B.low_side ? n - 1 : n - s - 1;
  if (&shrink == &A) write_ctrl(A, a_lo, a_hi, true, &err);
  else write_ctrl(B, b_lo, b_hi, true, &err);
  if (!shrink.issued.empty()) {
    Launch& R = *launches_[shrink.issued.front()];
    R.n_resizes += 1;
    track_resize(R, shrink.epoch, 1, t0);
  }
  if (&grow == &A) write_ctrl(A, a_lo, a_hi, true, &err);
  else write_ctrl(B, b_lo, b_hi, true, &err);
  if (!grow.issued.empty()) {
    Launch& R = *launches_[grow.issued.back()];
    R.n_resizes += 1;
    track_resize(R, grow.epoch, 2, t0);
  }
  grow_running(grow, g_lo, g_hi, &err);
}

void Server::schedule() {
  std::string err;
  while (!waiting_.empty() && !profiling_) {
    if (active_.empty()) {
      const uint32_t qid = waiting_.front();
      waiting_.pop_front();
      bypassed_.erase(qid);
      Queue& Q = *queues_[qid];
      Q.active = true;
      Q.explicit_range = false;
      active_.push_back(qid);
      write_ctrl(Q, 0, uint32_t(n_sms_ - 1), false, &err);
      while (!Q.pending.empty()) {
        Launch& L = *launches_[Q.pending.front()];
        Q.pending.pop_front();
        batch_more_ = !Q.pending.empty();
        if (issue(L, Q, &err) != SLATE_OK) fail_launch(L, int(cudaErrorLaunchFailure));
      }
      batch_more_ = false;
      close_batch(Q, nullptr);
      continue;
    }
    if (active_.size() >= 2) {   // a co-running group: a k-way admission (NEXT-4), or wait
      if (!try_admit_kway()) break;
      continue;
    }
    Queue& A = *queues_[active_[0]];
    if (A.explicit_range) break;
    // the active kernel: the last launch issued on A (or pending on it)
    const Launch* LA = nullptr;
    if (!A.issued.empty()) LA = launches_[A.issued.back()].get();
    if (!LA || LA->desc.placement == SLATE_PLACE_SOLO) break;
    const int catA = category_of(*LA);
    if (catA < 0) break;
    std::vector<uint32_t> cats, byp;
    std::vector<uint32_t> qids;
    for (uint32_t qid : waiting_) {
      const Queue& W = *queues_[qid];
      const Launch& H = *launches_[W.pending.front()];
      const int c = (H.desc.placement == SLATE_PLACE_SOLO) ? -1 : category_of(H);
      cats.push_back(c < 0 ? 99u : uint32_t(c));   // unknown profile or SOLO: never complementary
      byp.push_back(bypassed_[qid]);
      qids.push_back(qid);
    }
    int idx = slate_select(uint32_t(catA), cats.data(), byp.data(), uint32_t(cats.size()), 4,
                           policy_ == SLATE_POLICY_LITERAL ? 1 : 0);
    uint32_t s = uint32_t(n_sms_ / 2);
    if (idx >= 0) {
      const Launch& HB = *launches_[queues_[qids[idx]]->pending.front()];
      double g = 0;
      s = pair_split(*LA, A, HB, *queues_[qids[idx]], catA, int(cats[idx]), &g);
    } else if (policy_ == SLATE_POLICY_HYBRID && cats[0] != 99u && (catA >= 3) != (cats[0] >= 3)) {
      // reading Q31: Tab I keeps the head of the queue waiting, but the measured
      // solo curves and the queued work predict a co-run gain of >= min_gain_.
      // Only for a memory-intensive tenant (M_M, H_M) beside a compute one
      // (Q37): solo curves do not see two memory tenants sharing HBM
      const Launch& HB = *launches_[queues_[qids[0]]->pending.front()];
      double g = 0;
      const uint32_t s0 = pair_split(*LA, A, HB, *queues_[qids[0]], catA, int(cats[0]), &g);
      if (g >= min_gain_) {
        idx = 0;
        s = s0;
      }
    }
    if (std::getenv("SLATE_DEBUG"))
      fprintf(stderr, "[slate] select: active cat %d, head cat %u, idx %d, split %u (A work %zu, B work %zu)\n", catA,
              cats[0], idx, s, A.issued.size() + A.pending.size(),
              idx >= 0 ? queues_[qids[idx]]->pending.size() : size_t(0));
    if (idx < 0) break;
    for (int i = 0; i < idx; ++i) bypassed_[qids[i]] += 1;
    Queue& Bq = *queues_[qids[idx]];
    const uint32_t old_lo = A.lo, old_hi = A.hi;
    const double t0 = now_us();
    // A keeps the side its running launch has workers on
    const uint32_t n = uint32_t(n_sms_);
    const bool a_high = !A.issued.empty() && overlap(A.cov_lo, A.cov_hi, s, n - 1) > overlap(A.cov_lo, A.cov_hi, 0, n - s - 1);
    A.low_side = !a_high;
    write_ctrl(A, a_high ? s : 0, a_high ? n - 1 : n - s - 1, true, &err);   // shrink the running kernel
    if (!A.issued.empty()) {
      Launch& R = *launches_[A.issued.front()];
      track_resize(R, A.epoch, 1, t0);
      R.n_resizes += 1;
    }
    (void)old_lo;
    (void)old_hi;
    waiting_.erase(std::find(waiting_.begin(), waiting_.end(), Bq.id));
    bypassed_.erase(Bq.id);
    Bq.active = true;
    Bq.explicit_range = false;
    A.auto_split = Bq.auto_split = true;
    Bq.low_side = a_high;
    active_.push_back(Bq.id);
    write_ctrl(Bq, a_high ? 0 : n - s, a_high ? s - 1 : n - 1, false, &err);
    while (!Bq.pending.empty()) {
      Launch& L = *launches_[Bq.pending.front()];
      Bq.pending.pop_front();
      batch_more_ = !Bq.pending.empty();
      if (issue(L, Bq, &err) != SLATE_OK) fail_launch(L, int(cudaErrorLaunchFailure));
    }
    batch_more_ = false;
    close_batch(Bq, nullptr);
    break;   // at most two co-runners (reading Q13)
  }
}

// the queue has nothing left: its SMs go to the co-runner
void Server::release(Queue& Q) {
  std::string err;
  const bool kway = active_.size() > 2;
  Q.active = false;
  Q.explicit_range = false;
  Q.auto_split = false;
  active_.erase(std::remove(active_.begin(), active_.end(), Q.id), active_.end());
  if (kway) {   // a k-way group loses a member: the others share its SMs, re-split from the job curves
    bool all_auto = true;
    for (uint32_t other : active_) all_auto = all_auto && queues_[other]->auto_split && !queues_[other]->explicit_range;
    if (all_auto) {
      std::vector<std::vector<uint32_t>> sms;
      std::vector<std::vector<double>> ms;
      bool ok = true;
      for (uint32_t other : active_) {
        std::vector<uint32_t> s;
        std::vector<double> t;
        ok = ok && job_curve(*queues_[other], &s, &t);
        sms.push_back(s);
        ms.push_back(t);
      }
      std::vector<uint32_t> shares(active_.size(), uint32_t(n_sms_) / uint32_t(active_.size()));
      if (ok) {
        std::vector<const uint32_t*> sp;
        std::vector<const double*> mp;
        std::vector<uint32_t> np;
        for (size_t i = 0; i < sms.size(); ++i) {
          sp.push_back(sms[i].data());
          mp.push_back(ms[i].data());
          np.push_back(uint32_t(sms[i].size()));
        }
        slate_choose_split_k(sp.data(), mp.data(), np.data(), uint32_t(sms.size()), uint32_t(n_sms_), 2,
                             shares.data());
      }
      apply_shares(active_, shares);
      schedule();
      return;
    }
  }
  for (uint32_t other : active_) queues_[other]->auto_split = false;
  if (active_.size() == 1) {
    // the survivor claims the released SMs, explicit placement or not
    Queue& A = *queues_[active_[0]];
    if (A.lo != 0 || A.hi != uint32_t(n_sms_ - 1)) {
      const uint32_t old_lo = A.lo, old_hi = A.hi;
      const double t0 = now_us();
      write_ctrl(A, 0, uint32_t(n_sms_ - 1), true, &err);
      if (!A.issued.empty()) {
        Launch& R = *launches_[A.issued.front()];
        track_resize(R, A.epoch, 2, t0);
        R.n_resizes += 1;
      }
      grow_running(A, old_lo, old_hi, &err);
    }
  }
  schedule();
}

int Server::resize(uint32_t q, uint64_t l, uint32_t lo, uint32_t hi, std::string* err) {
  if (lo > hi || hi >= uint32_t(n_sms_)) {
    if (err) *err = "bad SM range";
    return SLATE_EINVAL;
  }
  std::lock_guard<std::mutex> g(mu_);
  auto li = launches_.find(l);
  if (li == launches_.end() || li->second->queue != q) return SLATE_ENOTFOUND;
  Queue& Q = *queues_[q];
  Launch& L = *li->second;
  const uint32_t old_lo = Q.lo, old_hi = Q.hi;
  const bool shrink = lo > old_lo || hi < old_hi;
  const bool grow = lo < old_lo || hi > old_hi;
  const double t0 = now_us();
  int rc = write_ctrl(Q, lo, hi, true, err);
  if (rc != SLATE_OK) return rc;
  if (!Q.active) {
    Q.active = true;
    active_.push_back(Q.id);
  }
  Q.explicit_range = true;
  if (L.state == 2) return SLATE_DONE;
  // measure on the queue's running launch
  if (!Q.issued.empty()) {
    Launch& R = *launches_[Q.issued.front()];
    R.n_resizes += 1;
    if (shrink || grow) track_resize(R, Q.epoch, shrink ? 1 : 2, t0);
  }
  if (grow) rc = grow_running(Q, old_lo, old_hi, err);
  return rc;
}

// a resize applied while R runs: measured (Q30) for the first 16 of the launch
void Server::track_resize(Launch& R, uint32_t epoch, int kind, double t0) {
  Queue& Q = *queues_[R.queue];
  if (kind == 2) {
    // a grow re-admits ranks: a shrink still pending was overtaken before it
    // completed (its workers may now stay) -- it has no completion to time;
    // counted apart (n_superseded), not as a latency
    for (auto it = Q.pending_resize.begin(); it != Q.pending_resize.end();) {
      if (it->kind == 1 && it->epoch < epoch) {
        auto li = launches_.find(it->lid);
        if (li != launches_.end()) li->second->n_superseded += 1;
        it = Q.pending_resize.erase(it);
      } else {
        ++it;
      }
    }
  }
  if (R.resize_us.size() >= 16) return;
  const size_t fr = first_running(Q);
  const uint64_t run = fr < Q.issued.size() ? Q.issued[fr] : (Q.issued.empty() ? 0 : Q.issued.back());
  Q.pending_resize.push_back({epoch, kind, t0, R.id, int(R.resize_us.size()), run});
  R.resize_us.push_back(-1);
  R.resize_kind.push_back(uint8_t(kind));
}

// the full device time of a mirror word's low kMirrorNsBits bits: the value
// nearest the device clock's reading at host time t (us)
unsigned long long Server::unwrap_mirror_ns(unsigned long long w, double t) const {
  const unsigned long long mask = (1ull << kMirrorNsBits) - 1, low = w & mask;
  double dev_us = 0;
  if (!clk_base_ns_ || !host_to_dev_us(t, &dev_us)) return low;
  const long long ref = (long long)clk_base_ns_ + (long long)(dev_us * 1e3);
  long long full = (long long)((ref & ~(long long)mask) | (long long)low);
  const long long half = 1ll << (kMirrorNsBits - 1);
  if (full > ref + half) full -= 1ll << kMirrorNsBits;
  else if (full < ref - half) full += 1ll << kMirrorNsBits;
  return (unsigned long long)full;
}

// completion stamp (device ns) -> latency from the host's resize call (Q30)
void Server::record_resize(const Queue::PendingResize& pr, unsigned long long done_ns, double t) {
  auto li = launches_.find(pr.lid);
  if (li == launches_.end()) return;
  Launch& R = *li->second;
  double t0_dev;
  if (clk_base_ns_ && done_ns && host_to_dev_us(pr.t0_us, &t0_dev))
    R.resize_us[pr.idx] = std::max(0.0, double(int64_t(done_ns - clk_base_ns_)) * 1e-3 - t0_dev);
  else
    R.resize_us[pr.idx] = t - pr.t0_us;
  if (std::getenv("SLATE_DEBUG"))
    fprintf(stderr, "[slate] resize kind %d (%s) epoch %u of launch %llu (tenant kind %u, %u top-ups): %.3f us on the device clock, %.3f us host-observed\n",
            pr.kind, pr.kind == 1 ? "shrink" : "grow", pr.epoch, (unsigned long long)R.id, R.k->desc.kind,
            unsigned(R.n_topups), R.resize_us[pr.idx], t - pr.t0_us);
}

// A resize applies to the queue, whichever of its launches is running: a
// shrink ends when the launch holding workers outside the range has retired
// them (its mirror's shrink epoch) or has ended altogether (`ended`, its last
// block's stamp: later launches start inside the range); a grow ends when a
// worker of any of the queue's launches joined under the new epoch.
void Server::resolve_resizes(Queue& Q, double t, const Launch* ended) {
  for (auto it = Q.pending_resize.begin(); it != Q.pending_resize.end();) {
    unsigned long long done_ns = 0;
    bool done = false;
    // Only launches running at the call can stamp it: from the one that was
    // running then (recorded at the call; it may have finished since -- the
    // poller cannot run while a long launch_n holds the lock) onward -- not the
    // whole done prefix, which in a batch can be hundreds of launches long
    const size_t fr = first_running(Q);
    const size_t j0 = size_t(std::lower_bound(Q.issued.begin(), Q.issued.end(), it->run) - Q.issued.begin());
    for (size_t j = std::min(j0, fr); j < Q.issued.size(); ++j) {
      const Launch& L = *launches_[Q.issued[j]];
      if (L.slot < 0) continue;
      const HostMirror& m = h_mirror_[L.slot];
      const unsigned long long w = it->kind == 1 ? m.shrink : m.join;
      if (w && mirror_epoch(w) >= it->epoch) {
        done_ns = unwrap_mirror_ns(w, t);
        done = true;
        break;
      }
      if (it->kind == 1 && j >= fr) break;   // only the oldest running launch can hold out-of-range workers
    }
    bool via_end = false;
    if (!done && ended && it->kind == 1 && ended->slot >= 0) {
      // a launch that ended without retiring a worker ends the shrink -- but not
      // one that had ended before the call (a batch's finished members retire
      // together at the batch's end; their stamps predate the resize)
      const unsigned long long e = h_mirror_[ended->slot].done;
      double t0_dev;
      const bool before = clk_base_ns_ && e && host_to_dev_us(it->t0_us, &t0_dev) &&
                          double(int64_t(e - clk_base_ns_)) * 1e-3 < t0_dev;
      if (!before) {
        done_ns = e;
        done = via_end = true;
      }
    }
    if (done) {
      record_resize(*it, done_ns, t);
      if (std::getenv("SLATE_DEBUG") && via_end) fprintf(stderr, "[slate]   (resolved by the launch's end)\n");
      it = Q.pending_resize.erase(it);
    } else {
      ++it;
    }
  }
}

// ------------------------------------------------------------------ poller
bool Server::launch_done_events(Launch& L) {
  for (cudaEvent_t e : L.ev_done) {
    const cudaError_t r = cudaEventQuery(e);
    if (r == cudaErrorNotReady) return false;
    if (r != cudaSuccess) {   // sticky kernel error: the launch is over
      L.error = int(r);
      return true;
    }
  }
  return true;
}

void Server::poll_once() {
  const double t = now_us();
  std::vector<uint32_t> idle;
  for (auto& kv : queues_) {
    Queue& Q = *kv.second;
    if (!Q.pending_resize.empty()) resolve_resizes(Q, t, nullptr);
    while (!Q.issued.empty()) {
      Launch& L = *launches_[Q.issued.front()];
      if (!launch_done_events(L)) {
        // the server watchdog: a kernel cannot be preempted, but a
        // launch running past the limit is reported -- its syncs return
        // ECUDA instead of waiting forever (the context may be wedged)
        if (watchdog_us_ > 0 && !L.watchdog_fired && t - L.t_issue_us > watchdog_us_) {
          L.watchdog_fired = true;
          Q.watchdog = true;
          fprintf(stderr, "[slate] watchdog: launch %llu of queue %u running for %.1f s (limit %.1f s)\n",
                  (unsigned long long)L.id, Q.id, (t - L.t_issue_us) * 1e-6, watchdog_us_ * 1e-6);
          cv_.notify_all();
        }
        break;
      }
      if (!Q.pending_resize.empty()) resolve_resizes(Q, t, &L);
      if (L.slot >= 0) {
        std::memcpy(L.snapshot, h_snap_ + size_t(L.slot) * kTaskCtlHeader, kTaskCtlHeader);
        L.has_snapshot = true;
        free_slot(L.slot);
        L.slot = -1;
      }
      L.state = 2;
      finished_.push_back(L.id);
      if (L.error && !Q.first_error) Q.first_error = L.error;
      if (L.fused && Q.n_fused) Q.n_fused -= 1;
      Q.issued.pop_front();
      if (Q.issued.empty()) Q.topup_ends.clear();
      else {                      // the next launch starts now, on the queue's current range
        Q.cov_lo = Q.lo;
        Q.cov_hi = Q.hi;
      }
      cv_.notify_all();
    }
    if (Q.issued.empty()) Q.pending_resize.clear();   // nothing left to observe them on
    drain_deferred(Q);
    if (Q.active && Q.issued.empty() && Q.pending.empty() && Q.deferred.empty()) idle.push_back(Q.id);
  }
  flush_free();
  for (uint32_t q : idle) release(*queues_[q]);
  if (finished_.size() > 2 * keep_finished_) retire_finished();
}

void Server::poller_main() {
  cudaSetDevice(device_);
  std::unique_lock<std::mutex> g(mu_);
  while (!stop_) {
    bool busy = false;
    for (auto& kv : queues_)
      if (!kv.second->issued.empty() || !kv.second->deferred.empty()) busy = true;
    if (!busy) {
      cv_.wait_for(g, std::chrono::milliseconds(2));
      continue;
    }
    poll_once();
    g.unlock();
    std::this_thread::yield();
    g.lock();
  }
}

// ------------------------------------------------------------------ sync / query
int Server::sync(uint32_t q, uint64_t l, int64_t timeout_us, std::string* err, bool through_watchdog) {
  std::unique_lock<std::mutex> g(mu_);
  const auto deadline = std::chrono::steady_clock::now() + std::chrono::microseconds(timeout_us < 0 ? 0 : timeout_us);
  auto done = [&]() -> bool {
    if (l) {
      auto it = launches_.find(l);
      return it == launches_.end() || it->second->state == 2 || (it->second->watchdog_fired && !through_watchdog);
    }
    auto qi = queues_.find(q);
    return qi == queues_.end() || (qi->second->watchdog && !through_watchdog) ||
           (qi->second->issued.empty() && qi->second->pending.empty() && qi->second->deferred.empty());
  };
  // a launch id below the retention window completed long ago (ids are monotonic)
  if (l && launches_.find(l) == launches_.end()) return l < next_launch_id_ ? SLATE_OK : SLATE_ENOTFOUND;
  while (!done()) {
    if (timeout_us < 0) {
      cv_.wait_for(g, std::chrono::milliseconds(5));
    } else {
      if (std::chrono::steady_clock::now() >= deadline) {
        if (err) *err = "slate_sync timed out";
        return SLATE_ETIMEDOUT;
      }
      cv_.wait_until(g, std::min(deadline, std::chrono::steady_clock::now() + std::chrono::milliseconds(5)));
    }
  }
  int e = 0;   // per launch, or the queue's first error (no scan over every launch ever made)
  if (l) {
    auto it = launches_.find(l);
    if (it != launches_.end()) {
      e = it->second->error;
      if (it->second->watchdog_fired && !through_watchdog && it->second->state != 2) {
        if (err) *err = "watchdog: the launch ran longer than SLATE_WATCHDOG_S";
        return SLATE_ECUDA;
      }
    }
  } else {
    auto qi = queues_.find(q);
    if (qi != queues_.end()) {
      e = qi->second->first_error;
      if (!e && qi->second->watchdog && !through_watchdog) {
        if (err) *err = "watchdog: a launch of this session ran longer than SLATE_WATCHDOG_S";
        return SLATE_ECUDA;
      }
    }
  }
  if (e) {
    if (err) *err = std::string("CUDA error: ") + cudaGetErrorString(cudaError_t(e));
    return SLATE_ECUDA;
  }
  return SLATE_OK;
}

// Event times of a launch relative to the server's epoch event (ms).  A batch
// member (issued without events between kernels) is placed by its device
// stamps relative to the batch's first launch (workers: first task and last
// block), or, for original kernels, evenly between the batch's start and end.
void Server::launch_times(const Launch& L, double* start, double* end) const {
  auto ev_ms = [&](cudaEvent_t e) {
    float ms = 0;
    return (e && cudaEventElapsedTime(&ms, epoch_ev_, e) == cudaSuccess) ? double(ms) : -1.0;
  };
  auto snap = [](const Launch& X, unsigned long long* t0, unsigned long long* t1) {
    TaskCtl tc;
    std::memcpy(&tc, X.snapshot, kTaskCtlHeader);
    *t0 = tc.t_first;
    *t1 = tc.t_last;
    return X.has_snapshot && tc.t_first && tc.t_last;
  };
  if (L.fused && L.has_snapshot) {   // one tenant of a fused kernel: its own first task to its last block
    TaskCtl tc;
    std::memcpy(&tc, L.snapshot, kTaskCtlHeader);
    const double k0 = ev_ms(L.ev_start);
    if (k0 >= 0 && tc.t_enter && tc.t_first && tc.t_last) {
      *start = std::max(0.0, k0 + double(tc.t_first - tc.t_enter) * 1e-6);
      *end = std::max(*start, k0 + double(tc.t_last - tc.t_enter) * 1e-6);
      return;
    }
  }
  double s = ev_ms(L.ev_start ? L.ev_start : L.start_after), e = -1.0;
  for (cudaEvent_t x : L.ev_end) e = std::max(e, ev_ms(x));
  const Launch* F = &L;
  if (L.batch_first) {
    auto it = launches_.find(L.batch_first);
    if (it != launches_.end()) F = it->second.get();
  }
  if (s < 0 || e < 0) {
    const double fs = ev_ms(F->ev_start ? F->ev_start : F->start_after);
    unsigned long long f0, f1, l0, l1;
    if (snap(*F, &f0, &f1) && snap(L, &l0, &l1)) {                   // workers: device stamps
      const double off = fs - double(f0) * 1e-6;
      if (s < 0) s = off + double(l0) * 1e-6;
      if (e < 0) e = off + double(l1) * 1e-6;
    } else {                                                          // original kernels: evenly spread
      const double be = L.batch_end ? ev_ms(L.batch_end) : e;
      const double n = std::max(1u, L.batch_n), step = (be - fs) / n;
      if (s < 0) s = fs + step * L.batch_idx;
      if (e < 0) e = fs + step * (L.batch_idx + 1);
    }
  }
  *start = std::max(0.0, s);
  *end = std::max(*start, e);
}

int Server::query(uint64_t l, slate_launch_info* out, std::string* err) {
  std::unique_lock<std::mutex> g(mu_);
  auto it = launches_.find(l);
  if (it == launches_.end()) return SLATE_ENOTFOUND;
  Launch& L = *it->second;
  std::memset(out, 0, sizeof(*out));
  out->state = uint32_t(L.state);
  out->total_blocks = L.B;
  out->iters = L.iters;
  Queue* Q = queues_.count(L.queue) ? queues_[L.queue].get() : nullptr;
  if (Q) {
    out->sm_lo = Q->lo;
    out->sm_hi = Q->hi;
    out->epoch = Q->epoch;
  }
  out->n_resizes = L.n_resizes;
  out->n_topups = L.n_topups;
  for (int i = 0; i < 16; ++i) {
    out->resize_us[i] = i < int(L.resize_us.size()) ? L.resize_us[i] : -1.0;
    out->resize_kind[i] = i < int(L.resize_kind.size()) ? L.resize_kind[i] : 0;
  }
  TaskCtl tc;
  std::memset(&tc, 0, sizeof(tc));
  if (L.desc.mode == SLATE_MODE_STANDALONE) {
    if (L.state == 2) { out->blocks_done = L.B; }
  } else if (L.has_snapshot) {
    std::memcpy(&tc, L.snapshot, kTaskCtlHeader);
  } else if (L.slot >= 0) {
    CK(cudaMemcpyAsync(&tc, d_tc_ + L.slot, kTaskCtlHeader, cudaMemcpyDeviceToHost, copy_stream_));
    CK(cudaStreamSynchronize(copy_stream_));
  }
  if (L.desc.mode != SLATE_MODE_STANDALONE) {
    out->blocks_done = uint32_t(tc.done);
    out->tasks_done = uint32_t(tc.done >> 32);
    out->next_raw = tc.next;
    const uint64_t clamp = cdiv(L.B, L.iters) * L.iters;
    out->next_clamped = uint32_t(std::min<uint64_t>(tc.next, clamp));
    out->live_workers = uint32_t(tc.live_pending);
    out->workers_started = tc.started;
    out->t_first_ns = tc.t_first;
    out->t_last_ns = tc.t_last;
    out->shrink_epoch = tc.shrink_epoch;
    out->join_epoch = tc.join_epoch;
    out->t_enter_ns = tc.t_enter;
    out->n_superseded = L.n_superseded;
    out->t_exit_ns = tc.t_exit;
  }
  if (L.state == 2) {
    launch_times(L, &out->start_ms, &out->end_ms);
    if (L.desc.coverage) {
      std::vector<uint32_t> cov(L.B);
      CK(cudaMemcpyAsync(cov.data(), reinterpret_cast<void*>(L.desc.coverage), size_t(L.B) * 4, cudaMemcpyDeviceToHost,
                         copy_stream_));
      CK(cudaStreamSynchronize(copy_stream_));
      out->coverage_ok = std::all_of(cov.begin(), cov.end(), [](uint32_t v) { return v == 1; }) ? 1 : 0;
    }
  }
  return SLATE_OK;
}

// ------------------------------------------------------------------ profile
int Server::run_timed(const KernelEntry& k, const slate_launch_desc* d, uint32_t lo, uint32_t hi, int reps, double* ms,
                      std::string* err) {
  // a private queue: its own stream and resize word; kBatch control blocks.
  // A measurement is kBatch launches back to back (programmatic dependent
  // launch, no events between them, the early start where the kind allows it),
  // as a job's launches run: the per-launch time is the batch's span over kBatch.
  constexpr int kBatch = 16;
  std::vector<int> slots;
  uint64_t* ctrl;
  {
    std::lock_guard<std::mutex> g(mu_);
    while (int(slots.size()) < kBatch) {
      const int sl = alloc_slot();
      if (sl < 0) break;
      slots.push_back(sl);
    }
    if (int(slots.size()) < kBatch || free_ctrl_.empty()) {
      for (int sl : slots) free_slots_.push_back(sl);
      if (err) *err = "pool exhausted";
      return SLATE_ENOMEM;
    }
    ctrl = d_ctrl_pool_ + free_ctrl_.back() * 16;
    free_ctrl_.pop_back();
  }
  cudaStream_t st;
  CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  const uint64_t cv = pack_ctrl(1, lo, hi);
  CK(cudaMemcpyAsync(ctrl, &cv, 8, cudaMemcpyHostToDevice, st));
  uint32_t B = 0;
  validate(k, d, &B, nullptr);
  WorkerCommon w{};
  w.gx = d->grid[0]; w.gy = d->grid[1]; w.gz = d->grid[2]; w.B = B; w.occ = uint32_t(k.occ);
  w.iters = k.desc.iters ? k.desc.iters : auto_iters(B, k.occ, k.ops->max_auto_iters, k.ops->tasks_per_worker);
  w.bound_lo = 0; w.bound_hi = uint32_t(n_sms_ - 1); w.n_ranks = uint32_t(n_sms_);
  w.standby_timeout_ns = standby_timeout_ns_;
  w.ctrl = ctrl; w.mirror = nullptr; w.cov = nullptr; w.rank_of = d_rank_of_;
  w.ops = k.ops;
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  std::vector<double> times;
  for (int r = 0; r < reps + 1; ++r) {
    for (int sl : slots)
      CK(cudaMemcpyAsync(d_tc_ + sl, h_zero_, sizeof(TaskCtl), cudaMemcpyHostToDevice, st));
    CK(cudaEventRecord(e0, st));
    for (int i = 0; i < kBatch; ++i) {
      w.tc = d_tc_ + slots[i];
      w.pdl = i > 0 && k.ops->pdl_ok && pdl_enabled_;
      w.pdl_early = w.pdl && k.ops->pdl_early_ok && pdl_early_enabled_ &&
                    (!k.ops->outputs_disjoint || k.ops->outputs_disjoint(d->args)) ? 1u : 0u;
      CK(k.ops->launch_worker(w, d->args, worker_grid(k.occ, B, w.iters, lo == 0 && hi == uint32_t(n_sms_ - 1)), st));
    }
    CK(cudaEventRecord(e1, st));
    CK(cudaEventSynchronize(e1));
    float t;
    CK(cudaEventElapsedTime(&t, e0, e1));
    if (r > 0) times.push_back(t / kBatch);   // the first run warms up
  }
  std::sort(times.begin(), times.end());
  *ms = times[times.size() / 2];
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaStreamDestroy(st);
  std::lock_guard<std::mutex> g(mu_);
  for (int sl : slots) free_slot(sl);
  flush_free();
  free_ctrl_.push_back(int((ctrl - d_ctrl_pool_) / 16));
  return SLATE_OK;
}

int Server::profile(uint64_t kid, const slate_launch_desc* d, uint32_t flags, slate_profile_t* out, std::string* err) {
  const KernelEntry* kp;
  std::string key;
  {
    std::unique_lock<std::mutex> g(mu_);
    auto ki = kernels_.find(kid);
    if (ki == kernels_.end()) return SLATE_ENOTFOUND;
    kp = ki->second.get();
    uint32_t B;
    if (!validate(*kp, d, &B, err)) return SLATE_EINVAL;
    key = profile_key(*kp, d);
    auto pi = profiles_.find(key);
    if (pi != profiles_.end() && !(flags & SLATE_PROF_FORCE) &&
        (!(flags & SLATE_PROF_CURVE) || pi->second.p.n_curve > 1)) {
      *out = pi->second.p;
      return SLATE_OK;
    }
    // the profile needs the GPU to itself (P:L153 profiles are solo runs)
    cv_.wait(g, [&] { return active_.empty() && waiting_.empty() && !profiling_; });
    profiling_ = true;
  }
  slate_profile_t p{};
  double bytes, fp32, tc;
  work(*kp, d, &bytes, &fp32, &tc);
  p.bytes = bytes;
  p.flops = fp32 + tc;
  std::vector<uint32_t> pts = {uint32_t(n_sms_)};
  if (flags & SLATE_PROF_CURVE) {
    for (double f : {0.75, 0.5, 1.0 / 3.0, 0.25, 0.125}) pts.push_back(std::max<uint32_t>(1, uint32_t(std::lround(n_sms_ * f))));
  }
  int rc = SLATE_OK;
  for (size_t i = 0; i < pts.size() && rc == SLATE_OK; ++i) {
    double ms = 0;
    rc = run_timed(*kp, d, 0, pts[i] - 1, 3, &ms, err);
    p.curve_sms[i] = pts[i];
    p.curve_ms[i] = ms;
    p.n_curve = uint32_t(i + 1);
  }
  if (rc == SLATE_OK) {
    p.solo_ms = p.curve_ms[0];
    const double s = p.solo_ms * 1e-3;
    p.hbm_gbps = bytes / s / 1e9;
    p.fp32_gflops = fp32 / s / 1e9;
    p.tc_tflops = tc / s / 1e12;
    p.hbm_frac = p.hbm_gbps / peak_hbm_;
    p.fp32_frac = p.fp32_gflops / peak_fp32_;
    p.tc_frac = p.tc_tflops / peak_tc_;
    p.category = slate_classify(p.hbm_frac, p.fp32_frac, p.tc_frac, &p.c_level, &p.m_level);
  }
  std::lock_guard<std::mutex> g(mu_);
  profiling_ = false;
  if (rc == SLATE_OK) {
    profiles_[key].p = p;
    *out = p;
  }
  cv_.notify_all();
  schedule();
  return rc;
}

}  // namespace slate
