#include <algorithm>
// ipc.cu -- client side of the shared-memory transport (see ipc.h) and the
// per-kind pointer-field table used by the server to translate launch
// arguments.
#include <cstddef>
#include <cstring>
#include <thread>

#include <cuda.h>
#include <fcntl.h>
#include <signal.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <time.h>
#include <unistd.h>

#include "ipc.h"

namespace slate {

int pointer_fields(uint32_t kind, const size_t** offs) {
  static const size_t triad[] = {offsetof(slate_args_triad, a), offsetof(slate_args_triad, b),
                                 offsetof(slate_args_triad, c)};
  static const size_t copy[] = {offsetof(slate_args_copy, a), offsetof(slate_args_copy, b)};
  static const size_t sgemm[] = {offsetof(slate_args_sgemm, A), offsetof(slate_args_sgemm, B),
                                 offsetof(slate_args_sgemm, C)};
  static const size_t spmv[] = {offsetof(slate_args_spmv, rowptr), offsetof(slate_args_spmv, col),
                                offsetof(slate_args_spmv, val), offsetof(slate_args_spmv, x),
                                offsetof(slate_args_spmv, y)};
  static const size_t bs[] = {offsetof(slate_args_bs, S), offsetof(slate_args_bs, X), offsetof(slate_args_bs, T),
                              offsetof(slate_args_bs, call), offsetof(slate_args_bs, put),
                              offsetof(slate_args_bs, sigmas)};
  static const size_t stencil[] = {offsetof(slate_args_stencil, in), offsetof(slate_args_stencil, out)};
  static const size_t gemm[] = {offsetof(slate_args_gemm, A), offsetof(slate_args_gemm, B),
                                offsetof(slate_args_gemm, C)};
  static const size_t transpose[] = {offsetof(slate_args_transpose, in), offsetof(slate_args_transpose, out)};
  static const size_t qrng[] = {offsetof(slate_args_qrng, table), offsetof(slate_args_qrng, out)};
  static const size_t gauss[] = {offsetof(slate_args_gauss, a), offsetof(slate_args_gauss, b),
                                 offsetof(slate_args_gauss, m)};
  switch (kind) {
    case SLATE_KIND_TRIAD: *offs = triad; return 3;
    case SLATE_KIND_COPY: *offs = copy; return 2;
    case SLATE_KIND_SGEMM_NAIVE: *offs = sgemm; return 3;
    case SLATE_KIND_SPMV_CSR: *offs = spmv; return 5;
    case SLATE_KIND_BLACKSCHOLES: *offs = bs; return 6;
    case SLATE_KIND_STENCIL2D: *offs = stencil; return 2;
    case SLATE_KIND_GEMM_BF16: *offs = gemm; return 3;
    case SLATE_KIND_TRANSPOSE: *offs = transpose; return 2;
    case SLATE_KIND_SGEMM_TILED: *offs = sgemm; return 3;
    case SLATE_KIND_QRNG: *offs = qrng; return 2;
    case SLATE_KIND_GAUSS_FAN1: *offs = gauss; return 3;
    case SLATE_KIND_GAUSS_FAN2: *offs = gauss; return 3;
    default: *offs = nullptr; return 0;
  }
}

typedef CUresult (*GetAddressRangeFn)(CUdeviceptr*, size_t*, CUdeviceptr);

static double mono_us() {
  timespec ts;
  clock_gettime(CLOCK_MONOTONIC, &ts);
  return ts.tv_sec * 1e6 + ts.tv_nsec * 1e-3;
}

RemoteClient::RemoteClient() {}

RemoteClient::~RemoteClient() {
  if (shm_) munmap(shm_, sizeof(ShmLayout));
  if (fd_ >= 0) close(fd_);
}

int RemoteClient::connect(const char* endpoint, std::string* err) {
  fd_ = shm_open(endpoint, O_RDWR, 0);
  if (fd_ < 0) {
    if (err) *err = std::string("no slated server at ") + endpoint;
    return SLATE_EIPC;
  }
  void* p = mmap(nullptr, sizeof(ShmLayout), PROT_READ | PROT_WRITE, MAP_SHARED, fd_, 0);
  if (p == MAP_FAILED) {
    if (err) *err = "mmap of the endpoint failed";
    return SLATE_EIPC;
  }
  shm_ = static_cast<ShmLayout*>(p);
  if (shm_->hdr.magic != kShmMagic || shm_->hdr.version != kShmVersion || shm_->hdr.alive.load() != 1 ||
      kill(pid_t(shm_->hdr.server_pid), 0) != 0) {
    if (err) *err = "endpoint exists but no live slated server owns it";
    return SLATE_EIPC;
  }
  for (int i = 0; i < kSlots; ++i) {
    uint32_t expect = SLOT_FREE;
    if (shm_->slots[i].state.compare_exchange_strong(expect, SLOT_CLAIMED)) {
      slot_ = &shm_->slots[i];
      break;
    }
  }
  if (!slot_) {
    if (err) *err = "all session slots are taken";
    return SLATE_EIPC;
  }
  slot_->ack.store(0);
  slot_->client_pid = uint64_t(getpid());
  seq_ = slot_->req_seq.load();
  // the server's watcher gives the slot a session thread and a queue
  const double t0 = mono_us();
  while (slot_->state.load(std::memory_order_acquire) != SLOT_ACTIVE) {
    if (mono_us() - t0 > 10e6) {
      if (err) *err = "slated did not open the session";
      return SLATE_EIPC;
    }
    std::this_thread::sleep_for(std::chrono::microseconds(50));
  }
  return SLATE_OK;
}

int RemoteClient::call(Request& rq, Response* rs, std::string* err, bool long_wait) {
  if (!slot_) return SLATE_EIPC;
  std::memcpy(&slot_->req, &rq, sizeof(Request));
  const uint64_t seq = ++seq_;
  slot_->req_seq.store(seq, std::memory_order_release);
  const double t0 = mono_us();
  double last_check = t0;
  uint32_t spins = 0;
  while (slot_->resp_seq.load(std::memory_order_acquire) != seq) {
    if (++spins < 2000 && !long_wait) continue;
    const double now = mono_us();
    if (now - last_check > 100e3) {   // server gone?
      last_check = now;
      if (shm_->hdr.alive.load() != 1 || kill(pid_t(shm_->hdr.server_pid), 0) != 0) {
        if (err) *err = "slated server died";
        return SLATE_EIPC;
      }
    }
    std::this_thread::sleep_for(std::chrono::microseconds(now - t0 < 1000 ? 2 : 20));
  }
  std::memcpy(rs, &slot_->resp, sizeof(Response));
  if (rs->status < 0 && err) *err = rs->err;
  return rs->status;
}

int RemoteClient::detach(std::string* err) {
  Request rq{};
  rq.cmd = CMD_DETACH;
  Response rs;
  const int rc = call(rq, &rs, err, true);
  if (slot_) slot_->ack.store(1, std::memory_order_release);   // the server may now recycle the slot
  slot_ = nullptr;
  return rc;
}

int RemoteClient::info(slate_info* out, std::string* err) {
  Request rq{};
  rq.cmd = CMD_INFO;
  Response rs;
  const int rc = call(rq, &rs, err);
  if (rc == SLATE_OK) *out = rs.info;
  return rc;
}

int RemoteClient::share(uint64_t dev_ptr, size_t bytes, uint64_t* handle, std::string* err) {
  static GetAddressRangeFn range_fn = nullptr;
  if (!range_fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) != cudaSuccess || !f) {
      if (err) *err = "cuMemGetAddressRange unavailable";
      return SLATE_ECUDA;
    }
    range_fn = reinterpret_cast<GetAddressRangeFn>(f);
  }
  CUdeviceptr base = 0;
  size_t size = 0;
  if (range_fn(&base, &size, CUdeviceptr(dev_ptr)) != CUDA_SUCCESS || dev_ptr + bytes > base + size) {
    if (err) *err = "buffer is not inside one device allocation";
    return SLATE_EINVAL;
  }
  Request rq{};
  rq.cmd = CMD_SHARE;
  const cudaError_t e = cudaIpcGetMemHandle(&rq.handle, reinterpret_cast<void*>(base));
  if (e != cudaSuccess) {
    cudaGetLastError();
    if (err) *err = std::string("cudaIpcGetMemHandle: ") + cudaGetErrorString(e);
    return SLATE_EINVAL;
  }
  rq.alloc_base = uint64_t(base);
  rq.alloc_size = uint64_t(size);
  Response rs;
  const int rc = call(rq, &rs, err);
  if (rc == SLATE_OK) *handle = rs.out;
  return rc;
}

int RemoteClient::unshare(uint64_t handle, std::string* err) {
  Request rq{};
  rq.cmd = CMD_UNSHARE;
  rq.id = handle;
  Response rs;
  return call(rq, &rs, err);
}

int RemoteClient::register_kernel(const slate_kernel_desc* d, uint64_t* out, std::string* err) {
  Request rq{};
  rq.cmd = CMD_REGISTER;
  rq.kdesc = *d;
  Response rs;
  const int rc = call(rq, &rs, err);
  if (rc == SLATE_OK) *out = rs.out;
  return rc;
}

// NEXT-3 through an endpoint: the source in 256-byte chunks, then the registration
int RemoteClient::register_source(const slate_source_desc* d, uint64_t* out, std::string* err) {
  const size_t name_len = d->kernel_name ? std::strlen(d->kernel_name) : 0;
  if (!d->source || !d->kernel_name || name_len == 0 || name_len >= sizeof(SourceReg::name)) {
    if (err) *err = "need a source and a kernel name (< 192 characters)";
    return SLATE_EINVAL;
  }
  const size_t n = std::strlen(d->source);
  Response rs;
  for (size_t off = 0; off < n || off == 0; off += size_t(kMaxArgs)) {
    Request rq{};
    rq.cmd = CMD_SOURCE_CHUNK;
    rq.flags = off == 0 ? 1u : 0u;
    rq.lo = uint32_t(std::min(n - off, size_t(kMaxArgs)));
    std::memcpy(rq.args, d->source + off, rq.lo);
    const int rc = call(rq, &rs, err);
    if (rc != SLATE_OK) return rc;
    if (n == 0) break;
  }
  Request rq{};
  rq.cmd = CMD_REGISTER_SOURCE;
  SourceReg r{};
  r.bx = d->block_threads; r.by = d->block_y; r.bz = d->block_z; r.smem = d->smem_bytes;
  r.args_size = d->args_size; r.iters = d->iters; r.flags = d->flags;
  r.bytes_per_block = d->bytes_per_block; r.flops_per_block = d->flops_per_block;
  std::memcpy(r.name, d->kernel_name, name_len + 1);
  std::memcpy(rq.args, &r, sizeof(r));
  const int rc = call(rq, &rs, err, true);   // NVRTC: ~0.2 s on a cache miss
  if (rc == SLATE_OK) *out = rs.out;
  return rc;
}

static int pack_launch(Request& rq, const slate_launch_desc* d, std::string* err) {
  if (!d->args || d->args_size > uint32_t(kMaxArgs)) {
    if (err) *err = "args missing or too large";
    return SLATE_EINVAL;
  }
  rq.ldesc = *d;
  rq.ldesc.args = nullptr;
  std::memcpy(rq.args, d->args, d->args_size);
  return SLATE_OK;
}

int RemoteClient::launch(uint64_t k, const slate_launch_desc* d, uint64_t* out, std::string* err) {
  Request rq{};
  rq.cmd = CMD_LAUNCH;
  rq.id = k;
  int rc = pack_launch(rq, d, err);
  if (rc != SLATE_OK) return rc;
  Response rs;
  rc = call(rq, &rs, err);
  if (rc == SLATE_OK) *out = rs.out;
  return rc;
}

int RemoteClient::launch_n(uint64_t k, const slate_launch_desc* d, uint32_t n, uint64_t* first, std::string* err) {
  Request rq{};
  rq.cmd = CMD_LAUNCH;
  rq.id = k;
  rq.lo = n;   // launches in the batch (0 or 1: one)
  int rc = pack_launch(rq, d, err);
  if (rc != SLATE_OK) return rc;
  Response rs;
  rc = call(rq, &rs, err);
  if (rc == SLATE_OK) *first = rs.out;
  return rc;
}

int RemoteClient::resize(uint64_t l, uint32_t lo, uint32_t hi, std::string* err) {
  Request rq{};
  rq.cmd = CMD_RESIZE;
  rq.id = l;
  rq.lo = lo;
  rq.hi = hi;
  Response rs;
  return call(rq, &rs, err);
}

int RemoteClient::set_policy(uint32_t policy, std::string* err) {
  Request rq{};
  rq.cmd = CMD_POLICY;
  rq.lo = policy;
  Response rs;
  return call(rq, &rs, err);
}

int RemoteClient::set_split_objective(uint32_t objective, double slack, std::string* err) {
  Request rq{};
  rq.cmd = CMD_SPLIT;
  rq.lo = objective;
  std::memcpy(rq.args, &slack, sizeof(slack));
  Response rs;
  return call(rq, &rs, err);
}

int RemoteClient::sync(uint64_t l, int64_t timeout_us, std::string* err) {
  Request rq{};
  rq.cmd = CMD_SYNC;
  rq.id = l;
  rq.timeout_us = timeout_us;
  Response rs;
  return call(rq, &rs, err, true);
}

int RemoteClient::profile(uint64_t k, const slate_launch_desc* d, uint32_t flags, slate_profile_t* out,
                          std::string* err) {
  Request rq{};
  rq.cmd = CMD_PROFILE;
  rq.id = k;
  rq.flags = flags;
  int rc = pack_launch(rq, d, err);
  if (rc != SLATE_OK) return rc;
  Response rs;
  rc = call(rq, &rs, err, true);
  if (rc == SLATE_OK) *out = rs.prof;
  return rc;
}

int RemoteClient::query(uint64_t l, slate_launch_info* out, std::string* err) {
  Request rq{};
  rq.cmd = CMD_QUERY;
  rq.id = l;
  Response rs;
  const int rc = call(rq, &rs, err);
  if (rc == SLATE_OK) *out = rs.linfo;
  return rc;
}

}  // namespace slate
