// serve.cu -- the `slated` server loop (slate_serve): one CUDA context per GPU
// for every client process (P:L135 context funnelling), one CPU thread per
// session, commands over the shared-memory slots of ipc.h, device
// buffers imported once per allocation through CUDA IPC and every pointer
// argument rewritten to the server's mapping.
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <thread>
#include <vector>

#include <fcntl.h>
#include <signal.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include "capi_internal.h"
#include "ipc.h"
#include "server.h"

namespace slate {
namespace {

volatile sig_atomic_t g_stop = 0;
const bool g_debug = std::getenv("SLATE_DEBUG") != nullptr;
#define DBG(...) do { if (g_debug) { std::fprintf(stderr, __VA_ARGS__); std::fflush(stderr); } } while (0)
void on_signal(int) { g_stop = 1; }

// server-wide cache of opened IPC allocations (a handle can be opened once per context).
// An allocation no session references any more (refs 0) is closed by the
// watcher thread (reap_ipc), never on a session's issue path, and never under
// g_ipc_mu: cudaIpcCloseMemHandle waits for the device and holds the driver
// while it does, so closing from a session thread while other tenants ran
// stalled every session's issue (no grows reached the running launches) for
// 12-360 ms at the end of C4 runs.  The reaper waits for an idle device, but
// only so long: an unreferenced mapping is closed anyway once it is older than
// kMaxUnrefAge or the unreferenced mappings exceed kMaxUnrefBytes, so memory of
// clients that left is given back under continuous load (the age is long: a
// close stalls every session's issue, so it should land between jobs).  Contract (slate.h):
// a client keeps a shared allocation alive until slate_unshare_buffer /
// slate_detach of it returned; the server's mapping goes within kMaxUnrefAge.
struct Opened {
  void* ptr;
  int refs;
  uint64_t bytes;
  std::chrono::steady_clock::time_point unref_since;
};
std::mutex g_ipc_mu;      // the map
std::mutex g_ipc_close_mu;  // held while mappings are being closed (and by an open of a new handle)
std::map<std::string, Opened> g_ipc;
constexpr auto kMaxUnrefAge = std::chrono::seconds(30);   // 0.5 s closed C4's buffers mid-run (steps 41 -> 61 ms)
constexpr uint64_t kMaxUnrefBytes = 8ull << 30;

void unref_ipc_locked(const std::string& key) {
  auto it = g_ipc.find(key);
  if (it != g_ipc.end() && it->second.refs > 0 && --it->second.refs == 0)
    it->second.unref_since = std::chrono::steady_clock::now();
}

void reap_ipc(Server* srv, bool force) {
  std::lock_guard<std::mutex> gc(g_ipc_close_mu);
  std::vector<void*> close_now;
  {
    std::lock_guard<std::mutex> g(g_ipc_mu);
    const auto now = std::chrono::steady_clock::now();
    uint64_t unref_bytes = 0;
    bool any = false, old = false;
    for (const auto& kv : g_ipc)
      if (kv.second.refs == 0) {
        any = true;
        unref_bytes += kv.second.bytes;
        old = old || now - kv.second.unref_since > kMaxUnrefAge;
      }
    if (!any) return;
    const bool go = force || old || unref_bytes > kMaxUnrefBytes || !srv->busy();
    if (!go) return;
    for (auto it = g_ipc.begin(); it != g_ipc.end();) {
      if (it->second.refs == 0) {
        close_now.push_back(it->second.ptr);
        it = g_ipc.erase(it);
      } else {
        ++it;
      }
    }
  }
  for (void* p : close_now) cudaIpcCloseMemHandle(p);   // outside g_ipc_mu: sessions keep issuing
}

struct Import {
  uint64_t id, client_base, size;
  char* server_base;
  std::string key;
};

class Session {
 public:
  Session(Server* srv, Slot* slot, int device) : srv_(srv), slot_(slot), device_(device) {}
  void run();

 private:
  int handle(const Request& rq, Response& rs);
  bool translate(uint64_t& p, std::string* err) const;
  void release_imports();
  Server* srv_;
  Slot* slot_;
  int device_;
  uint32_t queue_ = 0;
  std::string source_;   // a user kernel's source being received (CMD_SOURCE_CHUNK)
  std::vector<Import> imports_;
  uint64_t next_import_ = 1;
};

bool Session::translate(uint64_t& p, std::string* err) const {
  if (p == 0) return true;
  for (const Import& im : imports_)
    if (p >= im.client_base && p < im.client_base + im.size) {
      p = reinterpret_cast<uint64_t>(im.server_base) + (p - im.client_base);
      return true;
    }
  if (err) *err = "device pointer outside every shared buffer (slate_share_buffer it first)";
  return false;
}

void Session::release_imports() {
  std::lock_guard<std::mutex> g(g_ipc_mu);
  for (const Import& im : imports_) unref_ipc_locked(im.key);   // closed by reap_ipc
  imports_.clear();
}

int Session::handle(const Request& rq, Response& rs) {
  std::string err;
  int rc = SLATE_OK;
  DBG("slated[q%u]: cmd %u id %llu\n", queue_, rq.cmd, (unsigned long long)rq.id);
  switch (rq.cmd) {
    case CMD_INFO:
      rs.info = srv_->info();
      rs.info.server_pid = uint64_t(getpid());
      break;
    case CMD_SHARE: {
      std::string key(reinterpret_cast<const char*>(&rq.handle), sizeof(rq.handle));
      void* ptr = nullptr;
      {
        std::unique_lock<std::mutex> gc(g_ipc_close_mu, std::defer_lock);
        std::unique_lock<std::mutex> g(g_ipc_mu);
        if (g_ipc.find(key) == g_ipc.end()) {   // a new mapping: not while the reaper closes (lock order close -> map)
          g.unlock();
          gc.lock();
          g.lock();
        }
        auto it = g_ipc.find(key);
        if (it != g_ipc.end()) {
          it->second.refs += 1;
          ptr = it->second.ptr;
        } else {
          const cudaError_t e = cudaIpcOpenMemHandle(&ptr, rq.handle, cudaIpcMemLazyEnablePeerAccess);
          if (e != cudaSuccess) {
            cudaGetLastError();
            err = std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e);
            rc = SLATE_EIPC;
            break;
          }
          g_ipc[key] = {ptr, 1, rq.alloc_size, std::chrono::steady_clock::time_point()};
        }
      }
      imports_.push_back({next_import_, rq.alloc_base, rq.alloc_size, static_cast<char*>(ptr), key});
      rs.out = next_import_++;
      break;
    }
    case CMD_UNSHARE: {
      rc = SLATE_ENOTFOUND;
      for (size_t i = 0; i < imports_.size(); ++i)
        if (imports_[i].id == rq.id) {
          {
            std::lock_guard<std::mutex> g(g_ipc_mu);
            unref_ipc_locked(imports_[i].key);
          }
          imports_.erase(imports_.begin() + long(i));
          rc = SLATE_OK;
          break;
        }
      break;
    }
    case CMD_REGISTER:
      rc = srv_->register_kernel(&rq.kdesc, &rs.out, &err);
      break;
    case CMD_SOURCE_CHUNK:
      if (rq.flags & 1) source_.clear();
      if (rq.lo > uint32_t(kMaxArgs) || source_.size() + rq.lo > (16u << 20)) {
        rc = SLATE_EINVAL;
        err = "source chunk too large (a source is at most 16 MiB)";
        break;
      }
      source_.append(reinterpret_cast<const char*>(rq.args), rq.lo);
      break;
    case CMD_REGISTER_SOURCE: {
      SourceReg r;
      std::memcpy(&r, rq.args, sizeof(r));
      r.name[sizeof(r.name) - 1] = 0;
      slate_source_desc d{};
      d.abi_version = SLATE_ABI_VERSION;
      d.block_threads = r.bx; d.block_y = r.by; d.block_z = r.bz;
      d.smem_bytes = r.smem; d.args_size = r.args_size; d.iters = r.iters; d.flags = r.flags;
      d.source = source_.c_str();
      d.kernel_name = r.name;
      d.bytes_per_block = r.bytes_per_block; d.flops_per_block = r.flops_per_block;
      rc = srv_->register_source(&d, &rs.out, &err);
      source_.clear();
      break;
    }
    case CMD_LAUNCH:
    case CMD_PROFILE: {
      // rewrite every pointer argument into the server's address space
      unsigned char args[kMaxArgs];
      std::memcpy(args, rq.args, sizeof(args));
      slate_launch_desc d = rq.ldesc;
      d.args = args;
      uint32_t kind = 0;
      if (!srv_->kernel_kind(rq.id, &kind)) {
        rc = SLATE_ENOTFOUND;
        err = "unknown kernel";
        break;
      }
      const size_t* offs;
      int nf = pointer_fields(kind, &offs);
      std::vector<size_t> user_offs;   // a runtime-compiled kernel: its own pointer parameters
      if (kind == SLATE_KIND_USER && srv_->kernel_ptr_fields(rq.id, &user_offs)) {
        offs = user_offs.data();
        nf = int(user_offs.size());
      }
      bool ok = d.args_size <= sizeof(args);
      for (int i = 0; ok && i < nf; ++i) ok = offs[i] + 8 <= d.args_size;
      if (!ok && err.empty()) err = "argument block smaller than the kernel's pointer parameters";
      for (int i = 0; ok && i < nf; ++i) {
        uint64_t p;
        std::memcpy(&p, args + offs[i], 8);
        ok = translate(p, &err);
        std::memcpy(args + offs[i], &p, 8);
      }
      if (ok) ok = translate(d.coverage, &err);
      if (!ok) {
        rc = SLATE_EINVAL;
        break;
      }
      if (rq.cmd == CMD_LAUNCH && rq.lo > 1) rc = srv_->launch_n(queue_, rq.id, &d, rq.lo, &rs.out, &err);
      else if (rq.cmd == CMD_LAUNCH) rc = srv_->launch(queue_, rq.id, &d, &rs.out, &err);
      else rc = srv_->profile(rq.id, &d, rq.flags, &rs.prof, &err);
      break;
    }
    case CMD_RESIZE:
      rc = srv_->resize(queue_, rq.id, rq.lo, rq.hi, &err);
      break;
    case CMD_SYNC:
      rc = srv_->sync(queue_, rq.id, rq.timeout_us, &err);
      break;
    case CMD_POLICY:
      rc = srv_->set_policy(rq.lo, &err);
      break;
    case CMD_SPLIT: {
      double slack;
      std::memcpy(&slack, rq.args, sizeof(slack));
      rc = srv_->set_split_objective(rq.lo, slack, &err);
      break;
    }
    case CMD_QUERY:
      rc = srv_->query(rq.id, &rs.linfo, &err);
      break;
    default:
      rc = SLATE_EINVAL;
      err = "unknown command";
  }
  rs.status = rc;
  DBG("slated[q%u]: cmd %u -> %d %s\n", queue_, rq.cmd, rc, err.c_str());
  std::strncpy(rs.err, err.c_str(), sizeof(rs.err) - 1);
  rs.err[sizeof(rs.err) - 1] = 0;
  return rc;
}

void Session::run() {
  cudaSetDevice(device_);
  queue_ = srv_->open_queue();
  DBG("slated: session for pid %llu -> queue %u\n", (unsigned long long)slot_->client_pid, queue_);
  uint64_t last = slot_->req_seq.load();
  slot_->resp_seq.store(last);
  slot_->state.store(queue_ ? SLOT_ACTIVE : SLOT_CLOSING, std::memory_order_release);
  auto idle_since = std::chrono::steady_clock::now();
  auto last_check = idle_since;
  bool detached = false;
  while (!g_stop && queue_) {
    const uint64_t seq = slot_->req_seq.load(std::memory_order_acquire);
    if (seq != last) {
      Request rq;
      std::memcpy(&rq, &slot_->req, sizeof(Request));
      Response rs;
      std::memset(&rs, 0, sizeof(rs));
      if (rq.cmd == CMD_DETACH) {
        std::string err;
        const auto t0 = std::chrono::steady_clock::now();
        rs.status = srv_->close_queue(queue_, 60000000, &err);
        const auto t1 = std::chrono::steady_clock::now();
        release_imports();
        const auto t2 = std::chrono::steady_clock::now();
        if (getenv("SLATE_CLOSE_TIMING"))
          fprintf(stderr, "slated[q%u]: detach close %.3f ms, release %.3f ms\n", queue_,
                  std::chrono::duration<double, std::milli>(t1 - t0).count(),
                  std::chrono::duration<double, std::milli>(t2 - t1).count());
        detached = true;
      } else {
        handle(rq, rs);
      }
      std::memcpy(&slot_->resp, &rs, sizeof(Response));
      last = seq;
      slot_->resp_seq.store(seq, std::memory_order_release);
      idle_since = std::chrono::steady_clock::now();
      if (detached) break;
      continue;
    }
    const auto now = std::chrono::steady_clock::now();
    if (now - last_check > std::chrono::milliseconds(100)) {   // client gone: clean up its session
      last_check = now;
      if (kill(pid_t(slot_->client_pid), 0) != 0) break;
    }
    if (now - idle_since < std::chrono::microseconds(200)) std::this_thread::yield();
    else std::this_thread::sleep_for(std::chrono::microseconds(20));
  }
  if (!detached && queue_) {
    std::string err;
    const auto t0 = std::chrono::steady_clock::now();
    srv_->close_queue(queue_, 60000000, &err);
    const auto t1 = std::chrono::steady_clock::now();
    release_imports();
    const auto t2 = std::chrono::steady_clock::now();
    if (getenv("SLATE_CLOSE_TIMING"))
      fprintf(stderr, "slated[q%u]: close %.3f ms, release %.3f ms\n", queue_,
              std::chrono::duration<double, std::milli>(t1 - t0).count(),
              std::chrono::duration<double, std::milli>(t2 - t1).count());
  }
  if (detached) {   // the client is reading its DETACH response: wait for its ack (or its exit)
    const auto t0 = std::chrono::steady_clock::now();
    while (!slot_->ack.load(std::memory_order_acquire) && kill(pid_t(slot_->client_pid), 0) == 0 &&
           std::chrono::steady_clock::now() - t0 < std::chrono::seconds(5))
      std::this_thread::sleep_for(std::chrono::microseconds(50));
  }
  DBG("slated: session of pid %llu closed (queue %u)\n", (unsigned long long)slot_->client_pid, queue_);
  // sequence numbers are never reset: the next client starts from the current value
  slot_->client_pid = 0;
  slot_->state.store(SLOT_FREE, std::memory_order_release);
}

}  // namespace
}  // namespace slate

extern "C" slate_status slate_serve(const char* endpoint, int device, uint32_t flags) {
  using namespace slate;
  (void)flags;
  if (!endpoint || endpoint[0] != '/') return SLATE_EINVAL;
  std::string err;
  int rc = SLATE_OK;
  Server* srv = get_local_server(device, &err, &rc);
  if (!srv) {
    fprintf(stderr, "slated: %s\n", err.c_str());
    return rc;
  }
  shm_unlink(endpoint);
  const int fd = shm_open(endpoint, O_CREAT | O_RDWR | O_EXCL, 0666);
  if (fd < 0 || ftruncate(fd, sizeof(ShmLayout)) != 0) return SLATE_EIPC;
  void* p = mmap(nullptr, sizeof(ShmLayout), PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  if (p == MAP_FAILED) return SLATE_EIPC;
  std::memset(p, 0, sizeof(ShmLayout));
  ShmLayout* shm = new (p) ShmLayout();
  shm->hdr.magic = kShmMagic;
  shm->hdr.version = kShmVersion;
  shm->hdr.nslots = kSlots;
  shm->hdr.server_pid = uint64_t(getpid());
  shm->hdr.info = srv->info();
  shm->hdr.info.server_pid = uint64_t(getpid());
  signal(SIGINT, on_signal);
  signal(SIGTERM, on_signal);
  shm->hdr.alive.store(1, std::memory_order_release);
  fprintf(stderr, "slated: serving %s on device %d (%u SMs)\n", endpoint, device, srv->info().num_sms);
  std::vector<std::thread> threads;
  uint32_t tick = 0;
  while (!g_stop) {
    for (int i = 0; i < kSlots; ++i) {
      Slot& s = shm->slots[i];
      if (s.state.load(std::memory_order_acquire) == SLOT_CLAIMED && s.client_pid) {
        s.state.store(SLOT_CLOSING);   // owned by the watcher until the session thread opens it
        DBG("slated: slot %d claimed by pid %llu\n", i, (unsigned long long)s.client_pid);
        threads.emplace_back([srv, &s, device] { Session(srv, &s, device).run(); });
      }
    }
    if (++tick % 256 == 0) reap_ipc(srv, false);   // ~every 50 ms
    std::this_thread::sleep_for(std::chrono::microseconds(200));
  }
  shm->hdr.alive.store(0);
  for (auto& t : threads) t.join();
  reap_ipc(srv, true);
  munmap(p, sizeof(ShmLayout));
  close(fd);
  shm_unlink(endpoint);
  return SLATE_OK;
}
