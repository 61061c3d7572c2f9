// capi.cu -- the extern "C" boundary of libslate (include/slate.h).
// In-process sessions talk to a per-device Server directly; sessions attached
// to an endpoint go through the shared-memory transport (ipc.cu).
#include <cstdio>
#include <cstring>
#include <map>
#include <memory>
#include <cstdlib>
#include <mutex>
#include <string>
#include <vector>

#include "capi_internal.h"
#include "ipc.h"
#include "server.h"

using slate::Server;

struct slate_session {
  Server* srv = nullptr;                 // in-process
  std::unique_ptr<slate::RemoteClient> remote;   // through an endpoint
  uint32_t queue = 0;
  std::mutex mu;
  std::string last_error;
  struct Shared { uint64_t id, base, bytes; };
  std::vector<Shared> shared;
  uint64_t next_share = 1;
};

namespace slate {
static std::mutex g_servers_mu;
static std::map<int, Server*> g_servers;   // in-process servers live until process exit

// At exit: stop every server's threads before the CUDA runtime tears the
// context down (registered after the runtime's own handler, so it runs first).
static void stop_servers_at_exit() {
  static const bool trace = std::getenv("SLATE_EXIT_TRACE") != nullptr;
  if (trace) fprintf(stderr, "[slate] exit: stopping server threads\n");
  std::lock_guard<std::mutex> g(g_servers_mu);
  for (auto& kv : g_servers) kv.second->stop_threads();
  if (trace) {
    fprintf(stderr, "[slate] exit: server threads stopped\n");
    for (auto& kv : g_servers) kv.second->report_busy_streams(5000.0);
  }
}

Server* get_local_server(int device, std::string* err, int* rc) {
  std::lock_guard<std::mutex> g(g_servers_mu);
  auto it = g_servers.find(device);
  if (it != g_servers.end()) return it->second;
  Server* s = new Server(device);
  *rc = s->init(err);
  if (*rc != SLATE_OK) {
    delete s;
    return nullptr;
  }
  g_servers[device] = s;
  // registered once the runtime is initialised (init made CUDA calls), so the
  // handler runs before the runtime's teardown
  static const bool registered = (std::atexit(stop_servers_at_exit), true);
  (void)registered;
  return s;
}
}  // namespace slate

namespace {
slate_status fail(slate_session* s, slate_status rc, const std::string& msg) {
  if (s) s->last_error = msg;
  return rc;
}
}  // namespace

extern "C" {

const char* slate_status_string(slate_status st) {
  switch (st) {
    case SLATE_OK: return "SLATE_OK";
    case SLATE_DONE: return "SLATE_DONE";
    case SLATE_EINVAL: return "SLATE_EINVAL";
    case SLATE_ENOMEM: return "SLATE_ENOMEM";
    case SLATE_ECUDA: return "SLATE_ECUDA";
    case SLATE_EIPC: return "SLATE_EIPC";
    case SLATE_ETIMEDOUT: return "SLATE_ETIMEDOUT";
    case SLATE_ENOTFOUND: return "SLATE_ENOTFOUND";
    case SLATE_ESTATE: return "SLATE_ESTATE";
    case SLATE_EUNSUPPORTED: return "SLATE_EUNSUPPORTED";
    default: return "SLATE_UNKNOWN";
  }
}

const char* slate_last_error(slate_session* s) { return s ? s->last_error.c_str() : "no session"; }

slate_status slate_kind_geometry(uint32_t kind, uint32_t* tile_m, uint32_t* tile_n) {
  if (!tile_m || !tile_n) return SLATE_EINVAL;
  switch (kind) {
    case SLATE_KIND_TRIAD: *tile_m = 1; *tile_n = 1024; return SLATE_OK;
    case SLATE_KIND_COPY: *tile_m = 1; *tile_n = 4096; return SLATE_OK;
    case SLATE_KIND_SGEMM_NAIVE: *tile_m = 16; *tile_n = 16; return SLATE_OK;
    case SLATE_KIND_SPMV_CSR: *tile_m = 1; *tile_n = 32; return SLATE_OK;
    case SLATE_KIND_BLACKSCHOLES: *tile_m = 1; *tile_n = 1024; return SLATE_OK;
    case SLATE_KIND_STENCIL2D: *tile_m = 8; *tile_n = 128; return SLATE_OK;
    case SLATE_KIND_TRANSPOSE: *tile_m = 32; *tile_n = 32; return SLATE_OK;
    case SLATE_KIND_SGEMM_TILED: *tile_m = 32; *tile_n = 32; return SLATE_OK;
    case SLATE_KIND_QRNG: *tile_m = 1; *tile_n = 1024; return SLATE_OK;
    case SLATE_KIND_GAUSS_FAN1: *tile_m = 256; *tile_n = 1; return SLATE_OK;
    case SLATE_KIND_GAUSS_FAN2: *tile_m = 16; *tile_n = 128; return SLATE_OK;
    case SLATE_KIND_GEMM_BF16: {
      const slate::KindOps* o = slate::kind_ops(kind);
      *tile_m = o && o->tile_m ? o->tile_m : 128;
      *tile_n = o && o->tile_n ? o->tile_n : 128;
      return SLATE_OK;
    }
    default: return SLATE_EINVAL;
  }
}

slate_status slate_attach(const char* endpoint, int device, slate_session** out) {
  if (!out) return SLATE_EINVAL;
  *out = nullptr;
  auto s = std::make_unique<slate_session>();
  std::string err;
  int rc = SLATE_OK;
  if (endpoint == nullptr) {
    if (device < 0) return SLATE_EINVAL;
    s->srv = slate::get_local_server(device, &err, &rc);
    if (!s->srv) return rc;
    s->queue = s->srv->open_queue();
    if (!s->queue) return SLATE_ENOMEM;
  } else {
    s->remote = std::make_unique<slate::RemoteClient>();
    rc = s->remote->connect(endpoint, &err);
    if (rc != SLATE_OK) return rc;
  }
  *out = s.release();
  return SLATE_OK;
}

slate_status slate_detach(slate_session* s) {
  if (!s) return SLATE_EINVAL;
  std::string err;
  int rc = SLATE_OK;
  {
    std::lock_guard<std::mutex> g(s->mu);
    if (s->srv) rc = s->srv->close_queue(s->queue, 60000000, &err);
    else if (s->remote) rc = s->remote->detach(&err);
  }
  delete s;
  return rc;
}

slate_status slate_get_info(slate_session* s, slate_info* out) {
  if (!s || !out) return SLATE_EINVAL;
  std::lock_guard<std::mutex> g(s->mu);
  if (s->srv) {
    *out = s->srv->info();
    return SLATE_OK;
  }
  std::string err;
  const int rc = s->remote->info(out, &err);
  return rc == SLATE_OK ? rc : fail(s, rc, err);
}

slate_status slate_share_buffer(slate_session* s, void* ptr, size_t bytes, uint64_t* handle) {
  const uint64_t dev_ptr = reinterpret_cast<uint64_t>(ptr);
  if (!s || !handle || !dev_ptr || !bytes) return fail(s, SLATE_EINVAL, "null or empty buffer");
  std::lock_guard<std::mutex> g(s->mu);
  cudaPointerAttributes attr;
  if (cudaPointerGetAttributes(&attr, reinterpret_cast<void*>(dev_ptr)) != cudaSuccess ||
      attr.type != cudaMemoryTypeDevice) {
    cudaGetLastError();
    return fail(s, SLATE_EINVAL, "not device memory");
  }
  if (s->remote) {
    std::string err;
    const int rc = s->remote->share(dev_ptr, bytes, handle, &err);
    return rc == SLATE_OK ? rc : fail(s, rc, err);
  }
  *handle = s->next_share++;
  s->shared.push_back({*handle, dev_ptr, bytes});
  return SLATE_OK;
}

slate_status slate_unshare_buffer(slate_session* s, uint64_t handle) {
  if (!s) return SLATE_EINVAL;
  std::lock_guard<std::mutex> g(s->mu);
  if (s->remote) {
    std::string err;
    const int rc = s->remote->unshare(handle, &err);
    return rc == SLATE_OK ? rc : fail(s, rc, err);
  }
  for (size_t i = 0; i < s->shared.size(); ++i)
    if (s->shared[i].id == handle) {
      s->shared.erase(s->shared.begin() + long(i));
      return SLATE_OK;
    }
  return fail(s, SLATE_ENOTFOUND, "unknown buffer handle");
}

slate_status slate_register_kernel(slate_session* s, const slate_kernel_desc* d, slate_kernel* out) {
  if (!s || !d || !out) return fail(s, SLATE_EINVAL, "null argument");
  std::lock_guard<std::mutex> g(s->mu);
  std::string err;
  const int rc = s->srv ? s->srv->register_kernel(d, out, &err) : s->remote->register_kernel(d, out, &err);
  return rc == SLATE_OK ? rc : fail(s, rc, err);
}

slate_status slate_launch(slate_session* s, slate_kernel k, const slate_launch_desc* d, slate_launch_id* out) {
  if (!s || !d || !out) return fail(s, SLATE_EINVAL, "null argument");
  std::lock_guard<std::mutex> g(s->mu);
  std::string err;
  const int rc = s->srv ? s->srv->launch(s->queue, k, d, out, &err) : s->remote->launch(k, d, out, &err);
  return rc == SLATE_OK ? rc : fail(s, rc, err);
}

slate_status slate_launch_n(slate_session* s, slate_kernel k, const slate_launch_desc* d, uint32_t n,
                            slate_launch_id* first) {
  if (!s || !d || !first || n == 0) return fail(s, SLATE_EINVAL, "null argument or n == 0");
  std::lock_guard<std::mutex> g(s->mu);
  std::string err;
  const int rc = s->srv ? s->srv->launch_n(s->queue, k, d, n, first, &err) : s->remote->launch_n(k, d, n, first, &err);
  return rc == SLATE_OK ? rc : fail(s, rc, err);
}

slate_status slate_launch_many(slate_session* s, uint32_t n, const slate_kernel* ks, const slate_launch_desc* ds,
                               slate_launch_id* first) {
  if (!s || !ks || !ds || !first || n == 0) return fail(s, SLATE_EINVAL, "null argument or n == 0");
  std::lock_guard<std::mutex> g(s->mu);
  std::string err;
  int rc = SLATE_OK;
  if (s->srv) {
    rc = s->srv->launch_many(s->queue, n, ks, ds, first, &err);
  } else {
    for (uint32_t i = 0; i < n && rc == SLATE_OK; ++i) {
      slate_launch_id id = 0;
      rc = s->remote->launch(ks[i], &ds[i], &id, &err);
      if (i == 0) *first = id;
    }
  }
  return rc == SLATE_OK ? rc : fail(s, rc, err);
}

slate_status slate_register_source(slate_session* s, const slate_source_desc* d, slate_kernel* out) {
  if (!s || !d || !out) return fail(s, SLATE_EINVAL, "null argument");
  std::lock_guard<std::mutex> g(s->mu);
  std::string err;
  const int rc = s->srv ? s->srv->register_source(d, out, &err) : s->remote->register_source(d, out, &err);
  return rc == SLATE_OK ? rc : fail(s, rc, err);
}

slate_status slate_resize(slate_session* s, slate_launch_id l, uint32_t lo, uint32_t hi) {
  if (!s) return SLATE_EINVAL;
  std::lock_guard<std::mutex> g(s->mu);
  std::string err;
  const int rc = s->srv ? s->srv->resize(s->queue, l, lo, hi, &err) : s->remote->resize(l, lo, hi, &err);
  return rc >= SLATE_OK ? rc : fail(s, rc, err);
}

slate_status slate_set_policy(slate_session* s, uint32_t policy) {
  if (!s) return SLATE_EINVAL;
  std::lock_guard<std::mutex> g(s->mu);
  std::string err;
  const int rc = s->srv ? s->srv->set_policy(policy, &err) : s->remote->set_policy(policy, &err);
  return rc >= SLATE_OK ? rc : fail(s, rc, err);
}

slate_status slate_launch_fused(slate_session* sa, slate_kernel ka, const slate_launch_desc* da, slate_session* sb,
                                slate_kernel kb, const slate_launch_desc* db, uint32_t sm_b, slate_launch_id* la,
                                slate_launch_id* lb) {
  if (!sa || !sb || !da || !db || !la || !lb) return fail(sa, SLATE_EINVAL, "null argument");
  if (!sa->srv || sa->srv != sb->srv)
    return fail(sa, SLATE_EUNSUPPORTED, "a fused pair needs two in-process sessions of one server");
  std::scoped_lock g(sa->mu, sb->mu);
  std::string err;
  const int rc = sa->srv->launch_fused(sa->queue, ka, da, sb->queue, kb, db, sm_b, la, lb, &err);
  return rc == SLATE_OK ? rc : fail(sa, rc, err);
}

slate_status slate_set_split_objective(slate_session* s, uint32_t objective, double slack) {
  if (!s) return SLATE_EINVAL;
  std::lock_guard<std::mutex> g(s->mu);
  std::string err;
  const int rc = s->srv ? s->srv->set_split_objective(objective, slack, &err)
                        : s->remote->set_split_objective(objective, slack, &err);
  return rc >= SLATE_OK ? rc : fail(s, rc, err);
}

slate_status slate_sync(slate_session* s, slate_launch_id l, int64_t timeout_us) {
  if (!s) return SLATE_EINVAL;
  std::string err;
  // not under the session mutex: other threads may keep launching on the session
  const int rc = s->srv ? s->srv->sync(s->queue, l, timeout_us, &err) : s->remote->sync(l, timeout_us, &err);
  if (rc != SLATE_OK) {
    std::lock_guard<std::mutex> g(s->mu);
    return fail(s, rc, err);
  }
  return rc;
}

slate_status slate_profile(slate_session* s, slate_kernel k, const slate_launch_desc* d, uint32_t flags,
                           slate_profile_t* out) {
  if (!s || !d || !out) return fail(s, SLATE_EINVAL, "null argument");
  std::string err;
  const int rc = s->srv ? s->srv->profile(k, d, flags, out, &err) : s->remote->profile(k, d, flags, out, &err);
  if (rc != SLATE_OK) {
    std::lock_guard<std::mutex> g(s->mu);
    return fail(s, rc, err);
  }
  return rc;
}

slate_status slate_query(slate_session* s, slate_launch_id l, slate_launch_info* out) {
  if (!s || !out) return fail(s, SLATE_EINVAL, "null argument");
  std::string err;
  const int rc = s->srv ? s->srv->query(l, out, &err) : s->remote->query(l, out, &err);
  if (rc != SLATE_OK) {
    std::lock_guard<std::mutex> g(s->mu);
    return fail(s, rc, err);
  }
  return rc;
}

}  // extern "C"
