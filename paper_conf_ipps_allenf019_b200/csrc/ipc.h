// ipc.h -- the shared-memory transport between client processes and a `slated`
// server (§IV-A: client library + daemon funnelling every client's
// kernels into ONE CUDA context; commands on a fast channel, kernel IO
// data in buffers shared between client and daemon).
//
// Layout of the POSIX shared-memory object named by the endpoint (e.g.
// "/slate-gpu0"): a header, then kSlots session slots.  A client claims a free
// slot with a CAS, the server's watcher gives the slot a session thread (one
// CPU thread per session) and a queue; each request/response is a
// sequence-numbered exchange in the slot (release/acquire on the sequence
// numbers, spin-then-sleep polling on both sides).  Device buffers travel as
// cudaIpcMemHandle_t; the server opens each allocation once and rewrites every
// pointer argument of a launch from the client's address space to its own
// mapping (the paper's shared-buffer -> GPU-pointer hash table).
#pragma once
#include <atomic>
#include <cstdint>
#include <string>
#include <cuda_runtime.h>
#include "../../include/slate.h"

namespace slate {

constexpr uint64_t kShmMagic = 0x534c415445495043ull;   // "SLATEIPC"
constexpr uint32_t kShmVersion = 1;
constexpr int kSlots = 64;
constexpr int kMaxArgs = 256;

enum Cmd : uint32_t {
  CMD_NONE = 0, CMD_INFO, CMD_SHARE, CMD_UNSHARE, CMD_REGISTER, CMD_LAUNCH, CMD_RESIZE, CMD_SYNC, CMD_PROFILE,
  CMD_QUERY, CMD_DETACH, CMD_POLICY,
  CMD_SOURCE_CHUNK,        // append args[0, lo) to the session's source buffer (flags & 1: start a new one)
  CMD_REGISTER_SOURCE,     // compile the buffered source: args holds a SourceReg (NEXT-3 through an endpoint)
  CMD_SPLIT                // the split objective: lo = objective, args = the slack (double)
};

// CMD_REGISTER_SOURCE's argument block (slate_source_desc without the strings)
struct SourceReg {
  uint32_t bx, by, bz, smem, args_size, iters, flags, pad;
  double bytes_per_block, flops_per_block;
  char name[192];
};
static_assert(sizeof(SourceReg) <= 256, "fits Request::args");

struct Request {
  uint32_t cmd;
  uint32_t flags;
  uint64_t id;             // kernel or launch handle / buffer handle
  uint32_t lo, hi;
  int64_t timeout_us;
  slate_kernel_desc kdesc;
  slate_launch_desc ldesc; // .args ignored: the blob is in args[]
  unsigned char args[kMaxArgs];
  cudaIpcMemHandle_t handle;
  uint64_t alloc_base, alloc_size;   // the client's allocation (SHARE)
};

struct Response {
  int32_t status;
  char err[240];
  uint64_t out;
  slate_info info;
  slate_profile_t prof;
  slate_launch_info linfo;
};

enum SlotState : uint32_t { SLOT_FREE = 0, SLOT_CLAIMED = 1, SLOT_ACTIVE = 2, SLOT_CLOSING = 3 };

struct alignas(128) Slot {
  std::atomic<uint32_t> state;
  std::atomic<uint32_t> ack;      // client read its DETACH response; the slot may be recycled
  std::atomic<uint64_t> req_seq;
  std::atomic<uint64_t> resp_seq;
  uint64_t client_pid;
  Request req;
  Response resp;
};

struct alignas(128) ShmHeader {
  uint64_t magic;
  uint32_t version;
  uint32_t nslots;
  uint64_t server_pid;
  std::atomic<uint32_t> alive;
  uint32_t pad;
  slate_info info;
};

struct ShmLayout {
  ShmHeader hdr;
  Slot slots[kSlots];
};

// byte offsets of the device-pointer fields of a kind's argument block
int pointer_fields(uint32_t kind, const size_t** offs);

class RemoteClient {
 public:
  RemoteClient();
  ~RemoteClient();
  int connect(const char* endpoint, std::string* err);
  int detach(std::string* err);
  int info(slate_info* out, std::string* err);
  int share(uint64_t dev_ptr, size_t bytes, uint64_t* handle, std::string* err);
  int unshare(uint64_t handle, std::string* err);
  int register_kernel(const slate_kernel_desc* d, uint64_t* out, std::string* err);
  int register_source(const slate_source_desc* d, uint64_t* out, std::string* err);
  int launch(uint64_t k, const slate_launch_desc* d, uint64_t* out, std::string* err);
  int launch_n(uint64_t k, const slate_launch_desc* d, uint32_t n, uint64_t* first, std::string* err);
  int resize(uint64_t l, uint32_t lo, uint32_t hi, std::string* err);
  int set_policy(uint32_t policy, std::string* err);
  int set_split_objective(uint32_t objective, double slack, std::string* err);
  int sync(uint64_t l, int64_t timeout_us, std::string* err);
  int profile(uint64_t k, const slate_launch_desc* d, uint32_t flags, slate_profile_t* out, std::string* err);
  int query(uint64_t l, slate_launch_info* out, std::string* err);

 private:
  int call(Request& rq, Response* rs, std::string* err, bool long_wait = false);
  ShmLayout* shm_ = nullptr;
  Slot* slot_ = nullptr;
  int fd_ = -1;
  uint64_t seq_ = 0;
};

}  // namespace slate
