// ipc.h -- client side of the shared-memory transport to a `slated` server
// (commands over a fast channel, data in shared buffers).
#pragma once
#include <cstdint>
#include <string>
#include "../../include/slate.h"

namespace slate {

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
  int launch(uint64_t k, const slate_launch_desc* d, uint64_t* out, std::string* err);
  int resize(uint64_t l, uint32_t lo, uint32_t hi, std::string* err);
  int sync(uint64_t l, int64_t timeout_us, std::string* err);
  int profile(uint64_t k, const slate_launch_desc* d, uint32_t flags, slate_profile_t* out, std::string* err);
  int query(uint64_t l, slate_launch_info* out, std::string* err);

 private:
  struct Impl;
  Impl* impl_;
};

}  // namespace slate
