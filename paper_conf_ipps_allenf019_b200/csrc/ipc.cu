// ipc.cu -- shared-memory transport (client side).  Placeholder until the
// slated daemon lands: every call reports SLATE_EIPC.
#include "ipc.h"

namespace slate {
struct RemoteClient::Impl {};
RemoteClient::RemoteClient() : impl_(nullptr) {}
RemoteClient::~RemoteClient() {}
static int no_ipc(std::string* err) {
  if (err) *err = "no slated server support in this build yet";
  return SLATE_EIPC;
}
int RemoteClient::connect(const char*, std::string* err) { return no_ipc(err); }
int RemoteClient::detach(std::string* err) { return no_ipc(err); }
int RemoteClient::info(slate_info*, std::string* err) { return no_ipc(err); }
int RemoteClient::share(uint64_t, size_t, uint64_t*, std::string* err) { return no_ipc(err); }
int RemoteClient::unshare(uint64_t, std::string* err) { return no_ipc(err); }
int RemoteClient::register_kernel(const slate_kernel_desc*, uint64_t*, std::string* err) { return no_ipc(err); }
int RemoteClient::launch(uint64_t, const slate_launch_desc*, uint64_t*, std::string* err) { return no_ipc(err); }
int RemoteClient::resize(uint64_t, uint32_t, uint32_t, std::string* err) { return no_ipc(err); }
int RemoteClient::sync(uint64_t, int64_t, std::string* err) { return no_ipc(err); }
int RemoteClient::profile(uint64_t, const slate_launch_desc*, uint32_t, slate_profile_t*, std::string* err) { return no_ipc(err); }
int RemoteClient::query(uint64_t, slate_launch_info*, std::string* err) { return no_ipc(err); }
}  // namespace slate
