// capi_internal.h -- process-wide in-process servers (one per device), shared by
// in-process sessions (capi.cu) and the slated loop (serve.cu).
#pragma once
#include <string>
#include "server.h"

namespace slate {
Server* get_local_server(int device, std::string* err, int* rc);
}
