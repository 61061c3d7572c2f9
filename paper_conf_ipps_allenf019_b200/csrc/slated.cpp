// slated -- the Slate daemon: one per GPU, all client processes' kernels funnel
// into its single CUDA context (§IV-A).
//   slated [--device G] [--endpoint /slate-gpuG]
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include "../../include/slate.h"

int main(int argc, char** argv) {
  int device = 0;
  std::string endpoint;
  for (int i = 1; i < argc; ++i) {
    if (!std::strcmp(argv[i], "--device") && i + 1 < argc) device = std::atoi(argv[++i]);
    else if (!std::strcmp(argv[i], "--endpoint") && i + 1 < argc) endpoint = argv[++i];
    else {
      std::fprintf(stderr, "usage: slated [--device G] [--endpoint /slate-gpuG]\n");
      return 2;
    }
  }
  if (endpoint.empty()) endpoint = "/slate-gpu" + std::to_string(device);
  const slate_status st = slate_serve(endpoint.c_str(), device, 0);
  if (st != SLATE_OK) std::fprintf(stderr, "slated: %s\n", slate_status_string(st));
  return st == SLATE_OK ? 0 : 1;
}
