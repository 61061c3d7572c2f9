// user_kernels.cu -- NEXT-3: Slate's runtime kernel transformation.
//
// The paper scans a user kernel's source with a FLEX scanner, injects the
// Lst1/Lst2 code (SM binding, task loop, block-index decode) and compiles the
// result with NVRTC.  Here the scanner finds `__global__ void <name>(...)`,
// turns the kernel into a __device__ body that takes its block index and the
// original grid as parameters (every `blockIdx` / `gridDim` token of the
// source is renamed to them), packs its parameter list into an argument
// struct, and generates around the body
//   * the tenant the worker template runs (slate_device.cuh: the same
//     worker_body as the built-in kinds -- Lst1, Lst2, the resize word), and
//   * the original kernel K(B,T): the body at the hardware blockIdx/gridDim.
// NVRTC compiles the generated source for sm_100a; the runtime API loads it
// (cudaLibraryLoadData) and the kernels are launched like built-in ones.
#include <dlfcn.h>
#include <sys/stat.h>
#include <unistd.h>
#include <atomic>
#include <cstdio>
#include <cstring>
#include <map>
#include <mutex>
#include <regex>
#include <string>
#include <vector>
#include "kernels.h"

namespace slate {

namespace {

// split a parameter list at top-level commas
std::vector<std::string> split_params(const std::string& s) {
  std::vector<std::string> out;
  int depth = 0;
  std::string cur;
  for (char ch : s) {
    if (ch == '(' || ch == '<' || ch == '[') ++depth;
    if (ch == ')' || ch == '>' || ch == ']') --depth;
    if (ch == ',' && depth == 0) {
      out.push_back(cur);
      cur.clear();
    } else {
      cur += ch;
    }
  }
  if (cur.find_first_not_of(" \t\r\n") != std::string::npos) out.push_back(cur);
  return out;
}

std::string trim(const std::string& s) {
  const size_t a = s.find_first_not_of(" \t\r\n"), b = s.find_last_not_of(" \t\r\n");
  return a == std::string::npos ? std::string() : s.substr(a, b - a + 1);
}

// the declared name of a parameter: its last identifier
std::string param_name(const std::string& p) {
  size_t e = p.size();
  while (e > 0 && !(isalnum(static_cast<unsigned char>(p[e - 1])) || p[e - 1] == '_')) --e;
  size_t b = e;
  while (b > 0 && (isalnum(static_cast<unsigned char>(p[b - 1])) || p[b - 1] == '_')) --b;
  return p.substr(b, e - b);
}

std::string replace_token(const std::string& s, const std::string& from, const std::string& to) {
  return std::regex_replace(s, std::regex("\\b" + from + "\\b"), to);
}

}  // namespace

bool transform_user_kernel(const char* src, const char* name, uint32_t bx, uint32_t by, uint32_t bz, uint32_t smem,
                           std::string* out, std::string* err) {
  by = by ? by : 1;
  bz = bz ? bz : 1;
  const uint64_t threads = uint64_t(bx) * by * bz;
  if (!src || !name || !*name || bx == 0 || threads > 1024 || by > 1024 || bz > 64) {
    if (err) *err = "need a source, a kernel name and a block of 1..1024 threads";
    return false;
  }
  std::string s(src);
  std::smatch m;
  const std::regex head("__global__\\s+(?:__launch_bounds__\\s*\\([^)]*\\)\\s*)?void\\s+" + std::string(name) +
                        "\\s*\\(");
  if (!std::regex_search(s, m, head)) {
    if (err) *err = std::string("no `__global__ void ") + name + "(` in the source";
    return false;
  }
  const size_t open = size_t(m.position(0) + m.length(0)) - 1;
  int depth = 0;
  size_t close = open;
  for (; close < s.size(); ++close) {
    if (s[close] == '(') ++depth;
    if (s[close] == ')' && --depth == 0) break;
  }
  if (close >= s.size()) {
    if (err) *err = "unbalanced parameter list";
    return false;
  }
  const std::string params = s.substr(open + 1, close - open - 1);
  std::vector<std::string> ps;
  for (const std::string& p : split_params(params))
    if (!trim(p).empty() && trim(p) != "void") ps.push_back(trim(p));
  // the kernel becomes a device function taking its block index, the original
  // grid, its thread index and the block shape: every blockIdx / gridDim /
  // threadIdx / blockDim token of the source is renamed to them, so the worker
  // can run the body with a decoded block index on a 1-D worker CTA of the
  // same thread count (threads linearised x-fastest, as the hardware forms
  // warps: the body's warp-level operations see the same lanes)
  std::string body = s.substr(0, size_t(m.position(0))) + "__device__ __forceinline__ void slate_user_body(" +
                     "const uint3 slate_bidx, const dim3 slate_gdim, const uint3 slate_tidx, const dim3 slate_bdim" +
                     (ps.empty() ? "" : ", ") + params + ")" + s.substr(close + 1);
  body = replace_token(body, "blockIdx", "slate_bidx");
  body = replace_token(body, "gridDim", "slate_gdim");
  body = replace_token(body, "threadIdx", "slate_tidx");
  body = replace_token(body, "blockDim", "slate_bdim");
  std::string fields, call, layout;
  uint32_t nptr = 0;
  for (const std::string& p : ps) {
    fields += "  " + replace_token(p, "__restrict__", "") + ";\n";
    call += ", a." + param_name(p);
    if (p.find('*') != std::string::npos) {   // a device pointer: rewritten by a server behind an endpoint
      layout += ", (unsigned int)offsetof(SlateUserArgs, " + param_name(p) + ")";
      ++nptr;
    }
  }
  // a body that stages through shared memory may not start block i+1 while
  // slow threads still read block i's shared data (the worker runs a task's
  // blocks back to back in one CTA): a barrier between blocks
  const bool shared = smem > 0 || std::regex_search(s, std::regex("\\b__shared__\\b"));
  const std::string T = std::to_string(threads), SM = std::to_string(smem), BX = std::to_string(bx),
                    BY = std::to_string(by), BZ = std::to_string(bz);
  std::string g;
  g += "// generated by slate_register_source (NEXT-3): the user kernel as a slate tenant\n";
  g += "#include <cuda/std/cstddef>   // offsetof\n";
  g += "#include \"slate_device.cuh\"\n\n";
  g += "// ---- the user's source; its kernel `" + std::string(name) + "` became a device body\n";
  g += body + "\n\n";
  g += "// ---- generated\n";
  g += "struct SlateUserArgs {\n" + fields + "};\n";
  g += "// {sizeof the argument struct, number of pointer parameters, their offsets}: read by the host\n";
  g += "extern \"C\" __device__ const unsigned int slate_user_layout[" + std::to_string(2 + nptr) +
       "] = {(unsigned int)sizeof(SlateUserArgs), " + std::to_string(nptr) + "u" + layout + "};\n";
  g += "__shared__ dim3 slate_user_gdim;   // the original grid, set by the worker's thread 0\n";
  g += "struct SlateUserTenant : slate::TenantBase {\n";
  g += "  using Args = SlateUserArgs;\n";
  g += "  static constexpr int kThreads = " + T + ", kMinBlocks = 1, kSmem = " + SM + ", kSmemStandalone = " + SM +
       ";\n";
  g += "  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t y, uint32_t z, char*) {\n";
  if (shared) g += "    __syncthreads();   // the previous block's shared-memory readers are done\n";
  g += "    const uint32_t t = threadIdx.x;\n";
  g += "    slate_user_body(make_uint3(x, y, z), slate_user_gdim, make_uint3(t % " + BX + "u, (t / " + BX + "u) % " +
       BY + "u, t / (" + BX + "u * " + BY + "u)), dim3(" + BX + ", " + BY + ", " + BZ + ")" + call + ");\n  }\n};\n";
  g += "extern \"C\" __global__ void __launch_bounds__(" + T +
       ") slate_user_worker(const __grid_constant__ SlateUserArgs a,\n"
       "                                                      const __grid_constant__ slate::UserWorkerCommon c) {\n";
  g += "  if (threadIdx.x == 0) slate_user_gdim = dim3(c.gx, c.gy, c.gz);   // read after the prologue's barrier\n";
  g += "  slate::WorkerParams<SlateUserArgs> p;\n";
  g += "  p.args = a;\n";
  g += "  p.gx = c.gx; p.gy = c.gy; p.gz = c.gz; p.B = c.B; p.iters = c.iters; p.occ = c.occ;\n";
  g += "  p.bound_lo = c.bound_lo; p.bound_hi = c.bound_hi; p.n_ranks = c.n_ranks;\n";
  g += "  p.standby_timeout_ns = c.standby_timeout_ns; p.base_epoch = c.base_epoch; p.is_topup = c.is_topup;\n";
  g += "  p.gate_first = c.gate_first; p.ranklog = c.ranklog; p.ctrl = c.ctrl; p.tc = c.tc; p.mirror = c.mirror;\n";
  g += "  p.cov = c.cov; p.rank_of = c.rank_of; p.pdl_early = 0;\n";
  g += "  slate::worker_body<SlateUserTenant>(p);\n}\n";
  g += "// the original kernel K(B,T), launched with the " + BX + " x " + BY + " x " + BZ + " block\n";
  g += "extern \"C\" __global__ void __launch_bounds__(" + T +
       ") slate_user_original(const __grid_constant__ SlateUserArgs a) {\n";
  g += "  slate_user_body(blockIdx, gridDim, threadIdx, blockDim" + call + ");\n}\n";
  *out = g;
  return true;
}

namespace {

struct UserKernel {
  cudaLibrary_t lib = nullptr;
  cudaKernel_t worker = nullptr, original = nullptr;
  uint32_t bx = 1, by = 1, bz = 1, smem = 0;
  uint32_t args_size = 0;           // sizeof the generated argument struct (read from the image)
  std::vector<size_t> ptr_offs;     // offsets of its pointer parameters
};

typedef int (*nvrtcCreateProgram_t)(void**, const char*, const char*, int, const char* const*, const char* const*);
typedef int (*nvrtcCompileProgram_t)(void*, int, const char* const*);
typedef int (*nvrtcGetSize_t)(void*, size_t*);
typedef int (*nvrtcGet_t)(void*, char*);
typedef int (*nvrtcDestroyProgram_t)(void**);
typedef int (*nvrtcVersion_t)(int*, int*);

void* nvrtc_handle() {
  static void* h = nullptr;
  if (h) return h;
  const char* env = getenv("SLATE_NVRTC");
  const char* cands[] = {env, "libnvrtc.so", "libnvrtc.so.12", "/usr/local/cuda/lib64/libnvrtc.so"};
  for (const char* c : cands)
    if (c && (h = dlopen(c, RTLD_NOW | RTLD_LOCAL))) break;
  return h;
}

std::string here_dir() {   // the directory of this library (csrc/ sits next to it)
  Dl_info info;
  if (dladdr(reinterpret_cast<void*>(&nvrtc_handle), &info) && info.dli_fname) {
    std::string p(info.dli_fname);
    const size_t k = p.rfind('/');
    return k == std::string::npos ? std::string(".") : p.substr(0, k);
  }
  return ".";
}

// ---- the compiled-image cache ("A compiled kernel image can be
// further cached").  Key: FNV-1a 64 of the generated source, the compile
// options and the NVRTC version.  Level 1, in process: the loaded library, so
// a second registration of the same kernel (another task size, flags) costs
// no compile and no load.  Level 2, on disk: the cubin, in $SLATE_RTC_CACHE
// (default $HOME/.cache/slate-rtc; "off" disables it), written atomically
// (temp file + rename), so another server process or a restarted slated skips
// NVRTC.  A cubin that fails to load is recompiled.
std::mutex g_rtc_mu;
std::map<uint64_t, UserKernel*> g_rtc_loaded;   // owned for the process lifetime (kernels may still run)
std::atomic<uint64_t> g_rtc_compiles{0}, g_rtc_mem_hits{0}, g_rtc_disk_hits{0};

uint64_t fnv1a(const std::string& s, uint64_t h = 1469598103934665603ull) {
  for (unsigned char ch : s) {
    h ^= ch;
    h *= 1099511628211ull;
  }
  return h;
}

std::string rtc_cache_dir() {
  const char* env = getenv("SLATE_RTC_CACHE");
  if (env && std::string(env) == "off") return std::string();
  if (env && *env) return std::string(env);
  const char* home = getenv("HOME");
  return home && *home ? std::string(home) + "/.cache/slate-rtc" : std::string();
}

bool read_file(const std::string& path, std::vector<char>* out) {
  FILE* f = fopen(path.c_str(), "rb");
  if (!f) return false;
  fseek(f, 0, SEEK_END);
  const long n = ftell(f);
  fseek(f, 0, SEEK_SET);
  bool ok = n > 0;
  if (ok) {
    out->resize(size_t(n));
    ok = fread(out->data(), 1, size_t(n), f) == size_t(n);
  }
  fclose(f);
  return ok;
}

void write_file_atomic(const std::string& dir, const std::string& path, const std::vector<char>& data) {
  if (dir.empty()) return;
  std::string d;   // mkdir -p
  for (size_t i = 0; i <= dir.size(); ++i) {
    if (i == dir.size() || dir[i] == '/') {
      if (!d.empty()) mkdir(d.c_str(), 0755);
    }
    if (i < dir.size()) d += dir[i];
  }
  const std::string tmp = path + ".tmp." + std::to_string(getpid());
  FILE* f = fopen(tmp.c_str(), "wb");
  if (!f) return;
  const bool ok = fwrite(data.data(), 1, data.size(), f) == data.size();
  fclose(f);
  if (!ok || rename(tmp.c_str(), path.c_str()) != 0) unlink(tmp.c_str());
}

bool nvrtc_compile(const std::string& gen, std::vector<char>* cubin, std::string* err) {
  void* h = nvrtc_handle();
  if (!h) {
    if (err) *err = "NVRTC (libnvrtc.so) not found";
    return false;
  }
  auto create = reinterpret_cast<nvrtcCreateProgram_t>(dlsym(h, "nvrtcCreateProgram"));
  auto compile = reinterpret_cast<nvrtcCompileProgram_t>(dlsym(h, "nvrtcCompileProgram"));
  auto log_size = reinterpret_cast<nvrtcGetSize_t>(dlsym(h, "nvrtcGetProgramLogSize"));
  auto get_log = reinterpret_cast<nvrtcGet_t>(dlsym(h, "nvrtcGetProgramLog"));
  auto cubin_size = reinterpret_cast<nvrtcGetSize_t>(dlsym(h, "nvrtcGetCUBINSize"));
  auto get_cubin = reinterpret_cast<nvrtcGet_t>(dlsym(h, "nvrtcGetCUBIN"));
  auto destroy = reinterpret_cast<nvrtcDestroyProgram_t>(dlsym(h, "nvrtcDestroyProgram"));
  if (!create || !compile || !log_size || !get_log || !cubin_size || !get_cubin || !destroy) {
    if (err) *err = "NVRTC entry points missing";
    return false;
  }
  void* prog = nullptr;
  if (create(&prog, gen.c_str(), "slate_user.cu", 0, nullptr, nullptr) != 0) {
    if (err) *err = "nvrtcCreateProgram failed";
    return false;
  }
  const std::string inc_csrc = "-I" + here_dir() + "/csrc";
  const char* cuda_home = getenv("CUDA_HOME");
  const std::string inc_cuda = std::string("-I") + (cuda_home ? cuda_home : "/usr/local/cuda") + "/include";
  const char* opts[] = {"--gpu-architecture=sm_100a", "-std=c++17", "-lineinfo", inc_csrc.c_str(), inc_cuda.c_str()};
  const int rc = compile(prog, 5, opts);
  size_t n = 0;
  log_size(prog, &n);
  std::string log(n, '\0');
  if (n) get_log(prog, &log[0]);
  if (rc != 0) {
    if (err) *err = "NVRTC failed:\n" + log;
    destroy(&prog);
    return false;
  }
  cubin_size(prog, &n);
  cubin->resize(n);
  get_cubin(prog, cubin->data());
  destroy(&prog);
  return true;
}

UserKernel* load_image(const std::vector<char>& cubin, std::string* err) {
  auto* u = new UserKernel();
  cudaError_t e = cudaLibraryLoadData(&u->lib, cubin.data(), nullptr, nullptr, 0, nullptr, nullptr, 0);
  if (e == cudaSuccess) e = cudaLibraryGetKernel(&u->worker, u->lib, "slate_user_worker");
  if (e == cudaSuccess) e = cudaLibraryGetKernel(&u->original, u->lib, "slate_user_original");
  void* lay = nullptr;
  size_t lay_bytes = 0;
  if (e == cudaSuccess) e = cudaLibraryGetGlobal(&lay, &lay_bytes, u->lib, "slate_user_layout");
  std::vector<uint32_t> layout(lay_bytes / 4);
  if (e == cudaSuccess && lay_bytes >= 8) e = cudaMemcpy(layout.data(), lay, lay_bytes, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess || layout.size() < 2 || layout.size() != 2 + layout[1]) {
    if (err)
      *err = std::string("loading the compiled user kernel: ") +
             (e != cudaSuccess ? cudaGetErrorString(e) : "bad slate_user_layout");
    cudaGetLastError();
    if (u->lib) cudaLibraryUnload(u->lib);
    delete u;
    return nullptr;
  }
  u->args_size = layout[0];
  for (size_t i = 2; i < layout.size(); ++i) u->ptr_offs.push_back(layout[i]);
  return u;
}

cudaError_t launch_user_worker(const WorkerCommon& w, const void* args, uint32_t grid, cudaStream_t st) {
  const UserKernel* u = static_cast<const UserKernel*>(w.ops ? w.ops->user_ctx : nullptr);
  if (!u) return cudaErrorInvalidValue;
  UserWorkerCommon c{};
  c.gx = w.gx; c.gy = w.gy; c.gz = w.gz; c.B = w.B; c.iters = w.iters; c.occ = w.occ;
  c.bound_lo = w.bound_lo; c.bound_hi = w.bound_hi; c.n_ranks = w.n_ranks;
  c.standby_timeout_ns = w.standby_timeout_ns; c.base_epoch = w.base_epoch; c.is_topup = w.is_topup;
  c.gate_first = w.gate_first; c.ranklog = w.ranklog; c.ctrl = w.ctrl; c.tc = w.tc; c.mirror = w.mirror;
  c.cov = w.cov; c.rank_of = w.rank_of;
  void* kargs[] = {const_cast<void*>(args), &c};
  return launch_kernel(reinterpret_cast<const void*>(u->worker), dim3(grid), dim3(u->bx * u->by * u->bz), kargs,
                       u->smem, st, w.pdl);
}

cudaError_t launch_user_original(const KindOps* ops, const void* args, dim3 grid, cudaStream_t st) {
  const UserKernel* u = static_cast<const UserKernel*>(ops->user_ctx);
  void* kargs[] = {const_cast<void*>(args)};
  return cudaLaunchKernel(reinterpret_cast<const void*>(u->original), grid, dim3(u->bx, u->by, u->bz), kargs, u->smem,
                          st);
}

}  // namespace

bool build_user_kind(const char* src, const char* name, uint32_t bx, uint32_t by, uint32_t bz, uint32_t smem,
                     uint32_t args_size, KindOps* ops, std::string* err, bool* compiled) {
  by = by ? by : 1;
  bz = bz ? bz : 1;
  std::string gen;
  if (!transform_user_kernel(src, name, bx, by, bz, smem, &gen, err)) return false;
  int major = 0, minor = 0;
  if (void* h = nvrtc_handle())
    if (auto ver = reinterpret_cast<nvrtcVersion_t>(dlsym(h, "nvrtcVersion"))) ver(&major, &minor);
  const uint64_t key = fnv1a("sm_100a -std=c++17 -lineinfo nvrtc " + std::to_string(major) + "." +
                             std::to_string(minor) + "\n" + here_dir() + "\n" + gen);
  char hex[17];
  snprintf(hex, sizeof(hex), "%016llx", static_cast<unsigned long long>(key));
  if (compiled) *compiled = false;
  UserKernel* u = nullptr;
  {
    std::lock_guard<std::mutex> g(g_rtc_mu);
    auto it = g_rtc_loaded.find(key);
    if (it != g_rtc_loaded.end()) {
      u = it->second;
      g_rtc_mem_hits += 1;
    }
  }
  if (!u) {
    const std::string dir = rtc_cache_dir();
    const std::string path = dir.empty() ? std::string() : dir + "/" + hex + ".cubin";
    std::vector<char> cubin;
    if (!path.empty() && read_file(path, &cubin) && (u = load_image(cubin, nullptr))) {
      g_rtc_disk_hits += 1;
    } else {
      if (!nvrtc_compile(gen, &cubin, err)) return false;
      if (!(u = load_image(cubin, err))) return false;
      g_rtc_compiles += 1;
      if (compiled) *compiled = true;
      if (!path.empty()) write_file_atomic(dir, path, cubin);
    }
    u->bx = bx; u->by = by; u->bz = bz; u->smem = smem;
    std::lock_guard<std::mutex> g(g_rtc_mu);
    auto it = g_rtc_loaded.find(key);
    if (it != g_rtc_loaded.end()) {   // another thread loaded it meanwhile: keep one
      cudaLibraryUnload(u->lib);
      delete u;
      u = it->second;
    } else {
      g_rtc_loaded[key] = u;
    }
  }
  if (args_size != u->args_size) {
    if (err)
      *err = "args_size " + std::to_string(args_size) + " != sizeof the kernel's parameter struct (" +
             std::to_string(u->args_size) + " bytes, parameters in declaration order with C alignment)";
    return false;
  }
  ops->worker_fn = reinterpret_cast<const void*>(u->worker);
  ops->standalone_fn = reinterpret_cast<const void*>(u->original);
  ops->threads = int(bx * by * bz);
  ops->smem = int(smem);
  ops->smem_standalone = int(smem);
  ops->args_size = args_size;
  ops->launch_worker = &launch_user_worker;
  ops->launch_standalone_ops = &launch_user_original;
  ops->pdl_ok = true;           // worker_body waits in griddepcontrol.wait
  ops->topup_anytime = true;    // worker_body's leave_main
  ops->user_threads = bx * by * bz;
  ops->user_ctx = u;            // owned by the image cache for the process lifetime
  ops->user_ptr_offsets = u->ptr_offs;
  return true;
}

}  // namespace slate

// the transformation alone (tests, no GPU)
extern "C" slate_status slate_transform_source(const char* source, const char* kernel_name, uint32_t block_x,
                                               uint32_t block_y, uint32_t block_z, uint32_t smem_bytes, char* out,
                                               size_t cap, size_t* len) {
  std::string g, err;
  if (!slate::transform_user_kernel(source, kernel_name, block_x, block_y, block_z, smem_bytes, &g, &err))
    return SLATE_EINVAL;
  if (len) *len = g.size();
  if (out && cap) {
    const size_t k = std::min(cap - 1, g.size());
    std::memcpy(out, g.data(), k);
    out[k] = '\0';
  }
  return SLATE_OK;
}

extern "C" void slate_rtc_stats(uint64_t* compiles, uint64_t* mem_hits, uint64_t* disk_hits) {
  if (compiles) *compiles = slate::g_rtc_compiles.load();
  if (mem_hits) *mem_hits = slate::g_rtc_mem_hits.load();
  if (disk_hits) *disk_hits = slate::g_rtc_disk_hits.load();
}
