// NVRTC specialiser: compiles (template ll_kernels.cuh + per-plan constants) for
// sm_100a, caches cubins in memory and on disk, loads them with cudaLibraryLoadData.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nvrtc.h>
#include <sys/stat.h>
#include <unistd.h>

#include <cstdio>
#include <cstdlib>
#include <fstream>
#include <sstream>
#include <mutex>
#include <thread>
#include <unordered_map>

#include "ll_internal.hpp"

namespace ll {

namespace {
const char* kTemplate =
#include "ll_kernels_embed.inc"
    ;

std::mutex g_mu;
std::unordered_map<std::string, cudaKernel_t> g_kernels;   // key -> kernel
std::vector<cudaLibrary_t> g_libs;

u64 fnv1a(const std::string& s, u64 h = 1469598103934665603ull) {
  for (unsigned char c : s) { h ^= c; h *= 1099511628211ull; }
  return h;
}

std::string self_dir() {
  Dl_info info;
  if (dladdr(reinterpret_cast<void*>(&self_dir), &info) && info.dli_fname) {
    std::string p = info.dli_fname;
    auto k = p.rfind('/');
    if (k != std::string::npos) return p.substr(0, k);
  }
  return ".";
}

std::string cache_dir() {
  const char* e = std::getenv("LL_JIT_CACHE");
  std::string d = e && *e ? std::string(e) : self_dir() + "/.ll_jit_cache";
  mkdir(d.c_str(), 0755);
  return d;
}

const char* kOpts[] = {"--gpu-architecture=sm_100a", "-std=c++17", "--generate-line-info", "-default-device", "-DNDEBUG"};

std::string full_source(const std::string& plan_src) {
  return std::string(kTemplate) + "\n// ---- plan specialisation ----\n" + plan_src;
}

std::string key_of(const std::string& full) {
  std::string k = full;
  for (auto* o : kOpts) k += o;
  int maj = 0, mi = 0;
  nvrtcVersion(&maj, &mi);
  k += std::to_string(maj) + "." + std::to_string(mi);
  char buf[32];
  snprintf(buf, sizeof buf, "%016llx", (unsigned long long)fnv1a(k));
  return buf;
}

std::string compile(const std::string& full, const char* name) {
  nvrtcProgram prog;
  if (nvrtcCreateProgram(&prog, full.c_str(), "ll_plan.cu", 0, nullptr, nullptr) != NVRTC_SUCCESS)
    fail(LL_ERR_NVRTC, "nvrtcCreateProgram failed");
  nvrtcResult r = nvrtcCompileProgram(prog, int(sizeof(kOpts) / sizeof(kOpts[0])), kOpts);
  if (r != NVRTC_SUCCESS) {
    size_t n = 0;
    nvrtcGetProgramLogSize(prog, &n);
    std::string log(n, '\0');
    nvrtcGetProgramLog(prog, &log[0]);
    nvrtcDestroyProgram(&prog);
    fail(LL_ERR_NVRTC, std::string("NVRTC compile of ") + name + " failed:\n" + log.substr(0, 4000));
  }
  size_t n = 0;
  nvrtcGetCUBINSize(prog, &n);
  std::string cubin(n, '\0');
  nvrtcGetCUBIN(prog, &cubin[0]);
  nvrtcDestroyProgram(&prog);
  return cubin;
}

// Read-only cache of the cubins build() pre-compiles for the benchmark / smoke plans
// (travels with the tree); the writable cache (LL_JIT_CACHE) holds everything else.
std::string prebuilt_dir() { return self_dir() + "/.ll_jit_prebuilt"; }

std::string read_file(const std::string& path) {
  std::ifstream f(path, std::ios::binary);
  if (!f) return std::string();
  std::stringstream ss;
  ss << f.rdbuf();
  return ss.str();
}

std::string cubin_for(const std::string& full, const char* name, std::string* key_out) {
  std::string key = key_of(full);
  if (key_out) *key_out = key;
  std::string path = cache_dir() + "/" + key + ".cubin";
  for (const std::string& p : {path, prebuilt_dir() + "/" + key + ".cubin"}) {
    std::string s = read_file(p);
    if (!s.empty()) return s;
  }
  std::string cubin = compile(full, name);
  // unique temp name per process and thread; a failed write (full disk) is not renamed
  // into the cache, the cubin in memory is still used
  std::ostringstream tn;
  tn << path << ".tmp" << getpid() << "." << std::this_thread::get_id();
  const std::string tmp = tn.str();
  bool ok;
  {
    std::ofstream f(tmp, std::ios::binary);
    f.write(cubin.data(), std::streamsize(cubin.size()));
    f.flush();
    ok = f.good();
  }
  if (ok) rename(tmp.c_str(), path.c_str());
  else std::remove(tmp.c_str());
  // keep the source beside it (ncu source view / inspection)
  std::ofstream(cache_dir() + "/" + key + ".cu") << full;
  return cubin;
}
}  // namespace

const char* kernel_template() { return kTemplate; }

std::string jit_precompile(const std::string& plan_src, const char* name) {
  std::lock_guard<std::mutex> g(g_mu);
  std::string key;
  cubin_for(full_source(plan_src), name, &key);
  return key;
}

void* jit_kernel(const std::string& plan_src, const char* name) {
  std::string full = full_source(plan_src);
  std::lock_guard<std::mutex> g(g_mu);
  std::string key;
  std::string cubin = cubin_for(full, name, &key);
  auto it = g_kernels.find(key);
  if (it != g_kernels.end()) return reinterpret_cast<void*>(it->second);
  cudaLibrary_t lib;
  cudaError_t e = cudaLibraryLoadData(&lib, cubin.data(), nullptr, nullptr, 0, nullptr, nullptr, 0);
  if (e != cudaSuccess) fail(LL_ERR_CUDA, std::string("cudaLibraryLoadData: ") + cudaGetErrorString(e));
  cudaKernel_t k;
  e = cudaLibraryGetKernel(&k, lib, name);
  if (e != cudaSuccess) fail(LL_ERR_CUDA, std::string("cudaLibraryGetKernel: ") + cudaGetErrorString(e));
  g_libs.push_back(lib);
  g_kernels[key] = k;
  return reinterpret_cast<void*>(k);
}

}  // namespace ll
