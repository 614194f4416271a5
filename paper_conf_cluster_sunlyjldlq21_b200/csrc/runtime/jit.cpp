// jit.cpp — code generation of kernel variants (csTuner: "the code generation writes the
// sampled parameter settings into CUDA kernels"; checked before generation so that
// only valid settings are compiled).  NVRTC compiles
// csrc/kernels/cst_kernels.cuh for sm_100a with the setting as compile-time constants;
// cubins are cached in memory and on disk ($CST_CACHE_DIR, default ~/.cache/cst).
#include <dlfcn.h>
#include <nvrtc.h>
#include <sys/stat.h>
#include <unistd.h>

#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <fstream>
#include <sstream>
#include <unordered_map>

#include "internal.h"

namespace {
#include "kernels_src.inc"  // kSrcParams, kSrcPtx, kSrcKernels (generated at build time)

// NVRTC is loaded at run time by absolute path: torch may already have mapped its own
// (older) libnvrtc.so.12, and binding to that copy through the shared soname silently
// changes the generated code.  Order: $CST_NVRTC_PATH, $CUDA_HOME/lib64, /usr/local/cuda.
struct Nvrtc {
  decltype(&nvrtcCreateProgram) create = nullptr;
  decltype(&nvrtcCompileProgram) compile = nullptr;
  decltype(&nvrtcGetProgramLogSize) log_size = nullptr;
  decltype(&nvrtcGetProgramLog) log = nullptr;
  decltype(&nvrtcGetCUBINSize) cubin_size = nullptr;
  decltype(&nvrtcGetCUBIN) cubin = nullptr;
  decltype(&nvrtcDestroyProgram) destroy = nullptr;
  decltype(&nvrtcGetErrorString) error = nullptr;
  decltype(&nvrtcVersion) version = nullptr;
  std::string path;
  int major = 0, minor = 0;
};

const Nvrtc* nvrtc_lib() {
  static Nvrtc n;
  static bool ok = false;
  static std::once_flag once;
  std::call_once(once, [] {
    std::vector<std::string> cands;
    if (const char* e = std::getenv("CST_NVRTC_PATH")) cands.push_back(e);
    if (const char* c = std::getenv("CUDA_HOME")) cands.push_back(std::string(c) + "/lib64/libnvrtc.so.12");
    cands.push_back("/usr/local/cuda/lib64/libnvrtc.so.12");
    cands.push_back("libnvrtc.so.12");
    for (const std::string& p : cands) {
      void* h = dlopen(p.c_str(), RTLD_NOW | RTLD_LOCAL);
      if (!h) continue;
      n.create = (decltype(n.create))dlsym(h, "nvrtcCreateProgram");
      n.compile = (decltype(n.compile))dlsym(h, "nvrtcCompileProgram");
      n.log_size = (decltype(n.log_size))dlsym(h, "nvrtcGetProgramLogSize");
      n.log = (decltype(n.log))dlsym(h, "nvrtcGetProgramLog");
      n.cubin_size = (decltype(n.cubin_size))dlsym(h, "nvrtcGetCUBINSize");
      n.cubin = (decltype(n.cubin))dlsym(h, "nvrtcGetCUBIN");
      n.destroy = (decltype(n.destroy))dlsym(h, "nvrtcDestroyProgram");
      n.error = (decltype(n.error))dlsym(h, "nvrtcGetErrorString");
      n.version = (decltype(n.version))dlsym(h, "nvrtcVersion");
      if (n.create && n.compile && n.log_size && n.log && n.cubin_size && n.cubin &&
          n.destroy && n.error && n.version) {
        n.version(&n.major, &n.minor);
        n.path = p;
        ok = true;
        return;
      }
    }
  });
  return ok ? &n : nullptr;
}

std::mutex g_mu;
std::unordered_map<std::string, std::string> g_mem;  // key -> cubin
std::atomic<uint64_t> g_compiles{0};

uint64_t fnv1a(const std::string& s, uint64_t h = 0xCBF29CE484222325ULL) {
  for (unsigned char c : s) {
    h ^= c;
    h *= 0x100000001B3ULL;
  }
  return h;
}

std::string cache_dir() {
  const char* d = std::getenv("CST_CACHE_DIR");
  if (d && *d) return d;
  const char* x = std::getenv("XDG_CACHE_HOME");
  if (x && *x) return std::string(x) + "/cst";
  const char* h = std::getenv("HOME");
  return std::string(h ? h : "/tmp") + "/.cache/cst";
}

void mkdirs(const std::string& p) {
  std::string cur;
  std::stringstream ss(p);
  std::string part;
  if (!p.empty() && p[0] == '/') cur = "/";
  while (std::getline(ss, part, '/')) {
    if (part.empty()) continue;
    cur += part + "/";
    mkdir(cur.c_str(), 0755);
  }
}

}  // namespace

namespace cst {

uint64_t jit_compile_count() { return g_compiles.load(); }

std::string nvrtc_description() {
  const Nvrtc* N = nvrtc_lib();
  if (!N) return "nvrtc: not found";
  return "nvrtc " + std::to_string(N->major) + "." + std::to_string(N->minor) + " (" + N->path + ")";
}

static std::string prefix_for(const StencilInfo& st, const Tuple& t, bool remote) {
  std::ostringstream o;
  o << "#define CST_KIND " << st.kind << "\n#define CST_R " << st.r << "\n";
  if (remote) o << "#define CST_REMOTE 1\n";
  static const char* names[F_COUNT] = {"TBX", "TBY", "TBZ", "STAGING", "CONST", "STREAM",
                                       "SD",  "SB",  "UFX", "UFY",     "UFZ",   "CMX",
                                       "CMY", "CMZ", "BMX", "BMY",     "BMZ",   "RET",
                                       "PF",  "BT",      "QSTORE"};
  for (int i = 0; i < F_COUNT; ++i) o << "#define CST_" << names[i] << " " << t[i] << "\n";
  o << "#include \"cst_kernels.cuh\"\n";
  return o.str();
}

cst_status jit_cubin(const StencilInfo& st, const Tuple& t, std::string* cubin,
                     double* compile_s, bool remote) {
  const std::string src = prefix_for(st, t, remote);
  std::vector<std::string> optv = {"--gpu-architecture=sm_100a", "-std=c++17", "-lineinfo",
                                   "--fmad=true", "-default-device", "-DCST_NVRTC=1"};
  // experiment hook: extra -D options (e.g. "-DCST_EMPTY_BARRIERS=1"), part of the cache key
  if (const char* e = std::getenv("CST_NVRTC_DEFINES")) {
    std::stringstream ss(e);
    std::string tok;
    while (ss >> tok) optv.push_back(tok);
  }
  std::vector<const char*> optp;
  for (const std::string& o : optv) optp.push_back(o.c_str());
  const char* const* opts = optp.data();
  const int nopts = (int)optp.size();
  const Nvrtc* N = nvrtc_lib();
  if (!N) return fail(CST_E_NVRTC, "libnvrtc.so.12 not found (set CST_NVRTC_PATH)");
  std::string keysrc = src + "nvrtc" + std::to_string(N->major) + "." + std::to_string(N->minor);
  for (int i = 0; i < nopts; ++i) keysrc += opts[i];
  uint64_t h = fnv1a(keysrc);
  h = fnv1a(kSrcParams, h);
  h = fnv1a(kSrcPtx, h);
  h = fnv1a(kSrcKernels, h);
  char key[32];
  std::snprintf(key, sizeof key, "%016llx", (unsigned long long)h);
  *compile_s = 0;
  {
    std::lock_guard<std::mutex> lk(g_mu);
    auto it = g_mem.find(key);
    if (it != g_mem.end()) {
      *cubin = it->second;
      return CST_OK;
    }
  }
  const std::string dir = cache_dir();
  const std::string path = dir + "/" + key + ".cubin";
  {
    std::ifstream f(path, std::ios::binary);
    if (f) {
      std::string data((std::istreambuf_iterator<char>(f)), std::istreambuf_iterator<char>());
      if (!data.empty()) {
        std::lock_guard<std::mutex> lk(g_mu);
        g_mem[key] = data;
        *cubin = data;
        return CST_OK;
      }
    }
  }
  const auto t0 = std::chrono::steady_clock::now();
  const char* hdr_src[3] = {kSrcParams, kSrcPtx, kSrcKernels};
  const char* hdr_names[3] = {"cst_params.h", "cst_ptx.cuh", "cst_kernels.cuh"};
  nvrtcProgram prog;
  if (N->create(&prog, src.c_str(), "cst_variant.cu", 3, hdr_src, hdr_names) != NVRTC_SUCCESS)
    return fail(CST_E_NVRTC, "nvrtcCreateProgram failed");
  const nvrtcResult rc = N->compile(prog, nopts, opts);
  if (rc != NVRTC_SUCCESS) {
    size_t n = 0;
    N->log_size(prog, &n);
    std::string log(n, '\0');
    if (n) N->log(prog, &log[0]);
    N->destroy(&prog);
    return fail(CST_E_NVRTC, std::string("nvrtc: ") + N->error(rc) + "\n" + log.substr(0, 4000));
  }
  size_t n = 0;
  N->cubin_size(prog, &n);
  std::string data(n, '\0');
  N->cubin(prog, &data[0]);
  N->destroy(&prog);
  ++g_compiles;
  *compile_s =
      std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
  {
    std::lock_guard<std::mutex> lk(g_mu);
    g_mem[key] = data;
  }
  mkdirs(dir);
  const std::string tmp = path + ".tmp" + std::to_string(getpid());
  {
    std::ofstream f(tmp, std::ios::binary);
    if (f) f.write(data.data(), (std::streamsize)data.size());
  }
  std::rename(tmp.c_str(), path.c_str());
  *cubin = data;
  return CST_OK;
}

}  // namespace cst
