// jit.cpp — per-plan kernel specialisation with NVRTC ("query compilation").
//
// The moderator picks a kernel per query; on B200 the cheapest kernel for a given
// schema is the one whose field program is compiled in. For each plan this module emits a JitSpec
// (key dtypes, dictionary sizes and mixed-radix strides, value dtypes, and every state field's kind,
// column, slot offset and dense-state position as compile-time constants), pastes it after the same
// device source libblugby is built from (blu_params.h + blu_device.cuh, embedded at build time), and
// compiles extern "C" entry points for sm_100a with NVRTC. Cubins are cached per source text in
// process and under $XDG_CACHE_HOME/blugby (or ~/.cache/blugby). Set BLU_GBY_JIT=0 to use only the
// precompiled schema-generic kernels (also the fallback when NVRTC is unavailable or fails).
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/stat.h>
#include <unistd.h>

#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "blu_internal.h"
#include "jit_sources.h"

namespace blu {

namespace {

// ---- NVRTC, loaded lazily (dlopen) so the library loads on machines without it -------------
typedef int nvrtcResult_t;
typedef struct _nvrtcProgram* nvrtcProgram_t;
struct Nvrtc {
  nvrtcResult_t (*create)(nvrtcProgram_t*, const char*, const char*, int, const char* const*, const char* const*);
  nvrtcResult_t (*compile)(nvrtcProgram_t, int, const char* const*);
  nvrtcResult_t (*cubin_size)(nvrtcProgram_t, size_t*);
  nvrtcResult_t (*cubin)(nvrtcProgram_t, char*);
  nvrtcResult_t (*log_size)(nvrtcProgram_t, size_t*);
  nvrtcResult_t (*log)(nvrtcProgram_t, char*);
  nvrtcResult_t (*destroy)(nvrtcProgram_t*);
  nvrtcResult_t (*version)(int*, int*);
  bool ok = false;
};

Nvrtc* nvrtc() {
  static Nvrtc n;
  static std::once_flag once;
  std::call_once(once, [] {
    // The toolkit's NVRTC first (same release as the nvcc that built the AOT kernels; the copy torch
    // bundles can be older and reject sm_100a-only PTX such as 256-bit loads), then the soname.
    const char* names[] = {"/usr/local/cuda/lib64/libnvrtc.so.12", "libnvrtc.so.12", "libnvrtc.so"};
    void* h = nullptr;
    for (const char* nm : names)
      if ((h = dlopen(nm, RTLD_NOW | RTLD_LOCAL))) break;
    if (!h) return;
    n.create = (decltype(n.create))dlsym(h, "nvrtcCreateProgram");
    n.compile = (decltype(n.compile))dlsym(h, "nvrtcCompileProgram");
    n.cubin_size = (decltype(n.cubin_size))dlsym(h, "nvrtcGetCUBINSize");
    n.cubin = (decltype(n.cubin))dlsym(h, "nvrtcGetCUBIN");
    n.log_size = (decltype(n.log_size))dlsym(h, "nvrtcGetProgramLogSize");
    n.log = (decltype(n.log))dlsym(h, "nvrtcGetProgramLog");
    n.destroy = (decltype(n.destroy))dlsym(h, "nvrtcDestroyProgram");
    n.version = (decltype(n.version))dlsym(h, "nvrtcVersion");
    n.ok = n.create && n.compile && n.cubin_size && n.cubin && n.log_size && n.log && n.destroy;
  });
  return &n;
}

const char* kPreamble = R"PRE(
#define BLU_JIT 1
typedef unsigned long long uint64_t;
typedef long long int64_t;
typedef unsigned int uint32_t;
typedef int int32_t;
typedef unsigned short uint16_t;
typedef unsigned char uint8_t;
typedef unsigned long long uintptr_t;
#define INT32_MAX 2147483647
#define INT32_MIN (-2147483647 - 1)
#define INT64_MAX 9223372036854775807LL
#define INT64_MIN (-9223372036854775807LL - 1)
#define UINT64_MAX 18446744073709551615ULL
)PRE";

template <class T>
std::string arr(const T* a, int n, int pad) {
  std::string s = "{";
  for (int i = 0; i < pad; ++i) {
    if (i) s += ",";
    s += std::to_string(i < n ? (long long)a[i] : 0LL);
    if (sizeof(T) == 8) s += "LL";
  }
  return s + "}";
}
std::string arru(const uint64_t* a, int n, int pad) {
  std::string s = "{";
  for (int i = 0; i < pad; ++i) {
    if (i) s += ",";
    s += std::to_string(i < n ? (unsigned long long)a[i] : 0ULL) + "ULL";
  }
  return s + "}";
}

std::string spec_source(const char* name, const Layout& L, uint32_t S, const uint32_t* soff) {
  int kdt[kMaxKeys], vdt[kMaxVals], kind[kMaxFields], col[kMaxFields], goff[kMaxFields], sg[kMaxFields], si[kMaxFields];
  for (int k = 0; k < L.n_keys; ++k) kdt[k] = L.key_dtype[k];
  for (int c = 0; c < L.n_vals; ++c) vdt[c] = L.val_dtype[c];
  for (int j = 0; j < L.n_fields; ++j) {
    kind[j] = L.f[j].kind;
    col[j] = L.f[j].col;
    goff[j] = L.f[j].goff;
    sg[j] = L.f[j].sgroup;
    si[j] = L.f[j].sidx;
  }
  std::string s = "namespace blu {\nstruct ";
  s += name;
  s += " {\n  static constexpr bool kStatic = true;\n";
  s += "  static constexpr int NK = " + std::to_string(L.n_keys) + ";\n";
  s += "  static constexpr int SPARSE = " + std::to_string(L.sparse) + ";\n";
  s += "  static constexpr int PADK = " + std::to_string(L.pad_keys) + ";\n";
  s += "  static constexpr int KDT[8] = " + arr(kdt, L.n_keys, 8) + ";\n";
  s += "  static constexpr unsigned long long DICT[8] = " + arru(L.dict, L.n_keys, 8) + ";\n";
  s += "  static constexpr unsigned long long STRIDE[8] = " + arru(L.stride, L.n_keys, 8) + ";\n";
  s += "  static constexpr int NV = " + std::to_string(L.n_vals) + ";\n";
  s += "  static constexpr int VDT[16] = " + arr(vdt, L.n_vals, 16) + ";\n";
  s += "  static constexpr int NF = " + std::to_string(L.n_fields) + ";\n";
  s += "  static constexpr int KIND[24] = " + arr(kind, L.n_fields, 24) + ";\n";
  s += "  static constexpr int COL[24] = " + arr(col, L.n_fields, 24) + ";\n";
  s += "  static constexpr int GOFF[24] = " + arr(goff, L.n_fields, 24) + ";\n";
  s += "  static constexpr int SGROUP[24] = " + arr(sg, L.n_fields, 24) + ";\n";
  s += "  static constexpr int SIDX[24] = " + arr(si, L.n_fields, 24) + ";\n";
  s += "  static constexpr unsigned long long SLOT = " + std::to_string(L.slot_bytes) + "ULL;\n";
  s += "  static constexpr unsigned long long DOMAIN = " + std::to_string((unsigned long long)L.domain) + "ULL;\n";
  s += "  static constexpr int LOCKOFF = " + std::to_string(L.lock_off) + ";\n";
  // the launch's shared-memory table (path (a) dense table, hot-key front or bucket table): entries
  // and per-field byte offsets, so field addresses are immediates instead of parameter loads
  int so[kMaxFields];
  for (int j = 0; j < L.n_fields; ++j) so[j] = soff ? (int)soff[j] : 0;
  s += "  static constexpr unsigned STAB = " + std::to_string(S) + "u;\n";
  s += "  static constexpr int SOFF[24] = " + arr(so, L.n_fields, 24) + ";\n";
  s += "  static constexpr int HOTREG = " + std::to_string(jit_hot_reg()) + ";\n";
  // MIN/MAX skip bounds (opt-in): 1 = path (a) dense tables, 2 = also the rank front
  const char* mb = benv("BLU_GBY_MMBOUND");
  s += std::string("  static constexpr int MMBOUND = ") + (mb && (mb[0] == '1' || mb[0] == '2') ? mb[0] : '0') + ";\n";
  const char* dd = benv("BLU_GBY_DEDUPE");
  s += std::string("  static constexpr int DEDUPE = ") + (dd && dd[0] == '1' ? "1" : "0") + ";\n";
  s += "};\n}  // namespace blu\n";
  return s;
}

uint64_t fnv1a(const std::string& s) {
  uint64_t h = 1469598103934665603ull;
  for (unsigned char c : s) {
    h ^= c;
    h *= 1099511628211ull;
  }
  return h;
}

std::string cache_dir() {
  const char* x = getenv("XDG_CACHE_HOME");
  std::string d = x && *x ? std::string(x) : std::string(getenv("HOME") ? getenv("HOME") : "/tmp") + "/.cache";
  d += "/blugby";
  mkdir(d.c_str(), 0755);
  return d;
}

struct Entry {
  cudaLibrary_t lib = nullptr;
  std::map<std::string, cudaKernel_t> kernels;
  bool failed = false;
};

std::mutex g_mu;
std::map<std::string, Entry> g_cache;  // key: full source text + device

bool compile(const std::string& src, std::vector<char>& cubin, std::string& log) {
  Nvrtc* n = nvrtc();
  if (!n->ok) {
    log = "NVRTC not available";
    return false;
  }
  nvrtcProgram_t prog;
  if (n->create(&prog, src.c_str(), "blu_jit.cu", 0, nullptr, nullptr) != 0) {
    log = "nvrtcCreateProgram failed";
    return false;
  }
  int major = 0, minor = 0;
  if (n->version) n->version(&major, &minor);
  const bool ldg256 = major > 12 || (major == 12 && minor >= 9);  // 256-bit LDG needs PTX ISA 8.8
  const char* opts[] = {"--gpu-architecture=sm_100a", "--std=c++17", "-lineinfo", "--device-as-default-execution-space", "--diag-suppress=128,177",
                        "-DNDEBUG", ldg256 ? "-DBLU_LDG256=1" : "-DBLU_LDG256=0"};
  int rc = n->compile(prog, 7, opts);
  size_t ls = 0;
  n->log_size(prog, &ls);
  log.assign(ls, '\0');
  if (ls) n->log(prog, &log[0]);
  if (rc != 0) {
    n->destroy(&prog);
    return false;
  }
  size_t cs = 0;
  n->cubin_size(prog, &cs);
  cubin.resize(cs);
  n->cubin(prog, cubin.data());
  n->destroy(&prog);
  return true;
}

}  // namespace

// The rank front's 0, 1 or 2 hottest keys summed in registers (BLU_GBY_HOT_REG=0/1/2)
int jit_hot_reg() {
  const char* e = benv("BLU_GBY_HOT_REG");  // read per plan execution (tests switch it)
  // default 1: C4 8.91 vs 9.18-9.36 ms (640 threads, one key); two keys measured slower (11.8-12.0 ms)
  const int h = e ? atoi(e) : 1;
  return jit_enabled() ? (h < 0 ? 0 : h > 2 ? 2 : h) : 0;
}

bool jit_enabled() {
  const char* e = benv("BLU_GBY_JIT");
  return !(e && e[0] == '0');
}

// Returns a kernel handle (usable with cudaLaunchKernel / cudaFuncSetAttribute) for `entry` in the
// program made of `spec_src` + `entry_src`, or nullptr (caller falls back to the generic kernels).
thread_local JitProbe* t_probe = nullptr;
void jit_probe_begin(JitProbe* pr) { t_probe = pr; }
void jit_probe_end() { t_probe = nullptr; }
bool jit_probe_active() { return t_probe != nullptr; }

// Experiment switches (benchmarks): BLU_GBY_JIT_DEFS=A,B compiles the kernels with #define A 1 ...
static std::string jit_defs() {
  std::string out;
  const char* d = benv("BLU_GBY_JIT_DEFS");
  if (!d) return out;
  std::string cur;
  for (const char* c = d;; ++c) {
    if (*c == ',' || *c == 0) {
      if (!cur.empty()) out += "#define " + cur + " 1\n";
      cur.clear();
      if (!*c) break;
    } else {
      cur += *c;
    }
  }
  return out;
}

// Compile-only probe (blu_gby_jit_probe): NVRTC compile of the program, no module load, no launch.
static void probe_compile(const std::string& body) {
  JitProbe& pr = *t_probe;
  ++pr.programs;
  if (!nvrtc()->ok) {
    ++pr.failed;
    pr.log += "NVRTC not found\n";
    return;
  }
  std::string src = std::string(kPreamble) + jit_defs() + kSrc_blu_params_h + "\n" + kSrc_blu_device_cuh + "\n" + body;
  std::vector<char> cubin;
  std::string log;
  if (!compile(src, cubin, log) || cubin.empty()) {
    ++pr.failed;
    pr.log += log.empty() ? std::string("compile failed\n") : log;
  }
}

const void* jit_kernel(const std::string& spec_src, const std::string& entry_src, const char* entry) {
  if (!jit_enabled()) return nullptr;
  if (const char* dump = benv("BLU_GBY_JIT_DUMP")) {  // write the program text (SASS inspection offline)
    std::string fn = std::string(dump) + "/" + entry + ".cu";
    std::string src = std::string(kPreamble) + jit_defs() + kSrc_blu_params_h + "\n" + kSrc_blu_device_cuh + "\n" +
                      spec_src + entry_src;
    if (FILE* f = fopen(fn.c_str(), "w")) {
      fwrite(src.data(), 1, src.size(), f);
      fclose(f);
    }
    std::vector<char> cubin;
    std::string log;
    if (compile(src, cubin, log))
      if (FILE* f = fopen((std::string(dump) + "/" + entry + ".cubin").c_str(), "wb")) {
        fwrite(cubin.data(), 1, cubin.size(), f);
        fclose(f);
      }
  }
  if (t_probe) {
    probe_compile(jit_defs() + spec_src + entry_src);
    return nullptr;
  }
  int dev = 0;
  cudaGetDevice(&dev);
  const std::string body = jit_defs() + spec_src + entry_src;
  const std::string key = std::to_string(dev) + "\n" + body;
  std::lock_guard<std::mutex> lk(g_mu);
  Entry& e = g_cache[key];
  if (e.failed) return nullptr;
  if (!e.lib) {
    std::string src = std::string(kPreamble) + jit_defs() + kSrc_blu_params_h + "\n" + kSrc_blu_device_cuh + "\n" + body;
    int major = 0, minor = 0;
    if (nvrtc()->ok && nvrtc()->version) nvrtc()->version(&major, &minor);
    const uint64_t h = fnv1a(src + std::to_string(major) + "." + std::to_string(minor));
    char fn[64];
    snprintf(fn, sizeof fn, "/jit_%016llx.cubin", (unsigned long long)h);
    const std::string path = cache_dir() + fn;
    std::vector<char> cubin;
    if (FILE* f = fopen(path.c_str(), "rb")) {
      fseek(f, 0, SEEK_END);
      long sz = ftell(f);
      fseek(f, 0, SEEK_SET);
      cubin.resize(sz > 0 ? (size_t)sz : 0);
      if (sz <= 0 || fread(cubin.data(), 1, (size_t)sz, f) != (size_t)sz) cubin.clear();
      fclose(f);
    }
    if (cubin.empty()) {
      std::string log;
      if (!compile(src, cubin, log)) {
        if (benv("BLU_GBY_JIT_VERBOSE")) fprintf(stderr, "blugby JIT compile failed:\n%s\n", log.c_str());
        e.failed = true;
        return nullptr;
      }
      std::string tmp = path + ".tmp" + std::to_string(getpid());
      if (FILE* f = fopen(tmp.c_str(), "wb")) {
        fwrite(cubin.data(), 1, cubin.size(), f);
        fclose(f);
        rename(tmp.c_str(), path.c_str());
      }
    }
    if (cudaLibraryLoadData(&e.lib, cubin.data(), nullptr, nullptr, 0, nullptr, nullptr, 0) != cudaSuccess) {
      cudaGetLastError();
      e.failed = true;
      e.lib = nullptr;
      return nullptr;
    }
  }
  auto it = e.kernels.find(entry);
  if (it != e.kernels.end()) return (const void*)it->second;
  cudaKernel_t k = nullptr;
  if (cudaLibraryGetKernel(&k, e.lib, entry) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  e.kernels[entry] = k;
  return (const void*)k;
}

std::string jit_spec(const char* name, const Layout& L, uint32_t S, const uint32_t* soff) {
  return spec_source(name, L, S, soff);
}

}  // namespace blu
