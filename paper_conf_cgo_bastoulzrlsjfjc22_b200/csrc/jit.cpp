// jit.cpp — compiles generated kernels for sm_100a with NVRTC.
//
// NVRTC is loaded with dlopen so that libfop.so loads (and plans) on a host
// without CUDA; compilation itself needs no GPU.  Identical sources are
// compiled once per process.
#include <dlfcn.h>

#include <cstdlib>
#include <mutex>
#include <string>
#include <unordered_map>
#include <vector>

#include "fop_internal.h"

namespace fop {

namespace {
typedef int nvrtcResult;
typedef struct _nvrtcProgram* nvrtcProgram;
struct Nvrtc {
  bool ok = false;
  std::string why;
  nvrtcResult (*create)(nvrtcProgram*, const char*, const char*, int, const char* const*, const char* const*);
  nvrtcResult (*compile)(nvrtcProgram, int, const char* const*);
  nvrtcResult (*logsize)(nvrtcProgram, size_t*);
  nvrtcResult (*log)(nvrtcProgram, char*);
  nvrtcResult (*cubinsize)(nvrtcProgram, size_t*);
  nvrtcResult (*cubin)(nvrtcProgram, char*);
  nvrtcResult (*destroy)(nvrtcProgram*);
  const char* (*errstr)(nvrtcResult);
};

Nvrtc& nvrtc() {
  static Nvrtc n;
  static std::once_flag once;
  std::call_once(once, [] {
    // The toolkit's NVRTC (12.9) first, by absolute path: a process that
    // imported torch already holds torch's bundled libnvrtc.so.12 (12.8),
    // whose ptxas rejects the sm_100a 256-bit LDG/STG forms; loading by
    // soname would silently return that copy.
    const char* cands[] = {getenv("FOP_NVRTC"), "/usr/local/cuda/lib64/libnvrtc.so.12",
                           "/usr/local/cuda-12.9/lib64/libnvrtc.so.12", "libnvrtc.so.12"};
    void* h = nullptr;
    for (const char* c : cands)
      if (c && (h = dlopen(c, RTLD_NOW | RTLD_LOCAL))) break;
    if (!h) {
      n.why = "cannot dlopen libnvrtc.so.12";
      return;
    }
#define SYM(field, name)                                 \
  *(void**)(&n.field) = dlsym(h, name);                  \
  if (!n.field) {                                        \
    n.why = std::string("libnvrtc lacks ") + name;       \
    return;                                              \
  }
    SYM(create, "nvrtcCreateProgram");
    SYM(compile, "nvrtcCompileProgram");
    SYM(logsize, "nvrtcGetProgramLogSize");
    SYM(log, "nvrtcGetProgramLog");
    SYM(cubinsize, "nvrtcGetCUBINSize");
    SYM(cubin, "nvrtcGetCUBIN");
    SYM(destroy, "nvrtcDestroyProgram");
    SYM(errstr, "nvrtcGetErrorString");
#undef SYM
    n.ok = true;
  });
  return n;
}

std::mutex cache_mu;
std::unordered_map<std::string, std::vector<char>>& cache() {
  static std::unordered_map<std::string, std::vector<char>> c;
  return c;
}
}  // namespace

bool jit_available() { return nvrtc().ok; }

void jit_compile(Launch& L) {
  {
    std::lock_guard<std::mutex> g(cache_mu);
    auto it = cache().find(L.src);
    if (it != cache().end()) {
      L.cubin = it->second;
      return;
    }
  }
  Nvrtc& n = nvrtc();
  if (!n.ok) fail(FOP_E_JIT, "NVRTC unavailable: " + n.why);
  nvrtcProgram prog;
  const char* hdr_src[] = {kDeviceHeader};
  const char* hdr_name[] = {"fop_device.cuh"};
  std::string fname = L.name + ".cu";
  if (n.create(&prog, L.src.c_str(), fname.c_str(), 1, hdr_src, hdr_name) != 0)
    fail(FOP_E_JIT, "nvrtcCreateProgram failed");
  // -fmad=false: ptxas may not contract a multiply and an add into one FMA,
  // even for the packed mul/add.rn.f32x2 forms (it does without this flag);
  // every FMA the kernels use is an explicit fma instruction.
  const char* opts[] = {"-arch=sm_100a", "-std=c++17", "-lineinfo", "-fmad=false"};
  nvrtcResult r = n.compile(prog, 4, opts);
  if (r != 0) {
    size_t ls = 0;
    n.logsize(prog, &ls);
    std::string log(ls, '\0');
    if (ls) n.log(prog, &log[0]);
    n.destroy(&prog);
    fail(FOP_E_JIT, std::string("NVRTC: ") + n.errstr(r) + "\n" + log + "\n--- source ---\n" + L.src);
  }
  size_t cs = 0;
  n.cubinsize(prog, &cs);
  L.cubin.resize(cs);
  n.cubin(prog, L.cubin.data());
  n.destroy(&prog);
  std::lock_guard<std::mutex> g(cache_mu);
  cache()[L.src] = L.cubin;
}

}  // namespace fop
