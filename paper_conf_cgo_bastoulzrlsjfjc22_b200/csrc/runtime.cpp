// runtime.cpp — loads the compiled kernels into the caller's CUDA context and
// launches them on the caller's stream (the hot path of fop_run).
//
// The CUDA driver API is reached through dlopen("libcuda.so.1") so the library
// loads on hosts without a driver (planning/compiling works there; running
// returns FOP_E_CUDA).  The caller (PyTorch) owns every device buffer and the
// stream; fop_run only enqueues: one kernel per launch of the plan.
#include <dlfcn.h>

#include <algorithm>

#include <cstddef>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>

#include "fop_internal.h"

namespace fop {

namespace {
typedef int CUresult;
typedef void* CUcontext;
typedef void* CUmodule;
typedef void* CUfunction;
typedef void* CUstream;
typedef int CUdevice;
typedef unsigned long long CUdeviceptr;
enum { CU_POINTER_ATTRIBUTE_CONTEXT = 1, CU_POINTER_ATTRIBUTE_DEVICE_ORDINAL = 9 };

struct Cuda {
  bool ok = false;
  std::string why;
  CUresult (*init)(unsigned);
  CUresult (*ctx_get)(CUcontext*);
  CUresult (*ctx_set)(CUcontext);
  CUresult (*primary_retain)(CUcontext*, CUdevice);
  CUresult (*ptr_attr)(void*, int, CUdeviceptr);
  CUresult (*mod_load)(CUmodule*, const void*);
  CUresult (*mod_func)(CUfunction*, CUmodule, const char*);
  CUresult (*launch)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, CUstream,
                     void**, void**);
  CUresult (*h2d)(CUdeviceptr, const void*, size_t, CUstream);
  CUresult (*d2h)(void*, CUdeviceptr, size_t, CUstream);
  CUresult (*errstr)(CUresult, const char**);
  CUresult (*func_attr)(CUfunction, int, int);
  CUresult (*ev_create)(void**, unsigned);
  CUresult (*ev_record)(void*, CUstream);
  CUresult (*ev_sync)(void*);
  CUresult (*ev_elapsed)(float*, void*, void*);
  CUresult (*ev_destroy)(void*);
  CUresult (*stream_capturing)(CUstream, int*);
  CUresult (*stream_create)(CUstream*, unsigned);
  CUresult (*stream_wait)(CUstream, void*, unsigned);
  CUresult (*launch_ex)(const void* config, CUfunction, void**, void**);
  CUresult (*mem_alloc)(CUdeviceptr*, size_t);
  CUresult (*mem_free)(CUdeviceptr);
  CUresult (*memset8)(CUdeviceptr, unsigned char, size_t);
  CUresult (*ctx_sync)();
  CUresult (*ipc_get)(fop_ipc_handle*, CUdeviceptr);
  CUresult (*ipc_open)(CUdeviceptr*, fop_ipc_handle, unsigned);
  CUresult (*ipc_close)(CUdeviceptr);
  CUresult (*tmap_encode)(void*, int, unsigned, void*, const uint64_t*, const uint64_t*, const unsigned*,
                          const unsigned*, int, int, int, int);
};
enum { CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES = 8, CU_FUNC_ATTRIBUTE_PREFERRED_SHARED_MEMORY_CARVEOUT = 9 };
// cuLaunchKernelEx configuration (layout of cuda.h's CUlaunchConfig /
// CUlaunchAttribute; the attribute value is a 64-byte union)
struct LaunchAttr {
  int id;
  char pad[4];
  unsigned char value[64];
};
struct LaunchConfig {
  unsigned grid[3], block[3], smem;
  CUstream stream;
  LaunchAttr* attrs;
  unsigned nattrs;
};
enum { CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION = 6 };
static_assert(sizeof(LaunchAttr) == 72, "CUlaunchAttribute layout");
static_assert(offsetof(LaunchConfig, stream) == 32 && offsetof(LaunchConfig, nattrs) == 48, "CUlaunchConfig layout");
enum { TMAP_UINT16 = 1, TMAP_INTERLEAVE_NONE = 0, TMAP_SWIZZLE_128B = 3, TMAP_L2_PROMO_256B = 3, TMAP_OOB_NONE = 0 };

Cuda& cuda() {
  static Cuda c;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
      c.why = "cannot dlopen libcuda.so.1 (no NVIDIA driver on this host)";
      return;
    }
#define SYM(field, name)                               \
  *(void**)(&c.field) = dlsym(h, name);                \
  if (!c.field) {                                      \
    c.why = std::string("libcuda lacks ") + name;      \
    return;                                            \
  }
    SYM(init, "cuInit");
    SYM(ctx_get, "cuCtxGetCurrent");
    SYM(ctx_set, "cuCtxSetCurrent");
    SYM(primary_retain, "cuDevicePrimaryCtxRetain");
    SYM(ptr_attr, "cuPointerGetAttribute");
    SYM(mod_load, "cuModuleLoadData");
    SYM(mod_func, "cuModuleGetFunction");
    SYM(launch, "cuLaunchKernel");
    SYM(h2d, "cuMemcpyHtoDAsync_v2");
    SYM(d2h, "cuMemcpyDtoHAsync_v2");
    SYM(errstr, "cuGetErrorString");
    SYM(func_attr, "cuFuncSetAttribute");
    SYM(ev_create, "cuEventCreate");
    SYM(ev_record, "cuEventRecord");
    SYM(ev_sync, "cuEventSynchronize");
    SYM(ev_elapsed, "cuEventElapsedTime");
    SYM(ev_destroy, "cuEventDestroy_v2");
    SYM(stream_capturing, "cuStreamIsCapturing");
    SYM(stream_create, "cuStreamCreate");
    SYM(stream_wait, "cuStreamWaitEvent");
    SYM(tmap_encode, "cuTensorMapEncodeTiled");
    SYM(launch_ex, "cuLaunchKernelEx");
    SYM(mem_alloc, "cuMemAlloc_v2");
    SYM(mem_free, "cuMemFree_v2");
    SYM(memset8, "cuMemsetD8_v2");
    SYM(ctx_sync, "cuCtxSynchronize");
    SYM(ipc_get, "cuIpcGetMemHandle");
    SYM(ipc_open, "cuIpcOpenMemHandle_v2");
    SYM(ipc_close, "cuIpcCloseMemHandle");
#undef SYM
    if (c.init(0) != 0) {
      c.why = "cuInit failed";
      return;
    }
    c.ok = true;
  });
  return c;
}

void check(CUresult r, const char* what) {
  if (r == 0) return;
  const char* s = nullptr;
  cuda().errstr(r, &s);
  fail(FOP_E_CUDA, std::string(what) + ": " + (s ? s : "unknown CUDA error") + " (" + std::to_string(r) + ")");
}

CUcontext current_context(void* const* ptrs, int n) {
  Cuda& c = cuda();
  CUcontext ctx = nullptr;
  check(c.ctx_get(&ctx), "cuCtxGetCurrent");
  if (ctx) return ctx;
  for (int i = 0; i < n; i++) {
    if (!ptrs[i]) continue;
    int dev = -1;
    if (c.ptr_attr(&dev, CU_POINTER_ATTRIBUTE_DEVICE_ORDINAL, (CUdeviceptr)ptrs[i]) == 0 && dev >= 0) {
      check(c.primary_retain(&ctx, dev), "cuDevicePrimaryCtxRetain");
      check(c.ctx_set(ctx), "cuCtxSetCurrent");
      return ctx;
    }
  }
  fail(FOP_E_CUDA, "no current CUDA context and no device pointer to infer one from");
}

int64_t span_bytes(const fop_tensor& t) {
  int64_t n = 1;
  for (int r = 0; r < t.rank; r++) {
    if (t.shape[r] == 0) return 0;   // empty tensor
    n += (t.shape[r] - 1) * t.stride[r];
  }
  return n * esize(t.dtype);
}

CUfunction load_fn(const Launch& L, std::vector<void*>& mods) {
  CUmodule m = nullptr;
  CUfunction f = nullptr;
  check(cuda().mod_load(&m, L.cubin.data()), "cuModuleLoadData");
  check(cuda().mod_func(&f, m, L.name.c_str()), "cuModuleGetFunction");
  if (L.tma && L.smem > 48 * 1024)
    check(cuda().func_attr(f, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, (int)L.smem), "cuFuncSetAttribute");
  // FOP_CARVEOUT=<percent>: one shared-memory carveout preference for every kernel
  // (measurement knob: kernels with different carveouts back to back make the SM
  // reconfigure its L1/shared split between them)
  if (const char* cv = std::getenv("FOP_CARVEOUT"); cv && *cv)
    check(cuda().func_attr(f, CU_FUNC_ATTRIBUTE_PREFERRED_SHARED_MEMORY_CARVEOUT, std::atoi(cv)), "cuFuncSetAttribute");
  else if (const char* ct = std::getenv("FOP_CARVEOUT_TMA"); L.tma && ct && *ct)   // the TMA kernels only
    check(cuda().func_attr(f, CU_FUNC_ATTRIBUTE_PREFERRED_SHARED_MEMORY_CARVEOUT, std::atoi(ct)), "cuFuncSetAttribute");
  mods.push_back(m);
  return f;
}

Plan::Loaded& loaded_for(Plan& p, CUcontext ctx) {
  for (auto& l : p.loaded)
    if (l.ctx == ctx) return l;
  Plan::Loaded l;
  l.ctx = ctx;
  for (size_t i = 0; i < p.launches.size(); i++) {
    l.fns.push_back(load_fn(p.launches[i], l.mods));
    l.nmods.push_back(nullptr);
    l.nfns.push_back(nullptr);
    std::vector<void*> vf;
    if (i < p.variants.size())
      for (const Launch& V : p.variants[i]) vf.push_back(load_fn(V, l.mods));
    l.vfns.push_back(vf);
    l.choice.push_back(vf.empty() ? 0 : -1);
  }
  p.loaded.push_back(l);
  return p.loaded.back();
}

CUfunction narrow_fn(Plan& p, Plan::Loaded& l, size_t i) {
  if (l.nfns[i]) return l.nfns[i];
  Launch& N = p.narrow[i];
  if (N.cubin.empty()) {
    generate(p, N, (int)i);
    jit_compile(N);
  }
  CUmodule m = nullptr;
  CUfunction f = nullptr;
  check(cuda().mod_load(&m, N.cubin.data()), "cuModuleLoadData(narrow)");
  check(cuda().mod_func(&f, m, N.name.c_str()), "cuModuleGetFunction(narrow)");
  l.nmods[i] = m;
  l.nfns[i] = f;
  return f;
}

// L2 conditioning for the auto-tuner, compiled once per process and loaded
// once per context: fop_l2_flush streams a scratch buffer larger than L2
// (kTuneScratchBytes; B200's L2 is 126 MB) through it; fop_l2_dirty then
// writes the first bytes of the scratch, leaving that many dirty lines.
constexpr size_t kTuneScratchBytes = size_t(320) << 20;
CUfunction l2_flush_fn(Plan::Loaded& l) {
  if (l.flush_fn) return (CUfunction)l.flush_fn;
  static Launch F;
  static std::once_flag once;
  static std::string err;
  std::call_once(once, [] {
    F.name = "fop_l2_flush";
    F.src =
        "#include \"fop_device.cuh\"\n"
        "extern \"C\" __global__ void __launch_bounds__(256) fop_l2_flush(const uint4* p, unsigned long long n) {\n"
        "  unsigned acc = 0;\n"
        "  for (unsigned long long i = blockIdx.x * 256ull + threadIdx.x; i < n; i += gridDim.x * 256ull) {\n"
        "    unsigned a, b, c, e;\n"
        "    asm volatile(\"ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];\"\n"
        "                 : \"=r\"(a), \"=r\"(b), \"=r\"(c), \"=r\"(e) : \"l\"(p + i));\n"
        "    acc ^= a ^ e;\n"
        "  }\n"
        "  // a data-dependent store keeps the loads (scratch contents are garbage anyway)\n"
        "  if (acc == 0x9e3779b9u) ((unsigned*)p)[threadIdx.x] = acc;\n"
        "}\n"
        "extern \"C\" __global__ void __launch_bounds__(256) fop_l2_dirty(uint4* p, unsigned long long n) {\n"
        "  for (unsigned long long i = blockIdx.x * 256ull + threadIdx.x; i < n; i += gridDim.x * 256ull)\n"
        "    p[i] = make_uint4(0u, 0u, 0u, 0u);\n"
        "}\n";
    try {
      jit_compile(F);
    } catch (const Error& e) {
      err = e.msg;
    }
  });
  if (F.cubin.empty()) return nullptr;
  CUmodule m = nullptr;
  CUfunction f = nullptr, w = nullptr;
  if (cuda().mod_load(&m, F.cubin.data()) != 0 || cuda().mod_func(&f, m, F.name.c_str()) != 0 ||
      cuda().mod_func(&w, m, "fop_l2_dirty") != 0)
    return nullptr;
  l.mods.push_back(m);
  l.flush_fn = f;
  l.dirty_fn = w;
  return f;
}
}  // namespace

void* current_context_or_null() {
  Cuda& c = cuda();
  if (!c.ok) return nullptr;
  CUcontext ctx = nullptr;
  if (c.ctx_get(&ctx) != 0) return nullptr;
  return ctx;
}

fop_status run_plan(Plan& p, void* const* ptrs, int nptrs, void* ws, void* stream, void* const* host_ptrs,
                    const fop_peer_group* peers, bool pdl) {
  const fop_desc& d = p.desc;
  if (nptrs != d.ntensors) fail(FOP_E_INVALID, "nptrs must equal desc.ntensors");
  if (p.peer_bytes) {   // every argument error is caught before any launch (the peers would wait)
    if (!peers) fail(FOP_E_INVALID, "this plan exchanges partial results across a peer group: run it with fop_run_peer");
    if (peers->world != p.opts.peer_world)
      fail(FOP_E_INVALID, "peer group world " + std::to_string(peers->world) + " != plan peer_world " +
                              std::to_string(p.opts.peer_world));
    if (peers->rank < 0 || peers->rank >= peers->world) fail(FOP_E_INVALID, "peer rank out of range");
    for (int q = 0; q < peers->world; q++)
      if (!peers->buf[q] || ((uintptr_t)peers->buf[q] % 256))
        fail(FOP_E_INVALID, "exchange buffer of rank " + std::to_string(q) + " is NULL or not 256-byte aligned");
    for (const auto& L : p.launches)
      for (int t = 0; t < d.ntensors; t++)
        if (L.peer && ptrs[t] && ((uintptr_t)ptrs[t] % (uintptr_t)L.align[t]))
          fail(FOP_E_ALIGN, "tensor " + std::to_string(t) + " is not aligned for the planned vector width (peer "
                            "exchanges need the same kernel on every rank)");
  }
  for (auto& L : p.launches)
    if (L.cubin.empty()) fail(FOP_E_INVALID, "plan was built with opts.jit = 0: nothing to run");
  Cuda& c = cuda();
  if (!c.ok) fail(FOP_E_CUDA, c.why);
  if (p.ws_bytes && !ws) fail(FOP_E_INVALID, "this plan needs a workspace of fop_plan_workspace_bytes() bytes");
  for (int t = 0; t < d.ntensors; t++) {
    if (!ptrs[t] && d.t[t].role != FOP_TEMP && span_bytes(d.t[t]) > 0)
      fail(FOP_E_INVALID, "NULL pointer for tensor " + std::to_string(t));
    if (ptrs[t] && ((uintptr_t)ptrs[t] % esize(d.t[t].dtype)))
      fail(FOP_E_ALIGN, "tensor " + std::to_string(t) + " is not aligned to its element size");
  }
  if (const char* dbg = std::getenv("FOP_DEBUG_RUN"); dbg && *dbg == '1') {
    std::fprintf(stderr, "[fop] run_plan ws=%p stream=%p pdl=%d nlaunch=%zu ptrs:", ws, stream, (int)pdl,
                 p.launches.size());
    for (int t = 0; t < nptrs; t++) std::fprintf(stderr, " %p", ptrs[t]);
    std::fprintf(stderr, "\n");
  }
  bool any_copy = false;
  for (int t = 0; t < d.ntensors && host_ptrs; t++) any_copy |= host_ptrs[t] && span_bytes(d.t[t]) > 0;
  if (p.launches.empty() && !any_copy) return FOP_OK;   // every statement has an empty domain
  CUcontext ctx = current_context(ptrs, nptrs);
  CUstream st = (CUstream)stream;

  if (host_ptrs) {  // end-to-end: inputs host -> device
    for (int t = 0; t < d.ntensors; t++)
      if ((d.t[t].role == FOP_IN || d.t[t].role == FOP_INOUT) && host_ptrs[t] && span_bytes(d.t[t]) > 0)
        check(c.h2d((CUdeviceptr)ptrs[t], host_ptrs[t], (size_t)span_bytes(d.t[t]), st), "cuMemcpyHtoDAsync");
  }

  struct Args {  // mirrors FopArgs of fop_device.cuh

    char* p[16];
    char* ws;
    char* peer[8];
    unsigned rank, world;
    unsigned zero;   // always 0 (fop::nofuse's opaque zero)
  } args;
  std::memset(&args, 0, sizeof args);
  if (peers && p.peer_bytes) {
    for (int q = 0; q < peers->world; q++) args.peer[q] = (char*)peers->buf[q];
    args.rank = (unsigned)peers->rank;
    args.world = (unsigned)peers->world;
  }
  for (int t = 0; t < d.ntensors; t++) {
    args.p[t] = (char*)ptrs[t];
    if (d.t[t].role == FOP_TEMP && p.temp_off[t] >= 0) args.p[t] = (char*)ws + p.temp_off[t];
  }
  args.ws = (char*)ws;

  std::lock_guard<std::mutex> g(p.mu);
  Plan::Loaded& l = loaded_for(p, ctx);
  // pdl: the plan's first kernel is launched with programmatic stream
  // serialization (fop_run_many; the caller guarantees the plans are
  // independent).  The kernels carry no explicit trigger, so it starts when
  // the previous kernel completes (stream order kept) but its launch is
  // processed early (device/fop_device.cuh, programmatic dependent launch)
  bool pdl_next = pdl;
  auto launch = [&](CUfunction f, unsigned grid, unsigned block, unsigned smem, void** params, const char* what) {
    if (pdl_next) {
      pdl_next = false;
      LaunchAttr a;
      std::memset(&a, 0, sizeof a);
      a.id = CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION;
      a.value[0] = 1;
      LaunchConfig cfg;
      std::memset(&cfg, 0, sizeof cfg);
      cfg.grid[0] = grid;
      cfg.grid[1] = cfg.grid[2] = 1;
      cfg.block[0] = block;
      cfg.block[1] = cfg.block[2] = 1;
      cfg.smem = smem;
      cfg.stream = st;
      cfg.attrs = &a;
      cfg.nattrs = 1;
      check(c.launch_ex(&cfg, f, params, nullptr), what);
      return;
    }
    check(c.launch(f, grid, 1, 1, block, 1, 1, smem, st, params, nullptr), what);
  };
  auto launch_one = [&](Launch* G, CUfunction f) {
    if (G->tma) {  // tensor maps for this run's base addresses (cached for the last pair)
      const char* gin = args.p[G->tma_in_tensor] + G->tma_in_base * 2;
      const char* gout = args.p[G->tma_out_tensor] + G->tma_out_base * 2;
      if (gin != G->tma_last_in || gout != G->tma_last_out) {
        unsigned box[5] = {64, 64, 1, 1, 1}, es[5] = {1, 1, 1, 1, 1};
        const char* pe = std::getenv("FOP_TMA_L2PROMO");   // 0 none, 1 64B, 2 128B, 3 256B
        int promo = pe && *pe ? std::atoi(pe) : TMAP_L2_PROMO_256B;
        check(c.tmap_encode(&G->tma_map_in, TMAP_UINT16, (unsigned)G->tma_rank, (void*)gin, G->tma_in_dim,
                            G->tma_in_stride, box, es, TMAP_INTERLEAVE_NONE, TMAP_SWIZZLE_128B, promo,
                            TMAP_OOB_NONE), "cuTensorMapEncodeTiled(in)");
        check(c.tmap_encode(&G->tma_map_out, TMAP_UINT16, (unsigned)G->tma_rank, (void*)gout, G->tma_out_dim,
                            G->tma_out_stride, box, es, TMAP_INTERLEAVE_NONE, TMAP_SWIZZLE_128B, promo,
                            TMAP_OOB_NONE), "cuTensorMapEncodeTiled(out)");
        G->tma_last_in = gin;
        G->tma_last_out = gout;
      }
      void* params[] = {&args, &G->tma_map_in, &G->tma_map_out};
      launch(f, (unsigned)G->grid, (unsigned)G->block, (unsigned)G->smem, params, "cuLaunchKernel(tma)");
      return;
    }
    void* params[] = {&args};
    launch(f, (unsigned)G->grid, (unsigned)G->block, 0, params, "cuLaunchKernel");
  };

  // Auto-tuning (opts.autotune): the first run of a launch on this context
  // times each candidate geometry (CUDA events on the caller's stream) and
  // keeps the fastest.  All candidates compute the same results
  // (bit-identical for ASSIGN; reductions within R16), and the plan is
  // idempotent, so the extra launches only cost time once.
  //
  // Back-to-back launches on the same buffers would rank geometries by their
  // behaviour when repeating themselves: L2-hot for operators that fit in a
  // few L2s (BERT LayerNorm: that ranking kept a geometry 9 % slower from
  // HBM), and with the previous instance's tail and write-back overlapping
  // for large ones (cfg3: the register tiles tie back to back, the TMA tiles
  // are 4 % faster after another operator, profiles/r02/tune_protocol_r02.log).
  // So every timed launch is preceded by a read of a scratch buffer larger
  // than L2 (the previous launch's dirty lines are written back during it),
  // then by a write of as many bytes as the plan outputs: each candidate
  // starts as it would inside a pipeline, inputs in HBM and the previous
  // operator's outputs dirty in L2.  FOP_TUNE_HOT=1: back-to-back timing.
  auto tune = [&](size_t i) {
    int capturing = 0;
    if (c.stream_capturing(st, &capturing) != 0 || capturing) return -1;
    void *e0 = nullptr, *e1 = nullptr;
    check(c.ev_create(&e0, 0), "cuEventCreate");
    check(c.ev_create(&e1, 0), "cuEventCreate");
    CUfunction flush = nullptr;
    CUdeviceptr scratch = 0;
    const char* hot = std::getenv("FOP_TUNE_HOT");
    if (!(hot && *hot == '1')) {
      flush = l2_flush_fn(l);
      if (flush && c.mem_alloc(&scratch, kTuneScratchBytes) != 0) scratch = 0;   // no room: time L2-hot
      // defined contents: the flush kernel only reads it to evict L2, but compute-sanitizer's
      // initcheck (rightly) reports reads of never-written memory
      if (scratch && c.memset8(scratch, 0, kTuneScratchBytes) != 0) {
        c.mem_free(scratch);
        scratch = 0;
      }
    }
    // steady state of a pipeline: the inputs are not in L2 and the previous
    // launch's outputs are still dirty in it (written back during this one)
    int64_t out_bytes = 0;
    for (int t = 0; t < d.ntensors; t++)
      if (d.t[t].role == FOP_OUT || d.t[t].role == FOP_INOUT) out_bytes += span_bytes(d.t[t]);
    unsigned long long dirty16 = (unsigned long long)std::min<int64_t>(out_bytes, int64_t(96) << 20) / 16;
    auto run_flush = [&]() {
      unsigned long long n16 = kTuneScratchBytes / 16;
      const unsigned g = (unsigned)(p.opts.sm_count > 0 ? 2 * p.opts.sm_count : 296);
      void* fp[] = {&scratch, &n16};
      launch(flush, g, 256, 0, fp, "cuLaunchKernel(l2 flush)");
      if (dirty16) {
        void* dp[] = {&scratch, &dirty16};
        launch((CUfunction)l.dirty_fn, g, 256, 0, dp, "cuLaunchKernel(l2 dirty)");
      }
    };
    // hot: `reps` back-to-back launches of candidate k after one warm-up;
    // cold: the median of `reps` single launches, each after an L2 flush
    auto time_k = [&](size_t k, int reps) {
      Launch* G = k == 0 ? &p.launches[i] : &p.variants[i][k - 1];
      CUfunction f = k == 0 ? l.fns[i] : l.vfns[i][k - 1];
      launch_one(G, f);
      float ms = 0.f;
      if (scratch) {
        std::vector<float> v;
        for (int r = 0; r < reps; r++) {
          run_flush();
          check(c.ev_record(e0, st), "cuEventRecord");
          launch_one(G, f);
          check(c.ev_record(e1, st), "cuEventRecord");
          check(c.ev_sync(e1), "cuEventSynchronize");
          check(c.ev_elapsed(&ms, e0, e1), "cuEventElapsedTime");
          v.push_back(ms);
        }
        std::sort(v.begin(), v.end());
        return v[v.size() / 2];
      }
      check(c.ev_record(e0, st), "cuEventRecord");
      for (int r = 0; r < reps; r++) launch_one(G, f);
      check(c.ev_record(e1, st), "cuEventRecord");
      check(c.ev_sync(e1), "cuEventSynchronize");
      check(c.ev_elapsed(&ms, e0, e1), "cuEventElapsedTime");
      return ms / reps;
    };
    int reps = 7;
    if (!scratch) {
      // enough repetitions that a batch lasts >= 0.25 ms (event resolution ~2 us)
      float t0 = time_k(0, 3);
      reps = t0 > 0.f ? (int)(0.25f / t0) + 1 : 3;
      reps = reps < 3 ? 3 : (reps > 40 ? 40 : reps);
    }
    // the default geometry is the rule the sweeps settled on: a candidate
    // replaces it only when it is clearly faster (> 1.5 %), not on timing noise
    // (BERT LayerNorm: candidates within 3 % swapped ranks between runs; at 2 %
    // cfg2's 32-byte geometry, 2.0-3.0 % ahead in every cold timing and 6.5 %
    // in steady state, lost to the default in one bench run of three)
    int best = 0;
    float best_ms = 0.f, def_ms = 0.f;
    std::vector<float> tlog;
    for (size_t k = 0; k <= l.vfns[i].size(); k++) {
      float ms = time_k(k, reps);
      tlog.push_back(ms);
      if (k == 0) def_ms = ms;
      if (k == 0 || ms < best_ms) {
        best = (int)k;
        best_ms = ms;
      }
    }
    // Candidates the cold timing cannot tell apart (within 1 % of the best) are
    // ranked by back-to-back timing — how they sustain bandwidth once running —
    // instead of by the order they were timed in (cfg2: the 32-byte geometry and
    // a 16-byte one tie at 100.4 us cold, 6547 vs 6249 GB/s back to back).
    // Only for operators well past L2 (back to back, a smaller one would run L2-hot).
    int64_t all_bytes = 0;
    for (int t = 0; t < d.ntensors; t++)
      if (d.t[t].role != FOP_TEMP) all_bytes += span_bytes(d.t[t]);
    std::vector<float> hlog(tlog.size(), 0.f);
    if (scratch && all_bytes >= (int64_t(384) << 20) &&
        !(std::getenv("FOP_TUNE_TIEBREAK") && *std::getenv("FOP_TUNE_TIEBREAK") == '0')) {
      std::vector<size_t> tied;
      for (size_t k = 0; k < tlog.size(); k++)
        if (tlog[k] <= 1.01f * best_ms) tied.push_back(k);
      if (tied.size() > 1) {
        const int hreps = std::max(3, std::min(40, (int)(0.25f / std::max(best_ms, 1e-4f)) + 1));
        float hbest = 0.f;
        for (size_t k : tied) {
          Launch* G = k == 0 ? &p.launches[i] : &p.variants[i][k - 1];
          CUfunction f = k == 0 ? l.fns[i] : l.vfns[i][k - 1];
          run_flush();
          launch_one(G, f);   // warm-up
          float ms = 0.f;
          check(c.ev_record(e0, st), "cuEventRecord");
          for (int r = 0; r < hreps; r++) launch_one(G, f);
          check(c.ev_record(e1, st), "cuEventRecord");
          check(c.ev_sync(e1), "cuEventSynchronize");
          check(c.ev_elapsed(&ms, e0, e1), "cuEventElapsedTime");
          hlog[k] = ms / hreps;
          if (k == tied[0] || hlog[k] < hbest) {
            hbest = hlog[k];
            best = (int)k;
          }
        }
        best_ms = tlog[best];
      }
    }
    if (best != 0 && best_ms > 0.985f * def_ms) best = 0;
    if (const char* lg = std::getenv("FOP_TUNE_LOG"); lg && *lg == '1') {   // diagnostics: the candidates' times
      std::fprintf(stderr, "[fop tune] launch %zu (%s): %s", i, scratch ? "cold" : "hot", p.launches[i].name.c_str());
      for (size_t k = 0; k < tlog.size(); k++) {
        std::fprintf(stderr, " v%zu=%.1fus", k, 1e3f * tlog[k]);
        if (hlog[k] > 0.f) std::fprintf(stderr, "(hot %.1f)", 1e3f * hlog[k]);
      }
      std::fprintf(stderr, " -> v%d\n", best);
    }
    if (scratch) {
      c.ev_sync(e1);
      c.mem_free(scratch);
    }
    c.ev_destroy(e0);
    c.ev_destroy(e1);
    return best;
  };

  for (size_t i = 0; i < p.launches.size(); i++) {
    Launch& L = p.launches[i];
    bool aligned = true;
    for (int t = 0; t < d.ntensors; t++)
      if (args.p[t] && ((uintptr_t)args.p[t] % (uintptr_t)L.align[t])) aligned = false;
    if (!aligned) {
      launch_one(&p.narrow[i], narrow_fn(p, l, i));
      continue;
    }
    int ch = l.choice[i];
    if (ch < 0 && p.opts.variant >= 0) {   // a forced candidate (fop.h: opts.variant), no timing
      l.choice[i] = ch = p.opts.variant <= (int)p.variants[i].size() ? p.opts.variant : 0;
    } else if (ch < 0) {
      int t = tune(i);
      if (t >= 0) l.choice[i] = ch = t;
      else ch = 0;   // capturing: default geometry, tune on a later eager run
    }
    bool var_aligned = true;
    if (ch > 0)
      for (int t = 0; t < d.ntensors; t++)
        if (args.p[t] && ((uintptr_t)args.p[t] % (uintptr_t)p.variants[i][ch - 1].align[t])) var_aligned = false;
    if (ch > 0 && var_aligned) launch_one(&p.variants[i][ch - 1], l.vfns[i][ch - 1]);
    else launch_one(&L, l.fns[i]);
  }

  if (host_ptrs) {  // device -> host results
    for (int t = 0; t < d.ntensors; t++)
      if ((d.t[t].role == FOP_OUT || d.t[t].role == FOP_INOUT) && host_ptrs[t] && span_bytes(d.t[t]) > 0)
        check(c.d2h(host_ptrs[t], (CUdeviceptr)ptrs[t], (size_t)span_bytes(d.t[t]), st), "cuMemcpyDtoHAsync");
  }
  return FOP_OK;
}

// ---------------------------------------------------------------- peer buffers (CUDA IPC)
void peer_alloc(size_t bytes, void** dev_ptr, fop_ipc_handle* handle) {
  Cuda& c = cuda();
  if (!c.ok) fail(FOP_E_CUDA, c.why);
  if (!dev_ptr || !handle || !bytes) fail(FOP_E_INVALID, "NULL argument or zero size");
  CUcontext ctx = nullptr;
  check(c.ctx_get(&ctx), "cuCtxGetCurrent");
  if (!ctx) fail(FOP_E_CUDA, "no current CUDA context (select and initialise the device first)");
  CUdeviceptr p = 0;
  check(c.mem_alloc(&p, bytes), "cuMemAlloc");
  CUresult r = c.memset8(p, 0, bytes);
  if (r == 0) r = c.ctx_sync();
  if (r == 0) r = c.ipc_get(handle, p);
  if (r != 0) {
    c.mem_free(p);
    check(r, "exchange buffer (memset / cuIpcGetMemHandle)");
  }
  *dev_ptr = (void*)p;
}
void peer_free(void* dev_ptr) {
  Cuda& c = cuda();
  if (!c.ok) fail(FOP_E_CUDA, c.why);
  if (dev_ptr) check(c.mem_free((CUdeviceptr)dev_ptr), "cuMemFree");
}
void peer_open(const fop_ipc_handle* handle, void** dev_ptr) {
  Cuda& c = cuda();
  if (!c.ok) fail(FOP_E_CUDA, c.why);
  if (!dev_ptr || !handle) fail(FOP_E_INVALID, "NULL argument");
  CUcontext ctx = nullptr;
  check(c.ctx_get(&ctx), "cuCtxGetCurrent");
  if (!ctx) fail(FOP_E_CUDA, "no current CUDA context (select and initialise the device first)");
  CUdeviceptr p = 0;
  check(c.ipc_open(&p, *handle, 1 /* CU_IPC_MEM_LAZY_ENABLE_PEER_ACCESS */), "cuIpcOpenMemHandle");
  *dev_ptr = (void*)p;
}
void peer_close(void* dev_ptr) {
  Cuda& c = cuda();
  if (!c.ok) fail(FOP_E_CUDA, c.why);
  if (dev_ptr) check(c.ipc_close((CUdeviceptr)dev_ptr), "cuIpcCloseMemHandle");
}

// ---------------------------------------------------------------- host pipeline
// fop_run_host_many: independent plans end to end from host buffers with the
// copies pipelined over two internal streams per context (created once, kept
// for the process): all inputs host->device in order on the first, each
// plan's kernels on the caller's stream once its inputs are in, its outputs
// device->host on the second while later inputs are still arriving.  The
// first copies wait for prior work on the caller's stream (which may still
// read the same device buffers) and the caller's stream waits for the last
// copy, so calls stay ordered with everything else on that stream.
namespace {
struct CopyStreams {
  CUcontext ctx = nullptr;
  CUstream h2d = nullptr, d2h = nullptr;
  std::vector<void*> ev;   // reusable (a wait captures the event's state when it is enqueued)
};
std::mutex g_cs_mu;
std::vector<CopyStreams> g_cs;

void* pool_event(CopyStreams& cs, size_t i) {
  Cuda& c = cuda();
  while (cs.ev.size() <= i) {
    void* e = nullptr;
    check(c.ev_create(&e, 2 /* CU_EVENT_DISABLE_TIMING */), "cuEventCreate");
    cs.ev.push_back(e);
  }
  return cs.ev[i];
}

int64_t copy_bytes(const Plan& p, void* const* host_ptrs, bool inputs) {
  int64_t b = 0;
  for (int t = 0; t < p.desc.ntensors; t++) {
    int r = p.desc.t[t].role;
    bool sel = inputs ? (r == FOP_IN || r == FOP_INOUT) : (r == FOP_OUT || r == FOP_INOUT);
    if (sel && host_ptrs[t]) b += span_bytes(p.desc.t[t]);
  }
  return b;
}

void copy_tensors(const Plan& p, void* const* ptrs, void* const* host_ptrs, CUstream st, bool inputs) {
  Cuda& c = cuda();
  const fop_desc& d = p.desc;
  for (int t = 0; t < d.ntensors; t++) {
    bool in = d.t[t].role == FOP_IN || d.t[t].role == FOP_INOUT;
    bool out = d.t[t].role == FOP_OUT || d.t[t].role == FOP_INOUT;
    if (!host_ptrs[t] || span_bytes(d.t[t]) == 0 || (inputs ? !in : !out)) continue;
    if (inputs) check(c.h2d((CUdeviceptr)ptrs[t], host_ptrs[t], (size_t)span_bytes(d.t[t]), st), "cuMemcpyHtoDAsync");
    else check(c.d2h(host_ptrs[t], (CUdeviceptr)ptrs[t], (size_t)span_bytes(d.t[t]), st), "cuMemcpyDtoHAsync");
  }
}
}  // namespace

fop_status run_host_many(Plan* const* plans, void* const* const* host_ptrs, void* const* const* dev_ptrs,
                         const int32_t* nptrs, void* const* ws, int n, void* stream) {
  Cuda& c = cuda();
  if (!c.ok) fail(FOP_E_CUDA, c.why);
  if (n <= 0) return FOP_OK;
  for (int k = 0; k < n; k++)
    if (!plans[k] || !host_ptrs[k] || !dev_ptrs[k]) fail(FOP_E_INVALID, "NULL plan or pointer table at " + std::to_string(k));
  CUcontext ctx = current_context(dev_ptrs[0], nptrs[0]);
  CUstream st = (CUstream)stream;
  std::lock_guard<std::mutex> g(g_cs_mu);
  CopyStreams* cs = nullptr;
  for (auto& x : g_cs)
    if (x.ctx == ctx) cs = &x;
  if (!cs) {
    CopyStreams x;
    x.ctx = ctx;
    check(c.stream_create(&x.h2d, 1 /* CU_STREAM_NON_BLOCKING */), "cuStreamCreate");
    check(c.stream_create(&x.d2h, 1), "cuStreamCreate");
    g_cs.push_back(x);
    cs = &g_cs.back();
  }
  // Order: the plans are independent and the two copy directions are a
  // two-machine flow shop, so Johnson's rule gives the shortest makespan:
  // plans with fewer input than output bytes first (by input bytes,
  // ascending), then the rest (by output bytes, descending); ties keep the
  // caller's order.
  std::vector<int> ord(n);
  std::vector<int64_t> hin(n), hout(n);
  for (int k = 0; k < n; k++) {
    ord[k] = k;
    hin[k] = copy_bytes(*plans[k], host_ptrs[k], true);
    hout[k] = copy_bytes(*plans[k], host_ptrs[k], false);
  }
  std::stable_sort(ord.begin(), ord.end(), [&](int a, int b) {
    bool fa = hin[a] < hout[a], fb = hin[b] < hout[b];
    if (fa != fb) return fa;
    return fa ? hin[a] < hin[b] : hout[a] > hout[b];
  });
  size_t ei = 0;
  void* e0 = pool_event(*cs, ei++);
  check(c.ev_record(e0, st), "cuEventRecord");
  check(c.stream_wait(cs->h2d, e0, 0), "cuStreamWaitEvent");
  check(c.stream_wait(cs->d2h, e0, 0), "cuStreamWaitEvent");
  for (int k : ord) {
    copy_tensors(*plans[k], dev_ptrs[k], host_ptrs[k], cs->h2d, true);
    void* ein = pool_event(*cs, ei++);
    check(c.ev_record(ein, cs->h2d), "cuEventRecord");
    check(c.stream_wait(st, ein, 0), "cuStreamWaitEvent");
    run_plan(*plans[k], dev_ptrs[k], nptrs[k], ws ? ws[k] : nullptr, stream, nullptr);
    void* ek = pool_event(*cs, ei++);
    check(c.ev_record(ek, st), "cuEventRecord");
    check(c.stream_wait(cs->d2h, ek, 0), "cuStreamWaitEvent");
    copy_tensors(*plans[k], dev_ptrs[k], host_ptrs[k], cs->d2h, false);
  }
  void* eout = pool_event(*cs, ei++);
  check(c.ev_record(eout, cs->d2h), "cuEventRecord");
  check(c.stream_wait(st, eout, 0), "cuStreamWaitEvent");
  return FOP_OK;
}

}  // namespace fop
