// abi.cpp — the extern "C" entry points declared in include/fop.h.
// Every entry point converts internal failures into a fop_status plus a
// thread-local message; nothing throws or aborts across the ABI.
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <exception>
#include <new>
#include <string>

#include "fop_internal.h"

struct fop_plan {
  fop::Plan p;
};

namespace fop {
static thread_local std::string g_err;
void set_error(const std::string& msg) { g_err = msg; }
void fail(fop_status s, const std::string& msg) { throw Error{s, msg}; }
}  // namespace fop

template <class F>
static fop_status guarded(F&& f) {
  try {
    return f();
  } catch (const fop::Error& e) {
    fop::set_error(e.msg);
    return e.status;
  } catch (const std::bad_alloc&) {
    fop::set_error("out of host memory");
    return FOP_E_NOMEM;
  } catch (const std::exception& e) {
    fop::set_error(e.what());
    return FOP_E_INVALID;
  } catch (...) {
    fop::set_error("unknown internal error");
    return FOP_E_INVALID;
  }
}

extern "C" {

int fop_abi_version(void) { return FOP_ABI_VERSION; }

void fop_plan_opts_default(fop_plan_opts* o) {
  if (!o) return;
  std::memset(o, 0, sizeof *o);
  o->w[0] = 5;  // w1: store vectorisation
  o->w[1] = 3;  // w2: load vectorisation
  o->w[2] = 1;  // w3: 1/M, short jumps
  o->w[3] = 1;  // w4: |C|, many stride-1 accesses
  o->w[4] = 1;  // w5: thread term
  o->thread_limit = 1024;  // R5
  o->max_scenarios = 8;
  o->max_vec_bytes = 16;   // 128-bit vector types
  o->readings = FOP_READING_R1_THREAD_TERM | FOP_READING_R6_STRIDE1_C;
  o->force_width = 0;
  o->coalesce_order = FOP_ORDER_MEMORY;  // measured faster on B200; PAPER kept as ablation
  o->sm_count = 148;
  o->jit = 1;
  o->autotune = 1;
  o->variant = -1;
}

fop_status fop_plan(const fop_desc* desc, const fop_plan_opts* opts, fop_plan_t** out) {
  if (out) *out = nullptr;
  return guarded([&] {
    if (!desc || !out) fop::fail(FOP_E_INVALID, "NULL descriptor or output pointer");
    auto* h = new struct fop_plan();
    try {
      fop::Plan& p = h->p;
      std::memcpy(&p.desc, desc, sizeof *desc);
      if (opts) std::memcpy(&p.opts, opts, sizeof *opts);
      else fop_plan_opts_default(&p.opts);
      if (p.opts.thread_limit <= 0) fop::fail(FOP_E_INVALID, "thread_limit must be > 0");
      if (p.opts.max_vec_bytes != 4 && p.opts.max_vec_bytes != 8 && p.opts.max_vec_bytes != 16 &&
          p.opts.max_vec_bytes != 32)
        fop::fail(FOP_E_INVALID, "max_vec_bytes must be 4, 8, 16 or 32");
      if (p.opts.peer_world < 0 || p.opts.peer_timeout_ms < 0) fop::fail(FOP_E_INVALID, "negative peer option");
      if (p.opts.variant < -1) fop::fail(FOP_E_INVALID, "variant must be -1 (auto-tune) or >= 0");
      fop::validate(p.desc);
      fop::plan_launches(p);
      // narrow (scalar) variants for misaligned base pointers: geometry now,
      // compiled on first use; workspace sized for the larger of the two
      p.narrow.clear();
      for (size_t i = 0; i < p.launches.size(); i++) {
        fop::Launch N = p.launches[i];
        N.scalar_variant = true;
        N.cubin.clear();
        N.src.clear();
        fop::finalize_launch_geometry(p, N);
        // a region of its own: kernels of another geometry place partial sums
        // and arrival counters at other offsets, so sharing a region would
        // let one variant's partials overwrite another's counters
        if (N.ws_bytes) {
          N.ws_off = (p.ws_bytes + 255) & ~size_t(255);
          p.ws_bytes = N.ws_off + N.ws_bytes;
        }
        p.narrow.push_back(N);
      }
      for (size_t i = 0; i < p.launches.size(); i++) {
        fop::generate(p, p.launches[i], (int)i);
        if (p.opts.jit) fop::jit_compile(p.launches[i]);
      }
      // auto-tuning candidates (fop.h: opts.autotune), only for idempotent plans
      p.tunable = true;
      for (size_t i = 0; i < p.launches.size(); i++) {
        const fop::Launch& L = p.launches[i];
        if (!L.seq.empty()) p.tunable = false;
        for (const auto& x : L.stmts) {
          if (p.desc.t[x.write.tensor].role == FOP_INOUT) p.tunable = false;
          for (size_t j = 0; j <= i; j++)
            for (const auto& a : p.launches[j].loads)
              if (a.tensor == x.write.tensor) p.tunable = false;
        }
      }
      p.variants.assign(p.launches.size(), {});
      if ((p.opts.autotune || p.opts.variant > 0) && p.opts.jit && p.tunable) {
        for (size_t i = 0; i < p.launches.size(); i++) {
          if (p.launches[i].peer) continue;   // every rank must run the same geometry (fop_run_peer)
          auto vs = fop::tuning_variants(p.launches[i], p.opts.sm_count > 0 ? p.opts.sm_count : 148);
          std::vector<std::string> seen = {p.launches[i].src};
          for (size_t k = 1; k < vs.size(); k++) {
            fop::Launch V = p.launches[i];
            V.knobs = vs[k];
            V.cubin.clear();
            V.src.clear();
            V.name_suffix = "_v" + std::to_string(k);
            fop::finalize_launch_geometry(p, V);
            V.ws_off = p.launches[i].ws_off;   // provisional: the duplicate check compares sources
            fop::generate(p, V, (int)i);
            // identical geometry up to the name: nothing to tune
            std::string body = V.src;
            for (size_t q = body.find(V.name_suffix); q != std::string::npos; q = body.find(V.name_suffix))
              body.erase(q, V.name_suffix.size());
            if (std::find(seen.begin(), seen.end(), body) != seen.end()) continue;
            seen.push_back(body);
            if (V.ws_bytes) {   // a region of its own (see the narrow variants above)
              V.ws_off = (p.ws_bytes + 255) & ~size_t(255);
              p.ws_bytes = V.ws_off + V.ws_bytes;
              V.src.clear();
              fop::generate(p, V, (int)i);
            }
            fop::jit_compile(V);
            p.variants[i].push_back(V);
          }
        }
      }
    } catch (...) {
      delete h;
      throw;
    }
    *out = h;
    return FOP_OK;
  });
}

fop_status fop_plan_info_get(const fop_plan_t* plan, fop_plan_info* o) {
  return guarded([&] {
    if (!plan || !o) fop::fail(FOP_E_INVALID, "NULL argument");
    const fop::Plan& p = plan->p;
    std::memset(o, 0, sizeof *o);
    o->nstmts = p.desc.nstmts;
    for (int s = 0; s < p.desc.nstmts; s++) {
      const fop::Scenarios& sc = p.scen[s];
      o->nscen[s] = sc.nscen;
      for (int k = 0; k < sc.nscen; k++) {
        o->scen_len[s][k] = sc.len[k];
        for (int q = 0; q < 3; q++) o->scenario[s][k][q] = q < sc.len[k] ? sc.loops[k][q] : -1;
      }
      for (int k = 0; k < p.desc.s[s].nloops; k++) o->inner_score[s][k] = sc.inner_score[k];
    }
    o->nlaunch = (int)p.launches.size();
    for (size_t i = 0; i < p.launches.size() && i < FOP_MAX_LAUNCH; i++) {
      const fop::Launch& L = p.launches[i];
      fop_launch_info& li = o->launch[i];
      li.kernel_class = L.kclass;
      li.main_stmt = L.main_stmt;
      li.stmt_mask = L.mask;
      li.vec_loop = L.virt_vec ? -1 : L.vec_loop;
      li.width = L.width;
      li.read_loop = L.read_loop;
      li.read_width = L.read_width;
      li.coal_loop = L.coal_loop;
      li.grid = L.grid;
      li.block = L.block;
      li.nseq = (int32_t)L.seq.size();
      for (size_t q = 0; q < L.seq.size() && q < FOP_MAX_LOOPS; q++) li.seq[q] = L.seq[q];
      li.scen_pick = L.scen_pick;
      li.fallback = L.fallback;
      li.peer_exchange = L.peer ? 1 : 0;
      li.nvariants = 1 + (i < p.variants.size() ? (int32_t)p.variants[i].size() : 0);
    }
    o->workspace_bytes = p.ws_bytes;
    for (int s = 0; s < p.desc.nstmts; s++) {
      o->ndeps[s] = (int32_t)std::min<size_t>(p.deps[s].size(), FOP_MAX_DEPS);
      for (int k = 0; k < o->ndeps[s]; k++) {
        for (int l = 0; l < FOP_MAX_LOOPS; l++) o->dep[s][k][l] = p.deps[s][k].dist[l];
        o->dep_anti[s][k] = p.deps[s][k].anti;
      }
    }
    return FOP_OK;
  });
}

size_t fop_plan_workspace_bytes(const fop_plan_t* plan) { return plan ? plan->p.ws_bytes : 0; }

fop_status fop_plan_source(const fop_plan_t* plan, int32_t i, const char** src) {
  return guarded([&] {
    const int n = plan ? (int)plan->p.launches.size() : 0;
    if (!plan || !src || i < -n || i >= n) fop::fail(FOP_E_INVALID, "bad launch index");
    if (i >= 0) {
      *src = plan->p.launches[i].src.c_str();
      return FOP_OK;
    }
    // -1 - k: the narrow (misaligned-pointer) variant of launch k, generated here if
    // no run has needed it yet (its kernel is compiled at first use)
    fop::Plan& p = const_cast<fop::Plan&>(plan->p);
    std::lock_guard<std::mutex> g(p.mu);
    fop::Launch& N = p.narrow[-1 - i];
    if (N.src.empty()) fop::generate(p, N, -1 - i);
    *src = N.src.c_str();
    return FOP_OK;
  });
}

fop_status fop_plan_cubin(const fop_plan_t* plan, int32_t i, const void** data, size_t* size) {
  return guarded([&] {
    if (!plan || !data || !size || i < 0 || i >= (int)plan->p.launches.size())
      fop::fail(FOP_E_INVALID, "bad launch index");
    *data = plan->p.launches[i].cubin.data();
    *size = plan->p.launches[i].cubin.size();
    return FOP_OK;
  });
}

fop_status fop_run(const fop_plan_t* plan, void* const* dev_ptrs, int32_t nptrs, void* workspace, void* stream) {
  return guarded([&] {
    if (!plan || !dev_ptrs) fop::fail(FOP_E_INVALID, "NULL plan or pointer table");
    return fop::run_plan(const_cast<fop_plan_t*>(plan)->p, dev_ptrs, nptrs, workspace, stream, nullptr);
  });
}

fop_status fop_run_host(const fop_plan_t* plan, void* const* host_ptrs, void* const* dev_ptrs, int32_t nptrs,
                        void* workspace, void* stream) {
  return guarded([&] {
    if (!plan || !dev_ptrs || !host_ptrs) fop::fail(FOP_E_INVALID, "NULL plan or pointer table");
    return fop::run_plan(const_cast<fop_plan_t*>(plan)->p, dev_ptrs, nptrs, workspace, stream, host_ptrs);
  });
}

fop_status fop_run_host_many(const fop_plan_t* const* plans, void* const* const* host_ptrs,
                             void* const* const* dev_ptrs, const int32_t* nptrs, void* const* workspaces,
                             int32_t n, void* stream) {
  return guarded([&] {
    if (n > 0 && (!plans || !host_ptrs || !dev_ptrs || !nptrs)) fop::fail(FOP_E_INVALID, "NULL argument");
    std::vector<fop::Plan*> ps((size_t)std::max(0, n));
    for (int k = 0; k < n; k++) {
      if (!plans[k]) fop::fail(FOP_E_INVALID, "NULL plan at " + std::to_string(k));
      ps[k] = &const_cast<fop_plan_t*>(plans[k])->p;
    }
    return fop::run_host_many(ps.data(), host_ptrs, dev_ptrs, nptrs, workspaces, n, stream);
  });
}

fop_status fop_run_many(const fop_plan_t* const* plans, void* const* const* dev_ptrs, const int32_t* nptrs,
                        void* const* workspaces, int32_t n, void* stream) {
  return guarded([&] {
    if (n > 0 && (!plans || !dev_ptrs || !nptrs)) fop::fail(FOP_E_INVALID, "NULL argument");
    for (int k = 0; k < n; k++) {
      if (!plans[k] || !dev_ptrs[k]) fop::fail(FOP_E_INVALID, "NULL plan or pointer table at " + std::to_string(k));
      if (plans[k]->p.peer_bytes) fop::fail(FOP_E_INVALID, "plan " + std::to_string(k) + " has a peer exchange: use fop_run_peer");
    }
    const char* pe = std::getenv("FOP_RUN_MANY_PDL");   // 0: plain launches (ablation)
    const bool no_pdl = pe && *pe == '0';
    bool first = true;   // the chain's first kernel waits for prior stream work as usual
    for (int k = 0; k < n; k++) {
      if (no_pdl) first = true;
      fop::Plan& p = const_cast<fop_plan_t*>(plans[k])->p;
      fop::run_plan(p, dev_ptrs[k], nptrs[k], workspaces ? workspaces[k] : nullptr, stream, nullptr, nullptr, !first);
      if (!p.launches.empty()) first = false;
    }
    return FOP_OK;
  });
}

size_t fop_plan_peer_bytes(const fop_plan_t* plan) { return plan ? plan->p.peer_bytes : 0; }

fop_status fop_run_peer(const fop_plan_t* plan, void* const* dev_ptrs, int32_t nptrs, void* workspace,
                        const fop_peer_group* group, void* stream) {
  return guarded([&] {
    if (!plan || !dev_ptrs) fop::fail(FOP_E_INVALID, "NULL plan or pointer table");
    return fop::run_plan(const_cast<fop_plan_t*>(plan)->p, dev_ptrs, nptrs, workspace, stream, nullptr, group);
  });
}

fop_status fop_peer_alloc(size_t bytes, void** dev_ptr, fop_ipc_handle* handle) {
  return guarded([&] {
    fop::peer_alloc(bytes, dev_ptr, handle);
    return FOP_OK;
  });
}
fop_status fop_peer_free(void* dev_ptr) {
  return guarded([&] {
    fop::peer_free(dev_ptr);
    return FOP_OK;
  });
}
fop_status fop_peer_open(const fop_ipc_handle* handle, void** dev_ptr) {
  return guarded([&] {
    fop::peer_open(handle, dev_ptr);
    return FOP_OK;
  });
}
fop_status fop_peer_close(void* dev_ptr) {
  return guarded([&] {
    fop::peer_close(dev_ptr);
    return FOP_OK;
  });
}

fop_status fop_plan_selected(const fop_plan_t* plan, int32_t i, const char** name, int64_t* grid, int32_t* block) {
  return guarded([&] {
    if (!plan || !name || i < 0 || i >= (int)plan->p.launches.size()) fop::fail(FOP_E_INVALID, "bad launch index");
    fop::Plan& p = const_cast<fop_plan_t*>(plan)->p;
    std::lock_guard<std::mutex> g(p.mu);
    const fop::Launch* L = &p.launches[i];
    void* ctx = fop::current_context_or_null();
    for (const auto& l : p.loaded)
      if (l.ctx == ctx && l.choice[i] > 0) L = &p.variants[i][l.choice[i] - 1];
    *name = L->name.c_str();
    if (grid) *grid = L->grid;
    if (block) *block = L->block;
    return FOP_OK;
  });
}

void fop_plan_destroy(fop_plan_t* plan) { delete plan; }

const char* fop_status_str(fop_status s) {
  switch (s) {
    case FOP_OK: return "FOP_OK";
    case FOP_E_INVALID: return "FOP_E_INVALID";
    case FOP_E_UNSUPPORTED: return "FOP_E_UNSUPPORTED";
    case FOP_E_ALIGN: return "FOP_E_ALIGN";
    case FOP_E_CUDA: return "FOP_E_CUDA";
    case FOP_E_NOMEM: return "FOP_E_NOMEM";
    case FOP_E_JIT: return "FOP_E_JIT";
  }
  return "FOP_E_UNKNOWN";
}

const char* fop_last_error(void) { return fop::g_err.c_str(); }

}  // extern "C"
