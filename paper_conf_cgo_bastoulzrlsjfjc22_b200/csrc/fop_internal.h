// fop_internal.h — host-side data structures of libfop (planner, codegen, runtime).
//
// Pipeline:  a1 validate  -> a2 analyse strides  ->
// a3 Algorithm 2 scenarios  -> a4 widths  -> a5 groups/classes/launches
// (+ a7 fusion)  -> codegen  -> NVRTC (sm_100a)  -> fop_run launches.
#pragma once

#include <cstdint>
#include <mutex>
#include <string>
#include <unordered_map>
#include <vector>

#include "../../include/fop.h"

namespace fop {

// ---------------------------------------------------------------- errors
void set_error(const std::string& msg);
struct Error {
  fop_status status;
  std::string msg;
};
[[noreturn]] void fail(fop_status s, const std::string& msg);

inline int esize(int dtype) { return (dtype == FOP_F16 || dtype == FOP_BF16) ? 2 : 4; }

// ---------------------------------------------------------------- a2
// An access as an affine function of the loop iterators (element units):
//   offset = base + sum_l coef[l] * i_l          (P:355 access functions)
struct Affine {
  int tensor = -1;
  int64_t base = 0;
  int64_t coef[FOP_MAX_LOOPS] = {0};
  bool same(const Affine& o) const {
    if (tensor != o.tensor || base != o.base) return false;
    for (int l = 0; l < FOP_MAX_LOOPS; l++)
      if (coef[l] != o.coef[l]) return false;
    return true;
  }
};

Affine affine_of(const fop_desc& d, const fop_access& a);

// ---------------------------------------------------------------- a3
struct Scenarios {
  int nscen = 0;
  int len[FOP_MAX_SCEN] = {0};
  int loops[FOP_MAX_SCEN][3] = {{0}};          // outermost -> innermost
  double inner_score[FOP_MAX_LOOPS] = {0};     // by statement loop position
};
Scenarios rank_scenarios(const fop_desc& d, int s, const fop_plan_opts& o);

// ---------------------------------------------------------------- N3
// A dependence of a statement on itself (validity): a distance
// vector over global loop ids, lexicographically positive in the statement's
// original loop order.  Statements here have uniform dependences only: a
// read of the target at a constant offset from the write (a recurrence), or
// the write-write pairs of a read-modify-write over the loops the target
// ignores (Fig. 2's Y over k).
struct Dep {
  int64_t dist[FOP_MAX_LOOPS] = {0};
  bool anti = false;   // the read happens before the write (else flow / output)
};
std::vector<Dep> self_dependences(const fop_desc& d, int s);
// Permutation-only legality of the schedule "parallel loops (threads) /
// seq loops in the given order (each thread) / vector loop" for deps.
bool schedule_legal(const std::vector<Dep>& deps, const std::vector<int>& seq, int vec_loop, int nloops,
                    const int* loops);

// ---------------------------------------------------------------- a5/a7
enum XOp {  // expanded DAG node kinds (fop_opcode values + internal ones)
  X_FWD = 100,     // value of an earlier ASSIGN statement of the same launch (registers)
  X_SCALAR = 101,  // value of an earlier REDUCE statement of the same launch (per row)
  X_SELF = 102     // read-modify-write: the running value of the statement's own target
};

struct XNode {
  int op = 0;       // fop_opcode or XOp
  int a = -1, b = -1;
  int cvt = 0;
  float imm = 0.f;
  int acc = -1;     // FOP_OP_LOAD: index into Launch::loads
  int src = -1;     // X_FWD / X_SCALAR: index into Launch::stmts
  mutable bool no_addsub = false;   // codegen: the value reaches the output without an add/sub
};

struct XStmt {
  int stmt = -1;            // descriptor statement index
  int kind = FOP_ASSIGN;
  int redop = FOP_RED_SUM;
  std::vector<XNode> nodes; // expanded DAG (inlined producers substituted)
  std::vector<XNode> fin;   // REDUCE finalize
  int result = -1;          // index of the statement value in nodes
  Affine write;
  int out_dtype = FOP_F32;
  bool store = true;        // result written to memory
  bool fwd = false;         // consumed later in the same launch
  bool move = false;        // pure element move (raw bits)
};

// a kernel loop: adjacent launch loops collapsed into one (loops
// contiguous for ALL accesses are merged); coefficient = that of members[0]
struct KLoop {
  std::vector<int> members;   // loop ids, innermost first
  int64_t extent = 1;
};

struct Launch {
  int kclass = FOP_CLASS_EW;
  int main_stmt = -1;
  uint32_t mask = 0;
  std::vector<XStmt> stmts;
  std::vector<Affine> loads;      // distinct load accesses (after inlining)
  std::vector<int> loops;         // loop ids the launch iterates (main statement loops)
  int vec_loop = -1;              // d_v
  int width = 1;                  // W (elements along d_v)
  int read_loop = -1, read_width = 0;  // TRANSPOSE
  int trans_load = -1;            // TRANSPOSE: index into loads of the transposed access
  int tr_smem = 0;                // TRANSPOSE staged through shared memory: 1 = d_r rows cannot carry vectors (flat
                                  // input tile), 2 = d_v rows cannot (flat output tile)
  int64_t tr_tv = 0;              // tr_smem 1: d_v rows per tile (tile = tr_tv x E[d_r]); 2: d_r rows per tile
  int coal_loop = -1;
  std::vector<int> order;         // launch loop order, innermost first (before collapse)
  std::vector<int> seq;           // EW read-modify-write / recurrence: loops walked in order by each thread (outer first)
  bool rec = false;               // recurrence: the target depends on every seq loop (stored every iteration)
  int seq_prefetch = 1;           // sequential launches: iterations of target-independent loads kept in flight
  bool force_w1 = false;          // no influence scenario feasible: no explicit vector type (width 1)
  std::vector<int> fwd_dist;      // recurrence: per load, iterations back along the last seq loop (0 = memory)
  bool virt_vec = false;          // no dependence-free loop: vec_loop is a placeholder of extent 1
  int scen_pick = 0;              // N3: scenario whose innermost loop carries the vector type (-1: none feasible)
  int fallback = 0;               // N3: 0 scenario as ranked, 1 looser (vector constraint only), 2 no influence, 3 fully sequential
  std::vector<std::pair<std::string, int>> knobs;   // geometry overrides of this variant (auto-tuning)
  std::string name_suffix;        // kernel name suffix of a tuning variant
  std::vector<KLoop> kl;          // kernel loops (see geometry.cpp for the per-class layout)
  int nsplit = 0;                 // ROW: #reduction kloops; COL: #parallel kloops; TR: 2
  std::vector<int> load_cb;       // per load: vector chunk bytes (0 = not contiguous along d_v)
  std::vector<int> load_cb_r;     // TRANSPOSE: per load chunk bytes along d_r
  std::vector<int> store_cb;      // per stmt: vector chunk bytes of the store (0 = scalar)
  int unroll = 1;
  int minblocks = 1;              // __launch_bounds__ min blocks/SM; grid-stride grids = SMs x minblocks
  int row_prefetch = 0;           // ROW: prefetch the next row's streaming loads
  int col_pipe = 0;               // COL: software-pipelined row batches
  int col_il = 1;                 // COL: chunks interleave over rows (grid sweeps rows together)
  int col_fin = 0;                // COL finalize: 0 fence + counter (default); 1/2 flag words (ablations)
  int row_hoist = 1;              // ROW: keep row-invariant loads in registers across rows
  int row_g = 1;                  // ROW: warps per row (> 1 for few long rows)
  int row_q = 1;                  // ROW: CTAs per row (a thread-block cluster) for few long rows
  int row_p = 1;                  // ROW: rows per warp (> 1 for rows of fewer than 16 vectors)
  int row_peel = 0;               // ROW: rows whose length/pitch admit no static vector: per-row shift to the
                                  // first aligned element, W-vectors in between, head + tail elements scalar
  int row_split = 0;              // ROW: > 0 = lanes also split the outer reduction iterations (S lane
                                  // subgroups of pow2(#vectors) lanes each), for rows of few vectors
                                  // under long outer reduction loops (e.g. BN statistics on NCHW)
  // TRANSPOSE through TMA (16-bit data): 64x64 tiles, tensor maps encoded per run
  int tma = 0;
  int tma_rank = 0, tma_stages = 4;
  int tma_in_tensor = -1, tma_out_tensor = -1;
  int64_t tma_in_base = 0, tma_out_base = 0;     // access base offsets (elements)
  uint64_t tma_in_dim[5] = {0}, tma_in_stride[5] = {0};    // strides in bytes of dims 1..rank-1
  uint64_t tma_out_dim[5] = {0}, tma_out_stride[5] = {0};
  int64_t tma_tiles = 0, tma_ntv = 0, tma_ntr = 0;
  // per-run tensor maps (runtime; cached for the last pointer pair, guarded by Plan::mu)
  struct alignas(64) TmaMap { uint64_t w[16]; };
  TmaMap tma_map_in, tma_map_out;
  const void* tma_last_in = nullptr;
  const void* tma_last_out = nullptr;
  int gv = 1, gr = 1;             // lanes along d_v / along the other tiled dim
  int64_t nchunks = 1;            // COL: row chunks
  int64_t work = 0;               // total work items (threads' units)
  // codegen / runtime
  std::string name, src;
  std::vector<char> cubin;
  int64_t grid = 1;
  int block = 256;
  size_t smem = 0;
  size_t ws_off = 0, ws_bytes = 0;  // COL_REDUCE partials + counters
  std::vector<int> align;         // per tensor: byte alignment the vector variant assumes
  bool scalar_variant = false;    // this launch is the narrow (W=1) variant
  int col_acqrel = 0;             // COL finalize: one acq_rel arrival atomic instead of membar.gl + relaxed atomic
  int col_fold = 0;               // COL: dense odd rows read as [R/P, P*E] (P rows per aligned group), folded at the end
  size_t fold_off = 0;            // COL fold: wide-column sums + counter, offset inside the launch's workspace
  int col_shift = 0;              // COL: full-width vectors over odd rows via per-row funnel shifts of aligned chunks
  int tr_om = 0;                  // TRANSPOSE smem (tr_smem 2): output-major tile (lane-contiguous scatter, vector read-out)
  int64_t period = 0;             // EW: kl[0] is (d_v x next loop) flattened; period accesses use c = flat % period
  std::vector<char> period_load;  // per load: read per element at c = flat index mod period (bias[c] over odd c)
  // multi-GPU (opts.peer_world >= 1): COL_REDUCE partials combined across the
  // peer group in the kernel's epilogue (fop.h, peer groups)
  bool peer = false;
  size_t peer_off = 0;            // this launch's region in the exchange buffer
  int64_t peer_slabs = 0;         // slabs (= exchange units) of the launch
};

// Exchange-buffer region of a peer-exchanging COL_REDUCE launch (fop.h, peer
// groups): [2 parities][world][slabs][SW] u64 words (fp32 sum | epoch << 32)
// | [slabs] u32 local run counters.  Offsets relative to Launch::peer_off.
struct PeerLayout {
  size_t data = 0, epoch = 0, total = 0;
};
inline PeerLayout peer_layout(const Launch& L, int world) {
  auto al = [](size_t x) { return (x + 255) & ~size_t(255); };
  PeerLayout r;
  const size_t sw = (size_t)L.gv * (size_t)L.width;
  r.data = 0;
  r.epoch = al(2 * (size_t)world * (size_t)L.peer_slabs * sw * sizeof(uint64_t));
  r.total = r.epoch + al((size_t)L.peer_slabs * sizeof(unsigned));
  return r;
}

struct Plan {
  fop_desc desc;
  fop_plan_opts opts;
  Scenarios scen[FOP_MAX_STMTS];
  std::vector<Dep> deps[FOP_MAX_STMTS];
  std::vector<Launch> launches;
  std::vector<int64_t> temp_off;  // per tensor: workspace byte offset (-1 = not materialised)
  size_t ws_bytes = 0;
  size_t peer_bytes = 0;          // exchange buffer (fop_plan_peer_bytes); 0 = no peer exchange
  // lazily built narrow variants (misaligned pointers), guarded by mu
  std::mutex mu;
  std::vector<Launch> narrow;     // same indexing as launches (empty src = not built)
  // auto-tuning candidates per launch (entry 0 = the launch itself is implicit)
  std::vector<std::vector<Launch>> variants;
  bool tunable = false;           // re-running the plan is idempotent (no in-place statements)
  struct Loaded {
    void* ctx;
    std::vector<void*> mods, fns, nmods, nfns;
    std::vector<std::vector<void*>> vfns;   // per launch: functions of variants[i]
    void* flush_fn = nullptr;               // auto-tuner's L2 flush / dirty kernels (runtime.cpp)
    void* dirty_fn = nullptr;
    std::vector<int> choice;                // per launch: -1 untuned, 0 = default, k = variants[i][k-1]
  };
  std::vector<Loaded> loaded;
};

// validate.cpp
void validate(const fop_desc& d);
bool empty_domain(const fop_desc& d, const fop_stmt& st);   // some loop of the statement has extent 0
// planner.cpp
void plan_launches(Plan& p);
void finalize_launch_geometry(const Plan& p, Launch& L);
int geometry_knob(const Launch& L, const char* name, int dflt);
std::vector<std::vector<std::pair<std::string, int>>> tuning_variants(const Launch& L, int sms);
// codegen.cpp
std::string generate(const Plan& p, Launch& L, int launch_index);
extern const char* kDeviceHeader;   // device/fop_device.cuh, embedded at build time
// jit.cpp
void jit_compile(Launch& L);
bool jit_available();
// runtime.cpp
fop_status run_host_many(Plan* const* plans, void* const* const* host_ptrs, void* const* const* dev_ptrs,
                         const int32_t* nptrs, void* const* ws, int n, void* stream);
fop_status run_plan(Plan& p, void* const* ptrs, int nptrs, void* ws, void* stream,
                    void* const* host_ptrs, const fop_peer_group* peers = nullptr, bool pdl = false);
void peer_alloc(size_t bytes, void** dev_ptr, fop_ipc_handle* handle);
void peer_free(void* dev_ptr);
void peer_open(const fop_ipc_handle* handle, void** dev_ptr);
void peer_close(void* dev_ptr);
void* current_context_or_null();   // the calling thread's CUDA context (nullptr without a driver)

}  // namespace fop
