// codegen.cpp — instantiates one of the four hand-written kernel skeletons
// (EW, TRANSPOSE, ROW_REDUCE, COL_REDUCE) for a launch of the plan.
//
// The planner has fixed everything a compiler would: the vector loop and
// width (a3/a4), the thread order and collapsed loops (a5), the fused DAG
// with inlined producers and forwarded values (a7).  The generated kernel
// bakes all of it in as compile-time constants — extents, strides, widths,
// grid — so the index arithmetic folds to shifts/multiply-highs and the
// vector accesses are single LDG/STG.128/.256 instructions.  This is the
// B200 counterpart of AKG's mapping pass + backend vectorisation pass
// (PAPER.md P:357): the vectorised loop is never mapped to threads, and its
// loads/stores use explicit vector types.
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <sstream>
#include <string>

#include "fop_internal.h"

namespace fop {

namespace {

const char* dtn(int dt) {
  switch (dt) {
    case FOP_F16: return "fop::F16";
    case FOP_BF16: return "fop::BF16";
    case FOP_I32: return "fop::I32";
    default: return "fop::F32";
  }
}

std::string fimm(float f) {
  unsigned u;
  std::memcpy(&u, &f, 4);
  char b[64];
  std::snprintf(b, sizeof b, "__uint_as_float(0x%08xu)", u);
  return b;
}

std::string num(int64_t v) { return std::to_string(v); }

struct Out {
  std::ostringstream s;
  int ind = 0;
  void l(const std::string& x) {
    for (int i = 0; i < ind; i++) s << "  ";
    s << x << "\n";
  }
};

// set per statement (see varies()): the statement's result is rounded to a
// 16-bit type, so transcendental fast forms are within one ulp
thread_local bool g_approx16 = false;
// set with it: the statement's result is fp16 (the GELU's short ftz form is
// exact enough down to fp16's subnormals; bf16/fp32 results take the wide form)
thread_local bool g_out_f16 = false;
// the statement is an integer statement (its target is i32, reading R30):
// int32 bits in the fp32 registers, integer node forms, no packed fp32x2 path
thread_local bool g_int = false;
// ... but only for nodes whose value reaches the output without an add or
// subtract on the way: a ~2^-22 relative error ahead of a cancellation is no
// longer within one 16-bit ulp (fuzz seed 21 case 294: -x2 / -1.5 + x0 + x1
// near 6.7e-5 came out 2 f16 ulps off with the x * rcp(c) form)
bool fast_ok(const XNode& n) { return g_approx16 && n.no_addsub; }

// C expression of a fused-DAG node given its operand expressions
std::string op_expr(const XNode& n, const std::string& a, const std::string& b) {
  if (g_int) {
    switch (n.op) {
      case FOP_OP_CONST: return "__int_as_float(" + std::to_string((long long)n.imm) + ")";
      case FOP_OP_ADD: return "fop::iadd(" + a + ", " + b + ")";
      case FOP_OP_SUB: return "fop::isub(" + a + ", " + b + ")";
      case FOP_OP_MUL: return "fop::imul(" + a + ", " + b + ")";
      case FOP_OP_MAX: return "fop::imax(" + a + ", " + b + ")";
      case FOP_OP_MIN: return "fop::imin(" + a + ", " + b + ")";
      case FOP_OP_NEG: return "fop::ineg(" + a + ")";
      case FOP_OP_ABS: return "fop::iabs(" + a + ")";
      case FOP_OP_RELU: return "fop::irelu(" + a + ")";
    }
    return "__int_as_float(0)";   // (validate() admits no other node in an integer statement)
  }
  if (fast_ok(n)) {
    if (n.op == FOP_OP_EXP) return std::string(g_out_f16 ? "fop::exp_fast(" : "fop::exp_fast_wide(") + a + ")";
    if (n.op == FOP_OP_SIGMOID) return std::string(g_out_f16 ? "fop::sigmoid_fast(" : "fop::sigmoid_fast_wide(") + a + ")";
  }
  switch (n.op) {
    case FOP_OP_CONST: return fimm(n.imm);
    case FOP_OP_ADD: return "__fadd_rn(" + a + ", " + b + ")";
    case FOP_OP_SUB: return "__fsub_rn(" + a + ", " + b + ")";
    case FOP_OP_MUL: return "__fmul_rn(" + a + ", " + b + ")";
    case FOP_OP_DIV: return "__fdiv_rn(" + a + ", " + b + ")";
    case FOP_OP_MAX: return "fop::op_max(" + a + ", " + b + ")";
    case FOP_OP_MIN: return "fop::op_min(" + a + ", " + b + ")";
    case FOP_OP_NEG: return "(-(" + a + "))";
    case FOP_OP_ABS: return "fabsf(" + a + ")";
    case FOP_OP_SQRT: return "__fsqrt_rn(" + a + ")";
    case FOP_OP_RELU: return "fop::op_relu(" + a + ")";
    case FOP_OP_EXP: return "expf(" + a + ")";
    case FOP_OP_LOG: return "logf(" + a + ")";
    case FOP_OP_TANH: return "tanhf(" + a + ")";
    case FOP_OP_SIGMOID: return "fop::op_sigmoid(" + a + ")";
    case FOP_OP_GELU_TANH: return std::string(g_out_f16 ? "fop::op_gelu_tanh(" : "fop::op_gelu_tanh_wide(") + a + ")";
    case FOP_OP_GELU_ERF: return "fop::op_gelu_erf(" + a + ")";
    case FOP_OP_CAST: return std::string("fop::round_to<") + dtn(n.cvt) + ">(" + a + ")";
  }
  return "0.f";
}

// Emission context for one statement at one "point" (work item).  Element
// expressions are built for an element index expression `e` (a loop variable
// in the scalar loop, 2*p / 2*p+1 in the packed loop).
struct DagCtx {
  std::function<std::string(int, const std::string&)> load;  // element expression of load k
  std::function<bool(int)> load_varies;
  std::function<std::string(int, const std::string&)> fwd;   // element expression of forwarded stmt
  std::function<std::string(int)> scalar;                    // per-row scalar of a REDUCE
  std::function<std::string(const std::string&)> self;       // read-modify-write running value
  std::string tag;                                           // name suffix
  std::string ev = "e";                                      // scalar element loop variable
};

// Decide the 16-bit fast forms of one statement (g_approx16, XNode::no_addsub).
// Called before ANY of the statement's nodes is emitted — per-CTA tables
// included — so every geometry variant of a launch makes the same choice and
// produces the same bits.
void decide_fast(const XStmt& x) {
  const char* e = std::getenv("FOP_APPROX16");
  g_approx16 = !(e && *e == '0') && x.kind == FOP_ASSIGN && esize(x.out_dtype) == 2 && x.out_dtype != FOP_I32;
  g_out_f16 = x.kind == FOP_ASSIGN && x.out_dtype == FOP_F16;
  g_int = x.out_dtype == FOP_I32;
  std::vector<bool> feeds(x.nodes.size(), false);   // value reaches an add/sub
  for (int i = (int)x.nodes.size() - 1; i >= 0; i--)
    for (size_t j = i + 1; j < x.nodes.size(); j++) {
      const XNode& q = x.nodes[j];
      if ((q.a == i || q.b == i) && (q.op == FOP_OP_ADD || q.op == FOP_OP_SUB || feeds[j])) feeds[i] = true;
    }
  for (size_t i = 0; i < x.nodes.size(); i++) x.nodes[i].no_addsub = !feeds[i];
}

std::vector<bool> varies(const XStmt& x, const DagCtx& c) {
  decide_fast(x);   // every statement emission starts here
  std::vector<bool> v(x.nodes.size(), false);
  for (size_t i = 0; i < x.nodes.size(); i++) {
    const XNode& n = x.nodes[i];
    if (n.op == FOP_OP_LOAD) v[i] = c.load_varies(n.acc);
    else if (n.op == X_FWD || n.op == X_SELF) v[i] = true;
    else if (n.op == X_SCALAR || n.op == FOP_OP_CONST) v[i] = false;
    else v[i] = (n.a >= 0 && v[n.a]) || (n.b >= 0 && v[n.b]);
  }
  return v;
}

std::string node_name(const XStmt& x, const std::vector<bool>& var, int i, const DagCtx& c) {
  return std::string(var[i] ? "v" : "c") + num(x.stmt) + "_" + num(i) + c.tag;
}

// per-statement node overrides: a non-empty entry replaces the node's whole
// cone by that expression (e.g. a shared-memory table lookup)
thread_local const std::vector<std::string>* g_over = nullptr;
bool overridden(int i) { return g_over && i < (int)g_over->size() && !(*g_over)[i].empty(); }
// an override of a varying node names its element as $E
std::string over_at(int i, const std::string& e) {
  std::string s = (*g_over)[i];
  for (size_t q = s.find("$E"); q != std::string::npos; q = s.find("$E", q + e.size())) s.replace(q, 2, "(" + e + ")");
  return s;
}

// reachable set from the result (not descending into overridden nodes)
std::vector<bool> reachable(const XStmt& x) {
  std::vector<bool> r(x.nodes.size(), false);
  if (x.result < 0) return r;
  r[x.result] = true;
  for (int i = x.result; i >= 0; i--) {
    if (!r[i] || overridden(i)) continue;
    if (x.nodes[i].a >= 0) r[x.nodes[i].a] = true;
    if (x.nodes[i].b >= 0) r[x.nodes[i].b] = true;
  }
  return r;
}

// emit nodes with var==want (scalar form); defines names
void emit_nodes(Out& o, const XStmt& x, const std::vector<bool>& var, bool want, const DagCtx& c,
                int skip = -1) {
  std::vector<bool> reach = reachable(x);
  for (size_t i = 0; i < x.nodes.size(); i++) {
    if (!reach[i] || var[i] != want || (int)i == skip) continue;
    const XNode& n = x.nodes[i];
    std::string e;
    if (overridden((int)i)) e = over_at((int)i, c.ev);
    else if (n.op == FOP_OP_LOAD) e = c.load(n.acc, c.ev);
    else if (n.op == X_FWD) e = c.fwd(n.src, c.ev);
    else if (n.op == X_SELF) e = c.self(c.ev);
    else if (n.op == X_SCALAR) e = c.scalar(n.src);
    else {
      std::string a = n.a >= 0 ? node_name(x, var, n.a, c) : "";
      std::string b = n.b >= 0 ? node_name(x, var, n.b, c) : "";
      e = op_expr(n, a, b);
    }
    o.l("const float " + node_name(x, var, (int)i, c) + " = " + e + ";");
  }
}

// packed (fp32x2) form of the varying nodes: one value = elements (2p, 2p+1)
std::string pair_name(const XStmt& x, int i, const DagCtx& c) {
  return "w" + num(x.stmt) + "_" + num(i) + c.tag;
}
void emit_nodes_packed(Out& o, const XStmt& x, const std::vector<bool>& var, const DagCtx& c, const std::string& p,
                       int skip = -1) {
  std::vector<bool> reach = reachable(x);
  const std::string e0 = "2 * " + p, e1 = "2 * " + p + " + 1";
  auto opnd = [&](int i) { return var[i] ? pair_name(x, i, c) : "fop::pk1(" + node_name(x, var, i, c) + ")"; };
  // a packed product must never be contracted into a later packed add/sub (see fop::nofuse):
  // every packed product is hidden at its source — not only where it feeds an add directly,
  // since ptxas also sees through value-preserving steps in between (max(p, p), a negation:
  // fuzz seed 51 case 289, one bf16 ulp off after (x0 - x1) * x1 -> max(p, p) + y)
  auto addend = [&](int i) { return opnd(i); };
  for (size_t i = 0; i < x.nodes.size(); i++) {
    if (!reach[i] || !var[i] || (int)i == skip) continue;
    const XNode& n = x.nodes[i];
    std::string e;
    if (overridden((int)i)) {   // a per-element table lookup
      o.l("const u64 " + pair_name(x, (int)i, c) + " = fop::pk(" + over_at((int)i, e0) + ", " + over_at((int)i, e1) + ");");
      continue;
    }
    switch (n.op) {
      case FOP_OP_LOAD: e = "fop::pk(" + c.load(n.acc, e0) + ", " + c.load(n.acc, e1) + ")"; break;
      case X_FWD: e = "fop::pk(" + c.fwd(n.src, e0) + ", " + c.fwd(n.src, e1) + ")"; break;
      case X_SELF: e = "fop::pk(" + c.self(e0) + ", " + c.self(e1) + ")"; break;
      case FOP_OP_ADD: e = "fop::add2(" + addend(n.a) + ", " + addend(n.b) + ")"; break;
      case FOP_OP_SUB: e = "fop::sub2(" + addend(n.a) + ", " + addend(n.b) + ")"; break;
      case FOP_OP_MUL: e = "fop::nofuse(fop::mul2(" + opnd(n.a) + ", " + opnd(n.b) + "), fop_zero)"; break;
      case FOP_OP_GELU_TANH:
        e = std::string(g_out_f16 ? "fop::op_gelu_tanh2(" : "fop::op_gelu_tanh2_wide(") + opnd(n.a) + ")";
        break;
      case FOP_OP_DIV:
        if (g_approx16 && !var[n.b]) {
          // ÷ loop-invariant d -> × r = RN(1/d), then one remainder step
          // (q = RN(a r); q += RN(a - q d) r, the remainder exact by FMA):
          // the quotient to within an fp32 ulp (Markstein's correction) even
          // where an add/sub follows and cancels, 1.5 packed FMAs per element
          const std::string dn = node_name(x, var, n.b, c), pa = opnd(n.a);
          e = "fop::div2_by(" + pa + ", " + dn + ")";
          break;
        }
        [[fallthrough]];
      default: {  // no packed form: per lane
        auto lane = [&](const char* f, int k) {
          return k < 0 ? std::string("") : (var[k] ? std::string("fop::") + f + "(" + pair_name(x, k, c) + ")"
                                                   : node_name(x, var, k, c));
        };
        e = "fop::pk(" + op_expr(n, lane("lo", n.a), lane("lo", n.b)) + ", " +
            op_expr(n, lane("hi", n.a), lane("hi", n.b)) + ")";
      }
    }
    o.l("const u64 " + pair_name(x, (int)i, c) + " = " + e + ";");
  }
}

// The element loop of one statement.  W even and packing on: pairs with
// FADD2/FMUL2/FFMA2; otherwise scalar.  A SUM reduction whose term ends in a
// product hands the two factors to `fma` (contracted into the accumulator,
// reading R23) instead of materialising the product.
struct Sink {
  std::function<void(const std::string&)> scalar;                          // value, element var c.ev
  std::function<void(const std::string&, const std::string&)> pair;        // packed value, pair var
  std::function<void(const std::string&, const std::string&, const std::string&)> pair_fma;  // a, b, pair var
};
thread_local bool g_packed = true;
void emit_elems(Out& o, const XStmt& x, const std::vector<bool>& var, const DagCtx& c, int W, const Sink& s) {
  bool packed = g_packed && W % 2 == 0 && s.pair && !g_int;
  if (!packed) {
    o.l("#pragma unroll");
    o.l("for (int " + c.ev + " = 0; " + c.ev + " < " + num(W) + "; ++" + c.ev + ") {");
    o.ind++;
    emit_nodes(o, x, var, true, c);
    s.scalar(node_name(x, var, x.result, c));
    o.ind--;
    o.l("}");
    return;
  }
  std::string p = c.ev + "p";
  const XNode& r = x.nodes[x.result];
  bool fma = s.pair_fma && r.op == FOP_OP_MUL && var[x.result];
  int uses = 0;
  for (auto& n : x.nodes) uses += (n.a == x.result) + (n.b == x.result);
  fma = fma && uses == 0;
  o.l("#pragma unroll");
  o.l("for (int " + p + " = 0; " + p + " < " + num(W / 2) + "; ++" + p + ") {");
  o.ind++;
  emit_nodes_packed(o, x, var, c, p, fma ? x.result : -1);
  auto opnd = [&](int i) { return var[i] ? pair_name(x, i, c) : "fop::pk1(" + node_name(x, var, i, c) + ")"; };
  if (fma) s.pair_fma(opnd(r.a), opnd(r.b), p);
  else if (var[x.result]) s.pair(pair_name(x, x.result, c), p);
  else s.pair("fop::pk1(" + node_name(x, var, x.result, c) + ")", p);
  o.ind--;
  o.l("}");
}

std::string fin_expr(Out& o, const XStmt& x, const std::string& acc, const std::string& tag) {
  if (x.fin.empty()) return acc;
  g_out_f16 = x.out_dtype == FOP_F16;   // (finalize nodes never take the fast forms: no_addsub unset)
  g_int = x.out_dtype == FOP_I32;
  for (size_t i = 0; i < x.fin.size(); i++) {
    const XNode& n = x.fin[i];
    std::string nm = "f" + num(x.stmt) + "_" + num(i) + tag;
    std::string e;
    if (n.op == FOP_OP_ACC) e = acc;
    else {
      std::string a = n.a >= 0 ? "f" + num(x.stmt) + "_" + num(n.a) + tag : "";
      std::string b = n.b >= 0 ? "f" + num(x.stmt) + "_" + num(n.b) + tag : "";
      e = op_expr(n, a, b);
    }
    o.l("const float " + nm + " = " + e + ";");
  }
  return "f" + num(x.stmt) + "_" + num(x.fin.size() - 1) + tag;
}

struct Gen {
  const Plan& p;
  Launch& L;
  const fop_desc& d;
  std::string idx;  // index type
  Out o;
  Gen(const Plan& p_, Launch& L_) : p(p_), L(L_), d(p_.desc) {}

  int64_t C(const Affine& a, int k) const { return a.coef[L.kl[k].members[0]]; }
  int es(int t) const { return esize(d.t[t].dtype); }
  bool written_here(int t) const {
    for (auto& x : L.stmts)
      if (x.write.tensor == t) return true;
    return false;
  }
  int64_t tensor_bytes(int t) const {
    int64_t n = 1;
    for (int r = 0; r < d.t[t].rank; r++) n += (d.t[t].shape[r] - 1) * d.t[t].stride[r];
    return n * es(t);
  }
  std::string pol(const Affine& a, bool broadcast) const {
    if (written_here(a.tensor) || d.t[a.tensor].role == FOP_INOUT) return "fop::LD_COHERENT";
    if (broadcast || tensor_bytes(a.tensor) <= (1 << 20)) return "fop::LD_CACHED";
    return "fop::LD_STREAM";
  }
  std::string spol() const {
    const char* e = std::getenv("FOP_STORE_POLICY");
    if (e && std::strcmp(e, "stream") == 0) return "fop::ST_STREAM";
    // ROW stores evict-first (st.global.cs, FOP_ROW_ST_STREAM=1): the row kernel
    // leaves DRAM idle (cfg4a: 2.6 TB/s under ncu), so its outputs' write-back
    // could happen inside its own window instead of the next operator's
    if (L.kclass == FOP_CLASS_ROW_REDUCE && geometry_knob(L, "FOP_ROW_ST_STREAM", 0)) return "fop::ST_STREAM";
    return "fop::ST_DEFAULT";
  }
  std::string ptr(int t, const std::string& off) const {
    return "(T" + num(t) + " + (u64)(" + off + ") * " + num(es(t)) + ")";
  }
  // base + sum_k coef_k * it_k over the given kernel loops
  std::string affine(const Affine& a, const std::vector<std::pair<int, std::string>>& its) const {
    std::string s = num(a.base);
    for (auto& kv : its) {
      int64_t c = C(a, kv.first);
      if (c == 0) continue;
      s += " + " + kv.second + (c == 1 ? "" : " * " + num(c));
    }
    return "(" + idx + ")(" + s + ")";
  }

  void header(const std::string& name, int /*unused*/) {
    const int minblocks = std::max(1, L.minblocks);
    o.l("// generated by libfop (planner + codegen); skeleton: " + name);
    if (const char* g = std::getenv("FOP_GELU_NR"); g && *g == '1') o.l("#define FOP_GELU_NR 1");
    o.l("#include \"fop_device.cuh\"");
    o.l("typedef " + idx + " idx_t;");
    o.l("extern \"C\" __global__ void __launch_bounds__(" + num(L.block) + ", " + num(minblocks) + ") " +
        (L.row_q > 1 ? "__cluster_dims__(" + num(L.row_q) + ", 1, 1) " : std::string("")) + L.name +
        "(const FopArgs args) {");
    o.ind++;
    for (int t = 0; t < d.ntensors; t++) {
      bool used = false;
      for (auto& a : L.loads) used |= a.tensor == t;
      for (auto& x : L.stmts) used |= x.write.tensor == t;
      if (!used) continue;
      o.l((written_here(t) ? std::string("char* __restrict__ T") : std::string("const char* __restrict__ T")) +
          num(t) + " = args.p[" + num(t) + "];");
    }
    o.l("const u64 fop_zero = (u64)args.zero;  (void)fop_zero;");
    if ((geometry_knob(L, "FOP_PDL_EMIT", 0) & 1) && geometry_knob(L, "FOP_PDL_POS", 1) == 0)
      o.l("fop::pdl_trigger();");
  }
  void footer() {
    const int emit = geometry_knob(L, "FOP_PDL_EMIT", 0);
    if ((emit & 1) && geometry_knob(L, "FOP_PDL_POS", 1) == 1) o.l("fop::pdl_trigger();");
    if (emit & 2) {
      if (geometry_knob(L, "FOP_PDL_WAITALL", 0)) o.l("fop::pdl_wait();");
      else o.l("if (blockIdx.x == 0u && threadIdx.x == 0u) fop::pdl_wait();");
    }
    o.ind--;
    o.l("}");
  }

  // decompose `var` (consumed) over kernel loops [k0, k1) into it names
  void decompose(const std::string& var, int k0, int k1, const std::string& tag,
                 std::vector<std::pair<int, std::string>>& its) {
    for (int k = k0; k < k1; k++) {
      std::string nm = "i" + num(k) + tag;
      if (k == k1 - 1) o.l("[[maybe_unused]] const idx_t " + nm + " = " + var + ";");
      else {
        o.l("[[maybe_unused]] const idx_t " + nm + " = " + var + " % " + num(L.kl[k].extent) + "u;");
        o.l(var + " /= " + num(L.kl[k].extent) + "u;");
      }
      its.push_back({k, nm});
    }
  }

  // ------------------------------------------------------------ shared-memory tables
  // An invariant sub-DAG (constant along the vector loop) that depends on ONE
  // kernel loop of small extent and contains a costly op (÷, √, exp, ...) —
  // BN's scale[c] = γ/√(var+ε), shift[c] — is evaluated once per CTA for every
  // value of that loop into shared memory, then looked up per vector, instead
  // of being recomputed for every vector.  Identical IEEE operations, so the
  // bits are unchanged.
  struct Table {
    int si, node, k;
    int64_t E;
    std::string name;
  };
  std::vector<Table> tables;
  std::vector<std::vector<std::string>> over;   // per statement: node -> lookup expression

  void plan_tables() {
    tables.clear();
    over.assign(L.stmts.size(), {});
    if (!geometry_knob(L, "FOP_SMEM_TABLES", 1)) return;
    int64_t bytes = 0;
    for (size_t si = 0; si < L.stmts.size(); si++) {
      const XStmt& x = L.stmts[si];
      size_t n = x.nodes.size();
      std::vector<uint32_t> dep(n, 0);
      std::vector<bool> costly(n, false), var(n, false);
      for (size_t i = 0; i < n; i++) {
        const XNode& q = x.nodes[i];
        if (q.op == FOP_OP_LOAD) {
          for (size_t k = 0; k < L.kl.size(); k++)
            if (C(L.loads[q.acc], (int)k) != 0) dep[i] |= 1u << k;
          // a flattened period launch: loop 0 is (c, r); only the period loads
          // depend on c alone, the others on the whole flat index (pseudo-loop 30)
          if (L.period && !L.period_load[q.acc] && (dep[i] & 1u)) dep[i] |= 1u << 30;
        } else if (q.op == X_FWD || q.op == X_SELF || q.op == X_SCALAR) {
          dep[i] = ~0u;
        } else if (q.op != FOP_OP_CONST) {
          dep[i] = (q.a >= 0 ? dep[q.a] : 0) | (q.b >= 0 ? dep[q.b] : 0);
          costly[i] = q.op == FOP_OP_DIV || q.op == FOP_OP_SQRT || (q.op >= FOP_OP_EXP && q.op <= FOP_OP_GELU_ERF) ||
                      (q.a >= 0 && costly[q.a]) || (q.b >= 0 && costly[q.b]);
        }
        var[i] = dep[i] & 1u;
      }
      over[si].assign(n, "");
      for (size_t i = 0; i < n; i++) {
        bool frontier = false;   // an invariant operand of a varying node
        for (size_t j = i + 1; j < n; j++)
          if (var[j] && (x.nodes[j].a == (int)i || x.nodes[j].b == (int)i)) frontier = true;
        // a cone over the vector loop alone (NHWC BatchNorm: scale[c] with c
        // = d_v) whose consumers mix in other loops: tabulated too, looked up
        // per element (tbl[iv + e]); needs whole vectors (no ragged tail)
        bool frontier0 = false;
        for (size_t j = i + 1; j < n; j++)
          if ((x.nodes[j].a == (int)i || x.nodes[j].b == (int)i) && (dep[j] & ~1u)) frontier0 = true;
        // (a flattened period launch: the cone depends on c = flat index mod period, any consumer)
        const bool vec_table = dep[i] == 1u && costly[i] && frontier0 && geometry_knob(L, "FOP_SMEM_TABLES_V", 1) &&
                               ((L.kl.size() > 1 && L.kl[0].extent % L.width == 0) || L.period);
        if (!vec_table && (var[i] || !costly[i] || !frontier || __builtin_popcount(dep[i]) != 1)) continue;
        int k = __builtin_ctz(dep[i]);
        int64_t E = k == 0 && L.period ? L.period : L.kl[k].extent;
        if ((k == 0 && !vec_table) || E > 8192 || bytes + E * 4 > 32 * 1024) continue;
        bytes += E * 4;
        Table t{(int)si, (int)i, k, E, "tbl" + num(x.stmt) + "_" + num(i)};
        tables.push_back(t);
      }
    }
  }

  // emit the table fills (before the grid-stride loop) and return whether any
  void emit_tables() {
    if (tables.empty()) return;
    for (const Table& t : tables) {
      const XStmt& x = L.stmts[t.si];
      decide_fast(x);   // the table's nodes take the same forms as the statement's own emission
      o.l("__shared__ __align__(16) float " + t.name + "[" + num(t.E) + "];");
      o.l("for (unsigned ti = threadIdx.x; ti < " + num(t.E) + "u; ti += " + num(L.block) + "u) {");
      o.ind++;
      // the cone of the table node, with its single loop bound to ti
      std::vector<bool> cone(x.nodes.size(), false);
      cone[t.node] = true;
      for (int i = t.node; i >= 0; i--) {
        if (!cone[i]) continue;
        if (x.nodes[i].a >= 0) cone[x.nodes[i].a] = true;
        if (x.nodes[i].b >= 0) cone[x.nodes[i].b] = true;
      }
      std::vector<std::pair<int, std::string>> its = {{t.k, "(idx_t)ti"}};
      for (int i = 0; i <= t.node; i++) {
        if (!cone[i]) continue;
        const XNode& q = x.nodes[i];
        std::string nm = t.name + "_" + num(i), e;
        if (q.op == FOP_OP_LOAD) {
          const Affine& a = L.loads[q.acc];
          e = "fop::sload<" + std::string(dtn(d.t[a.tensor].dtype)) + ", fop::LD_CACHED>(" +
              ptr(a.tensor, affine(a, its)) + ")";
        } else {
          e = op_expr(q, q.a >= 0 ? t.name + "_" + num(q.a) : "", q.b >= 0 ? t.name + "_" + num(q.b) : "");
        }
        o.l("const float " + nm + " = " + e + ";");
      }
      o.l(t.name + "[ti] = " + t.name + "_" + num(t.node) + ";");
      o.ind--;
      o.l("}");
    }
    o.l("__syncthreads();");
  }

  // ------------------------------------------------------------ EW
  void gen_ew() {
    const int W = L.width;
    const int U = L.unroll;
    const int64_t EV = L.kl[0].extent;
    const int64_t NV = (EV + W - 1) / W;
    const bool tail = EV % W != 0;
    const int64_t STRIDE = L.grid * L.block;
    bool raw = L.stmts.size() == 1 && L.stmts[0].move && es(L.stmts[0].write.tensor) == 2;
    header("EW (elementwise/broadcast, grid-stride over vectors of d_v)", 1);
    if (!raw) plan_tables();
    if (!tables.empty()) {
      // the table fill (cold parameter loads + ÷/√) delays each CTA's first
      // streaming loads: start the first iteration's vectors towards L2 now
      o.l("{");
      o.ind++;
      o.l("const idx_t tid0 = (idx_t)blockIdx.x * " + num(L.block) + "u + threadIdx.x;");
      for (int u = 0; u < U; u++) {
        std::string t = "_p" + num(u);
        o.l("if (tid0 + (idx_t)" + num(STRIDE * u) + "ull < (idx_t)" + num(L.work) + "ull) {");
        o.ind++;
        o.l("idx_t r" + t + " = tid0 + (idx_t)" + num(STRIDE * u) + "ull;");
        std::vector<std::pair<int, std::string>> pits;
        if (L.kl.size() > 1) {
          o.l("const idx_t j" + t + " = r" + t + " % " + num(NV) + "u;");
          o.l("r" + t + " /= " + num(NV) + "u;");
        } else {
          o.l("const idx_t j" + t + " = r" + t + ";");
        }
        pits.push_back({0, "(j" + t + " * " + num(W) + "u)"});
        decompose("r" + t, 1, (int)L.kl.size(), t, pits);
        for (size_t k = 0; k < L.loads.size(); k++)
          if (C(L.loads[k], 0) == 1 && L.load_cb[k])
            o.l("asm volatile(\"prefetch.global.L2 [%0];\" :: \"l\"(" + ptr(L.loads[k].tensor, affine(L.loads[k], pits)) +
                "));");
        o.ind--;
        o.l("}");
      }
      o.ind--;
      o.l("}");
    }
    emit_tables();
    // loads still needed per vector once tabled cones are cut off
    std::vector<bool> need(L.loads.size(), raw);
    for (size_t si = 0; si < L.stmts.size() && !raw; si++) {
      std::vector<std::string> probe = over.empty() ? std::vector<std::string>() : over[si];
      for (const Table& t : tables)
        if (t.si == (int)si) probe[t.node] = "x";
      g_over = &probe;
      std::vector<bool> r = reachable(L.stmts[si]);
      g_over = nullptr;
      for (size_t i = 0; i < r.size(); i++)
        if (r[i] && !(si < over.size() && !probe.empty() && !probe[i].empty()) &&
            L.stmts[si].nodes[i].op == FOP_OP_LOAD)
          need[L.stmts[si].nodes[i].acc] = true;
    }
    o.l("const idx_t tid = (idx_t)blockIdx.x * " + num(L.block) + "u + threadIdx.x;");
    o.l("#pragma unroll 1");
    o.l("for (idx_t g = tid; g < (idx_t)" + num(L.work) + "ull; g += (idx_t)" + num(STRIDE * U) + "ull) {");
    o.ind++;
    std::vector<std::vector<std::pair<int, std::string>>> its(U);
    for (int u = 0; u < U; u++) {
      std::string t = "_" + num(u);
      o.l("const idx_t g" + t + " = g + (idx_t)" + num(STRIDE * u) + "ull;");
      o.l("const bool ok" + t + " = g" + t + " < (idx_t)" + num(L.work) + "ull;");
      o.l("idx_t r" + t + " = g" + t + ";");
      if (L.kl.size() > 1) {
        o.l("const idx_t j" + t + " = r" + t + " % " + num(NV) + "u;");
        o.l("r" + t + " /= " + num(NV) + "u;");
      } else {
        o.l("const idx_t j" + t + " = r" + t + ";");
      }
      o.l("const idx_t iv" + t + " = j" + t + " * " + num(W) + "u;");
      its[u].push_back({0, "iv" + t});
      decompose("r" + t, 1, (int)L.kl.size(), t, its[u]);
      if (tail) o.l("const bool full" + t + " = iv" + t + " + " + num(W) + "u <= " + num(EV) + "u;");
      if (L.period) {   // c of each element: the flat index modulo the period (one wrap at most: W <= period)
        o.l("unsigned PC" + t + "[" + num(W) + "];");
        o.l("{ const unsigned c0_ = (unsigned)(iv" + t + " % " + num(L.period) + "u);");
        o.l("  #pragma unroll");
        o.l("  for (int e = 0; e < " + num(W) + "; ++e) PC" + t + "[e] = c0_ + e >= " + num(L.period) + "u ? c0_ + e - " +
            num(L.period) + "u : c0_ + e; }");
      }
      // loads
      for (size_t k = 0; k < L.loads.size(); k++) {
        if (!need[k]) continue;
        const Affine& a = L.loads[k];
        int64_t cv = C(a, 0);
        std::string off = affine(a, its[u]);
        std::string nm = "L" + num(k) + t;
        std::string dt = dtn(d.t[a.tensor].dtype);
        if (raw) {
          o.l("u32 " + nm + "[" + num(W) + "];");
          o.l("if (ok" + t + ") {");
          if (cv == 1 && !tail)
            o.l("  fop::vload_raw<" + num(es(a.tensor)) + ", " + num(W) + ", " + num(L.load_cb[k]) + ", " +
                pol(a, false) + ">(" + nm + ", " + ptr(a.tensor, off) + ");");
          else
            o.l("  for (int e = 0; e < " + num(W) + "; ++e) " + nm + "[e] = fop::sload_raw<" +
                num(es(a.tensor)) + ", " + pol(a, false) + ">(" + ptr(a.tensor, off + " + e * " + num(cv)) + ");");
          o.l("}");
          continue;
        }
        if (L.period && L.period_load[k]) {   // bias[c] over the flattened (c, r): one element per lane slot
          std::vector<std::pair<int, std::string>> rest(its[u].begin() + 1, its[u].end());
          std::string off0 = affine(a, rest);
          o.l("float " + nm + "[" + num(W) + "];");
          o.l("#pragma unroll");
          o.l("for (int e = 0; e < " + num(W) + "; ++e) " + nm + "[e] = ok" + t + " ? fop::sload<" + dt + ", " +
              pol(a, true) + ">(" + ptr(a.tensor, off0 + " + (idx_t)PC" + t + "[e] * " + num(cv)) + ") : 0.f;");
          continue;
        }
        if (cv == 0) {
          o.l("float " + nm + " = 0.f;");
          o.l("if (ok" + t + ") " + nm + " = fop::sload<" + dt + ", " + pol(a, true) + ">(" +
              ptr(a.tensor, off) + ");");
          continue;
        }
        o.l("float " + nm + "[" + num(W) + "];");
        o.l("if (ok" + t + ") {");
        o.ind++;
        std::string vec = cv == 1
            ? "fop::vload<" + dt + ", " + num(W) + ", " + num(L.load_cb[k]) + ", " + pol(a, false) + ">(" + nm +
                  ", " + ptr(a.tensor, off) + ");"
            : "for (int e = 0; e < " + num(W) + "; ++e) " + nm + "[e] = fop::sload<" + dt + ", " +
                  pol(a, false) + ">(" + ptr(a.tensor, off + " + e * " + num(cv)) + ");";
        if (tail) {
          o.l("if (full" + t + ") { " + vec + " }");
          o.l("else { for (int e = 0; e < " + num(W) + "; ++e) " + nm + "[e] = (iv" + t + " + e < " + num(EV) +
              "u) ? fop::sload<" + dt + ", " + pol(a, false) + ">(" +
              ptr(a.tensor, off + " + e * " + num(cv)) + ") : 0.f; }");
        } else {
          o.l(vec);
        }
        o.ind--;
        o.l("}");
      }
    }
    // compute + store
    for (int u = 0; u < U; u++) {
      std::string t = "_" + num(u);
      if (raw) {
        const XStmt& x = L.stmts[0];
        int k = x.nodes[x.result].acc;
        std::string off = affine(x.write, its[u]);
        int64_t cw = C(x.write, 0);
        o.l("if (ok" + t + ") {");
        if (cw == 1 && !tail)
          o.l("  fop::vstore_raw<" + num(es(x.write.tensor)) + ", " + num(W) + ", " + num(L.store_cb[0]) + ", " +
              spol() + ">(" + ptr(x.write.tensor, off) + ", L" + num(k) + t + ");");
        else
          o.l("  for (int e = 0; e < " + num(W) + "; ++e) " + std::string(tail ? "if (iv" + t + " + e < " + num(EV) + "u) " : "") +
              "fop::sstore_raw<" + num(es(x.write.tensor)) + ">(" +
              ptr(x.write.tensor, off + " + e * " + num(cw)) + ", L" + num(k) + t + "[e]);");
        o.l("}");
        continue;
      }
      for (size_t si = 0; si < L.stmts.size(); si++) {
        const XStmt& x = L.stmts[si];
        DagCtx c;
        c.tag = t;
        c.load_varies = [&](int k) { return C(L.loads[k], 0) != 0; };
        c.load = [&, t](int k, const std::string& e) {
          return C(L.loads[k], 0) != 0 ? "L" + num(k) + t + "[" + e + "]" : "L" + num(k) + t;
        };
        c.fwd = [&, t](int s, const std::string& e) { return "F" + num(L.stmts[s].stmt) + t + "[" + e + "]"; };
        c.scalar = [&](int) { return std::string("0.f"); };
        std::vector<std::string> ov(x.nodes.size());
        for (const Table& tb : tables)
          if (tb.si == (int)si)
            for (auto& kv : its[u])
              if (kv.first == tb.k) {  // slots past the end (ok false) still evaluate: keep the index in the table
                if (tb.k == 0 && L.period) {   // per element at c = flat index mod period
                  ov[tb.node] = tb.name + "[PC" + t + "[$E]]";
                } else if (tb.k == 0) {   // per element: the vector's W entries, read with 16 B shared loads
                  const std::string tv = "TV" + tb.name.substr(3) + t;
                  o.l("float " + tv + "[" + num(L.width) + "];");
                  o.l("#pragma unroll");
                  if (L.width % 4 == 0)
                    o.l("for (int q_ = 0; q_ < " + num(L.width / 4) + "; ++q_) reinterpret_cast<float4*>(" + tv +
                        ")[q_] = reinterpret_cast<const float4*>(&" + tb.name + "[ok" + t + " ? " + kv.second +
                        " : 0u])[q_];");
                  else
                    o.l("for (int q_ = 0; q_ < " + num(L.width) + "; ++q_) " + tv + "[q_] = " + tb.name + "[(ok" + t +
                        " ? " + kv.second + " : 0u) + q_];");
                  ov[tb.node] = tv + "[$E]";
                } else {
                  ov[tb.node] = tb.name + "[ok" + t + " ? " + kv.second + " : 0u]";
                }
              }
        g_over = &ov;
        auto var = varies(x, c);
        emit_nodes(o, x, var, false, c);
        std::string R = "R" + num(x.stmt) + t;
        o.l("float " + R + "[" + num(W) + "];");
        Sink sk;
        sk.scalar = [&](const std::string& v) { o.l(R + "[e] = " + v + ";"); };
        sk.pair = [&](const std::string& v, const std::string& p) {
          o.l("fop::upk(" + v + ", " + R + "[2 * " + p + "], " + R + "[2 * " + p + " + 1]);");
        };
        emit_elems(o, x, var, c, W, sk);
        g_over = nullptr;
        if (x.fwd) {
          o.l("float F" + num(x.stmt) + t + "[" + num(W) + "];");
          o.l("#pragma unroll");
          o.l("for (int e = 0; e < " + num(W) + "; ++e) F" + num(x.stmt) + t + "[e] = fop::round_to<" +
              dtn(x.out_dtype) + ">(" + R + "[e]);");
        }
        if (!x.store) continue;
        std::string off = affine(x.write, its[u]);
        int64_t cw = C(x.write, 0);
        std::string dt = dtn(x.out_dtype);
        std::string sc = "for (int e = 0; e < " + num(W) + "; ++e) " +
                         std::string(tail ? "if (iv" + t + " + e < " + num(EV) + "u) " : "") + "fop::sstore<" + dt +
                         ">(" + ptr(x.write.tensor, off + " + e * " + num(cw)) + ", " + R + "[e]);";
        o.l("if (ok" + t + ") {");
        if (cw == 1) {
          std::string vec = "fop::vstore<" + dt + ", " + num(W) + ", " + num(L.store_cb[si]) + ", " + spol() + ">(" +
                            ptr(x.write.tensor, off) + ", " + R + ");";
          if (tail) o.l("  if (full" + t + ") { " + vec + " } else { " + sc + " }");
          else o.l("  " + vec);
        } else {
          o.l("  " + sc);
        }
        o.l("}");
      }
    }
    o.ind--;
    o.l("}");
    footer();
  }

  // ------------------------------------------------------------ EW, read-modify-write / recurrence
  // Fig. 2(c) of the paper: forall (parallel loops) / for (the
  // loops carrying the statement's dependences, in original order) / forvec
  // (d_v).  Read-modify-write (the target ignores the sequential loops): each
  // thread owns W target elements, keeps their running values in registers
  // across the sequential loops (rounded to the target dtype after every
  // update, as the in-order program stores them) and stores once at the end.
  // Recurrence (row N3: the target depends on every sequential loop and is
  // read back at a constant distance): each iteration stores its result; a
  // read 1..4 iterations back along the innermost sequential loop comes from
  // a register ring holding this thread's last stored values, any other read
  // of the target from memory (coherent loads of this thread's own stores —
  // the planner proved every dependence stays inside one thread).
  void gen_ew_seq() {
    const int W = L.width;
    const int64_t EV = L.kl[0].extent;
    const int64_t NV = (EV + W - 1) / W;
    const bool tail = EV % W != 0;
    const int64_t STRIDE = L.grid * L.block;
    const XStmt& x = L.stmts[0];
    const fop_desc& dd = d;
    const bool rec = L.rec;
    header(rec ? "EW recurrence (forall / for in order / forvec, row N3)"
               : "EW read-modify-write (forall / for in order / forvec, Fig. 2(c))", 1);
    o.l("const idx_t tid = (idx_t)blockIdx.x * " + num(L.block) + "u + threadIdx.x;");
    o.l("#pragma unroll 1");
    o.l("for (idx_t g = tid; g < (idx_t)" + num(L.work) + "ull; g += (idx_t)" + num(STRIDE) + "ull) {");
    o.ind++;
    o.l("idx_t r = g;");
    if (L.kl.size() > 1) {
      o.l("const idx_t j = r % " + num(NV) + "u;");
      o.l("r /= " + num(NV) + "u;");
    } else {
      o.l("const idx_t j = r;");
    }
    o.l("const idx_t iv = j * " + num(W) + "u;");
    std::vector<std::pair<int, std::string>> its = {{0, "iv"}};
    decompose("r", 1, (int)L.kl.size(), "", its);
    std::string guard = tail ? "if (iv + e < " + num(EV) + "u) " : "";
    auto seq_terms = [&](const Affine& a) {
      std::string s;
      for (size_t q = 0; q < L.seq.size(); q++) {
        int64_t cq = a.coef[L.seq[q]];
        if (cq) s += " + s" + num(q) + (cq == 1 ? "" : " * " + num(cq));
      }
      return s;
    };
    std::string dto = dtn(x.out_dtype);
    std::string woff = affine(x.write, its);
    int64_t cw = C(x.write, 0);
    auto store_vals = [&](const std::string& off, const std::string& v) {
      if (cw == 1 && !tail && L.store_cb[0])
        o.l("fop::vstore<" + dto + ", " + num(W) + ", " + num(L.store_cb[0]) + ", fop::ST_DEFAULT>(" +
            ptr(x.write.tensor, off) + ", " + v + ");");
      else
        o.l("#pragma unroll\nfor (int e = 0; e < " + num(W) + "; ++e) " + guard + "fop::sstore<" + dto + ">(" +
            ptr(x.write.tensor, off + " + e * " + num(cw)) + ", " + v + "[e]);");
    };
    int maxd = 0;
    if (rec)
      for (int f : L.fwd_dist) maxd = std::max(maxd, f);
    if (!rec) {  // running values of the target, read once
      o.l("float ACC[" + num(W) + "];");
      o.l("#pragma unroll");
      o.l("for (int e = 0; e < " + num(W) + "; ++e) ACC[e] = 0.f;");
      o.l("#pragma unroll");
      o.l("for (int e = 0; e < " + num(W) + "; ++e) " + guard + "ACC[e] = fop::sload<" + dto +
          ", fop::LD_COHERENT>(" + ptr(x.write.tensor, woff + " + e * " + num(cw)) + ");");
    }
    // ring of this thread's last stored values.  Zero-initialised although
    // never read before being written: left undefined on loop entry, ptxas
    // 12.9 merged H2 with the new H1 (tools/probes/fibdbg.py, measured).
    for (int q = 1; q <= maxd; q++) {
      o.l("float H" + num(q) + "[" + num(W) + "];   // stored value " + num(q) + " iteration(s) back");
      o.l("#pragma unroll\nfor (int e = 0; e < " + num(W) + "; ++e) H" + num(q) + "[e] = 0.f;");
    }
    const size_t nseq = L.seq.size();
    const int sl = L.seq.back();
    const int64_t EL = dd.extent[sl];
    const std::string slast = "s" + num(nseq - 1);
    // Loads that vary along the innermost sequential loop and do not touch the
    // target are prefetched P iterations ahead into a per-slot register
    // buffer (the loop is unrolled by P, so slots are static registers): a
    // thread's sequential chain otherwise exposes one HBM round trip per
    // iteration.  Raw words when the vector is word-granular.
    const int P = L.seq_prefetch;
    std::vector<int> pf(L.loads.size(), 0);   // 0: no, 1: float buffer, 2: raw words
    for (size_t k = 0; k < L.loads.size(); k++) {
      const Affine& a = L.loads[k];
      if (P <= 1 || a.tensor == x.write.tensor || a.coef[sl] == 0) continue;
      int64_t cv = C(a, 0);
      int eb = es(a.tensor);
      pf[k] = (cv == 1 && !tail && L.load_cb[k] >= 4 && W * eb >= 4) ? 2 : 1;
    }
    auto words = [&](size_t k) { return W * es(L.loads[k].tensor) / 4; };
    // the memory load of load k at the current iteration values into float dst[W] (or a scalar)
    auto emit_load = [&](size_t k, const std::string& dst, const std::string& sexpr, bool decl) {
      const Affine& a = L.loads[k];
      int64_t cv = C(a, 0);
      std::string off = "(" + affine(a, its) + seq_terms(a) + ")";
      if (!sexpr.empty()) {   // the innermost sequential index replaced by sexpr
        int64_t cs = a.coef[sl];
        off = "(" + off + " + (" + sexpr + " - " + slast + ")" + (cs == 1 ? "" : " * " + num(cs)) + ")";
      }
      std::string dt = dtn(dd.t[a.tensor].dtype);
      if (cv == 0) {
        o.l(std::string(decl ? "float " : "") + dst + " = fop::sload<" + dt + ", " + pol(a, true) + ">(" +
            ptr(a.tensor, off) + ");");
        return;
      }
      if (decl) o.l("float " + dst + "[" + num(W) + "];");
      if (cv == 1 && !tail && L.load_cb[k]) {
        o.l("fop::vload<" + dt + ", " + num(W) + ", " + num(L.load_cb[k]) + ", " + pol(a, false) + ">(" + dst + ", " +
            ptr(a.tensor, off) + ");");
      } else {
        o.l("#pragma unroll");
        o.l("for (int e = 0; e < " + num(W) + "; ++e) " + dst + "[e] = " + (tail ? "(iv + e < " + num(EV) + "u) ? " : "") +
            "fop::sload<" + dt + ", " + pol(a, false) + ">(" + ptr(a.tensor, off + " + e * " + num(cv)) + ")" +
            (tail ? " : 0.f" : "") + ";");
      }
    };
    auto emit_fill = [&](size_t k, const std::string& slot, const std::string& sexpr) {
      const Affine& a = L.loads[k];
      if (pf[k] == 2) {
        std::string off = "(" + affine(a, its) + seq_terms(a) + ")";
        int64_t cs = a.coef[sl];
        off = "(" + off + " + (" + sexpr + " - " + slast + ")" + (cs == 1 ? "" : " * " + num(cs)) + ")";
        o.l("fop::vload_words<" + std::string(dtn(dd.t[a.tensor].dtype)) + ", " + num(W) + ", " + num(L.load_cb[k]) +
            ", " + pol(a, false) + ">(PB" + num(k) + "[" + slot + "], " + ptr(a.tensor, off) + ");");
      } else {
        emit_load(k, "PB" + num(k) + "[" + slot + "]", sexpr, false);
      }
    };
    for (size_t q = 0; q + 1 < nseq; q++) {
      o.l("#pragma unroll 1");
      o.l("for (idx_t s" + num(q) + " = 0; s" + num(q) + " < " + num(dd.extent[L.seq[q]]) + "u; ++s" + num(q) + ") {");
      o.ind++;
    }
    bool any_pf = false;
    for (int f : pf) any_pf |= f != 0;
    if (any_pf) {
      o.l("const idx_t " + slast + " = 0;   // prologue: iterations 0..P-1 of the innermost sequential loop");
      for (size_t k = 0; k < L.loads.size(); k++) {
        if (!pf[k]) continue;
        bool sc = C(L.loads[k], 0) == 0;
        if (pf[k] == 2) o.l("u32 PB" + num(k) + "[" + num(P) + "][" + num(words(k)) + "];");
        else o.l("float PB" + num(k) + "[" + num(P) + "]" + (sc ? "" : "[" + num(W) + "]") + ";");
      }
      o.l("#pragma unroll");
      o.l("for (int u = 0; u < " + num(P) + "; ++u) {");
      o.ind++;
      o.l("if ((idx_t)u < " + num(EL) + "u) {");
      o.ind++;
      for (size_t k = 0; k < L.loads.size(); k++)
        if (pf[k]) emit_fill(k, "u", "(idx_t)u");
      o.ind--;
      o.l("}");
      o.ind--;
      o.l("}");
      o.l("#pragma unroll 1");
      o.l("for (idx_t sb_ = 0; sb_ < " + num(EL) + "u; sb_ += " + num(P) + "u) {");
      o.ind++;
      o.l("#pragma unroll");
      o.l("for (int u = 0; u < " + num(P) + "; ++u) {");
      o.ind++;
      o.l("const idx_t " + slast + "_ = sb_ + (idx_t)u;");
      o.l("if (" + slast + "_ >= " + num(EL) + "u) break;");
      o.l("{");
      o.ind++;
      o.l("const idx_t " + slast + " = " + slast + "_;");
    } else {
      o.l("#pragma unroll 1");
      o.l("for (idx_t " + slast + " = 0; " + slast + " < " + num(EL) + "u; ++" + slast + ") {");
      o.ind++;
    }
    for (size_t k = 0; k < L.loads.size(); k++) {
      const Affine& a = L.loads[k];
      int64_t cv = C(a, 0);
      std::string nm = "L" + num(k);
      std::string dt = dtn(dd.t[a.tensor].dtype);
      int fd = rec && k < L.fwd_dist.size() ? L.fwd_dist[k] : 0;
      if (pf[k]) {   // take the prefetched slot, refill it P iterations ahead
        if (pf[k] == 2) {
          o.l("float " + nm + "[" + num(W) + "];");
          o.l("fop::cvt_words<" + dt + ", " + num(W) + ">(" + nm + ", PB" + num(k) + "[u]);");
        } else if (cv == 0) {
          o.l("const float " + nm + " = PB" + num(k) + "[u];");
        } else {
          o.l("float " + nm + "[" + num(W) + "];");
          o.l("#pragma unroll\nfor (int e = 0; e < " + num(W) + "; ++e) " + nm + "[e] = PB" + num(k) + "[u][e];");
        }
        o.l("if (" + slast + " + " + num(P) + "u < " + num(EL) + "u) {");
        o.ind++;
        emit_fill(k, "u", slast + " + " + num(P) + "u");
        o.ind--;
        o.l("}");
        continue;
      }
      if (cv == 0) {
        std::string off = "(" + affine(a, its) + seq_terms(a) + ")";
        std::string ld = "fop::sload<" + dt + ", " + pol(a, true) + ">(" + ptr(a.tensor, off) + ")";
        if (fd) o.l("const float " + nm + " = (" + slast + " >= " + num(fd) + "u) ? H" + num(fd) + "[0] : " + ld + ";");
        else o.l("const float " + nm + " = " + ld + ";");
        continue;
      }
      o.l("float " + nm + "[" + num(W) + "];");
      if (fd) {
        o.l("if (" + slast + " >= " + num(fd) + "u) {");
        o.l("  #pragma unroll");
        o.l("  for (int e = 0; e < " + num(W) + "; ++e) " + nm + "[e] = H" + num(fd) + "[e];");
        o.l("} else {");
        o.ind++;
      }
      emit_load(k, nm, "", false);
      if (fd) {
        o.ind--;
        o.l("}");
      }
    }
    DagCtx c;
    c.load_varies = [&](int k) { return C(L.loads[k], 0) != 0; };
    c.load = [&](int k, const std::string& e) {
      return C(L.loads[k], 0) != 0 ? "L" + num(k) + "[" + e + "]" : "L" + num(k);
    };
    c.fwd = [&](int, const std::string&) { return std::string("0.f"); };
    c.scalar = [&](int) { return std::string("0.f"); };
    c.self = [&](const std::string& e) { return "ACC[" + e + "]"; };
    auto var = varies(x, c);
    emit_nodes(o, x, var, false, c);
    o.l("float R[" + num(W) + "];");
    Sink sk;
    sk.scalar = [&](const std::string& v) { o.l("R[e] = " + v + ";"); };
    sk.pair = [&](const std::string& v, const std::string& p) {
      o.l("fop::upk(" + v + ", R[2 * " + p + "], R[2 * " + p + " + 1]);");
    };
    emit_elems(o, x, var, c, W, sk);
    if (rec) {
      store_vals("(" + woff + seq_terms(x.write) + ")", "R");
      for (int q = maxd; q >= 2; q--)
        o.l("#pragma unroll\nfor (int e = 0; e < " + num(W) + "; ++e) H" + num(q) + "[e] = H" + num(q - 1) + "[e];");
      if (maxd >= 1)
        o.l("#pragma unroll\nfor (int e = 0; e < " + num(W) + "; ++e) H1[e] = fop::round_to<" + dto + ">(R[e]);   // the stored value");
    } else {
      o.l("#pragma unroll");
      o.l("for (int e = 0; e < " + num(W) + "; ++e) ACC[e] = fop::round_to<" + dto + ">(R[e]);   // the stored value");
    }
    if (any_pf) {   // the unrolled block, the slot loop and the block loop
      for (int q = 0; q < 3; q++) {
        o.ind--;
        o.l("}");
      }
    } else {
      o.ind--;
      o.l("}");
    }
    for (size_t q = 0; q + 1 < nseq; q++) {
      o.ind--;
      o.l("}");
    }
    if (!rec) store_vals(woff, "ACC");
    o.ind--;
    o.l("}");
    footer();
  }

  // ------------------------------------------------------------ TRANSPOSE
  void gen_transpose() {
    const int W = L.width, WR = L.read_width;
    const int U = std::max(1, L.unroll);
    const int64_t NTV = L.kl[0].extent / W, NTR = L.kl[1].extent / WR;
    const int64_t TVH = (NTV + L.gv - 1) / L.gv;
    const int64_t TRH = (NTR + (int64_t)L.gr * U - 1) / ((int64_t)L.gr * U);
    const int64_t STRIDE = L.grid * L.block;
    const XStmt& x = L.stmts[0];
    bool raw = x.move && es(x.write.tensor) == 2;
    header("TRANSPOSE (register tiles W x WR, U per thread; both sides vectorised)", 1);
    o.l("const idx_t tid = (idx_t)blockIdx.x * " + num(L.block) + "u + threadIdx.x;");
    o.l("#pragma unroll 1");
    o.l("for (idx_t g = tid; g < (idx_t)" + num(L.work) + "ull; g += (idx_t)" + num(STRIDE) + "ull) {");
    o.ind++;
    o.l("idx_t t = g;");
    o.l("const idx_t tv_lo = t % " + num(L.gv) + "u; t /= " + num(L.gv) + "u;");
    o.l("const idx_t tr_lo = t % " + num(L.gr) + "u; t /= " + num(L.gr) + "u;");
    // traversal of the (tv_hi, tr_hi) tile grid by consecutive warps:
    // 0 = d_v tiles fastest (the resident warps cover a strip along d_v),
    // 1 = d_r tiles fastest, 2 = blocks of BV d_v tiles x all d_r tiles
    const int tro = geometry_knob(L, "FOP_TR_ORDER", 0);
    const int64_t BV = std::max(1, geometry_knob(L, "FOP_TR_BV", 8));
    if (tro == 1) {
      o.l("const idx_t tr_hi = t % " + num(TRH) + "u; t /= " + num(TRH) + "u;");
      if (L.kl.size() > 2) o.l("const idx_t tv_hi = t % " + num(TVH) + "u; t /= " + num(TVH) + "u;");
      else o.l("const idx_t tv_hi = t;");
    } else if (tro == 2) {
      const int64_t TVB = (TVH + BV - 1) / BV;
      o.l("const idx_t tv_m = t % " + num(BV) + "u; t /= " + num(BV) + "u;");
      o.l("const idx_t tr_hi = t % " + num(TRH) + "u; t /= " + num(TRH) + "u;");
      if (L.kl.size() > 2) o.l("const idx_t tv_b = t % " + num(TVB) + "u; t /= " + num(TVB) + "u;");
      else o.l("const idx_t tv_b = t;");
      o.l("const idx_t tv_hi = tv_b * " + num(BV) + "u + tv_m;");
    } else {
      o.l("const idx_t tv_hi = t % " + num(TVH) + "u; t /= " + num(TVH) + "u;");
      if (L.kl.size() > 2) o.l("const idx_t tr_hi = t % " + num(TRH) + "u; t /= " + num(TRH) + "u;");
      else o.l("const idx_t tr_hi = t;");
    }
    o.l("const idx_t tv = tv_hi * " + num(L.gv) + "u + tv_lo;");
    o.l("if (tv >= " + num(NTV) + "u) continue;");
    o.l("const idx_t iv = tv * " + num(W) + "u;");
    std::vector<std::pair<int, std::string>> outer;
    decompose("t", 2, (int)L.kl.size(), "", outer);
    // loads: A = vector along d_v [b][a]; B = vector along d_r [a][b]; S = scalar; G = gather [a][b]
    // A/B vectors are kept as raw words until the tile is computed (fewer registers per byte in flight)
    std::vector<char> kind(L.loads.size());
    std::vector<int> wpv(L.loads.size(), 0);
    std::vector<std::vector<std::pair<int, std::string>>> its(U);
    for (int u = 0; u < U; u++) {
      std::string t = "_" + num(u);
      o.l("const idx_t tr" + t + " = tr_hi * " + num((int64_t)L.gr * U) + "u + " + num((int64_t)u * L.gr) +
          "u + tr_lo;");
      o.l("const bool ok" + t + " = tr" + t + " < " + num(NTR) + "u;");
      o.l("const idx_t ir" + t + " = tr" + t + " * " + num(WR) + "u;");
      its[u] = {{0, "iv"}, {1, "ir" + t}};
      its[u].insert(its[u].end(), outer.begin(), outer.end());
      for (size_t k = 0; k < L.loads.size(); k++) {
        const Affine& a = L.loads[k];
        int64_t cv = C(a, 0), cr = C(a, 1);
        std::string off = affine(a, its[u]);
        std::string nm = "L" + num(k) + t;
        std::string dt = dtn(d.t[a.tensor].dtype);
        int eb = es(a.tensor);
        if (cv == 1 || cr == 1) {
          kind[k] = cv == 1 ? 'A' : 'B';
          int n_in = cv == 1 ? W : WR, n_out = cv == 1 ? WR : W;   // vector length, vector count
          int cb = cv == 1 ? L.load_cb[k] : L.load_cb_r[k];
          int64_t step = cv == 1 ? cr : cv;
          std::string vloop = cv == 1 ? "b" : "a";
          if (raw) {
            o.l("u32 " + nm + "[" + num(n_out) + "][" + num(n_in) + "];");
            o.l("#pragma unroll");
            o.l("for (int " + vloop + " = 0; " + vloop + " < " + num(n_out) + "; ++" + vloop + ") if (ok" + t +
                ") fop::vload_raw<" + num(eb) + ", " + num(n_in) + ", " + num(cb) + ", " + pol(a, false) + ">(" +
                nm + "[" + vloop + "], " + ptr(a.tensor, off + " + " + vloop + " * " + num(step)) + ");");
          } else if (n_in * eb >= 4 && cb >= 4) {
            wpv[k] = n_in * eb / 4;
            o.l("u32 W" + nm + "[" + num(n_out) + "][" + num(wpv[k]) + "];");
            o.l("#pragma unroll");
            o.l("for (int " + vloop + " = 0; " + vloop + " < " + num(n_out) + "; ++" + vloop + ") if (ok" + t +
                ") fop::vload_words<" + dt + ", " + num(n_in) + ", " + num(cb) + ", " + pol(a, false) + ">(W" + nm +
                "[" + vloop + "], " + ptr(a.tensor, off + " + " + vloop + " * " + num(step)) + ");");
          } else {
            o.l("float " + nm + "[" + num(n_out) + "][" + num(n_in) + "];");
            o.l("#pragma unroll");
            o.l("for (int " + vloop + " = 0; " + vloop + " < " + num(n_out) + "; ++" + vloop + ") if (ok" + t +
                ") fop::vload<" + dt + ", " + num(n_in) + ", " + num(cb) + ", " + pol(a, false) + ">(" + nm + "[" +
                vloop + "], " + ptr(a.tensor, off + " + " + vloop + " * " + num(step)) + ");");
          }
        } else if (cv == 0 && cr == 0) {
          kind[k] = 'S';
          o.l("float " + nm + " = 0.f;");
          o.l("if (ok" + t + ") " + nm + " = fop::sload<" + dt + ", " + pol(a, true) + ">(" + ptr(a.tensor, off) + ");");
        } else {
          kind[k] = 'G';
          o.l("float " + nm + "[" + num(W) + "][" + num(WR) + "];");
          o.l("#pragma unroll");
          o.l("for (int a = 0; a < " + num(W) + "; ++a)");
          o.l("#pragma unroll");
          o.l("for (int b = 0; b < " + num(WR) + "; ++b) if (ok" + t + ") " + nm + "[a][b] = fop::sload<" + dt +
              ", " + pol(a, false) + ">(" + ptr(a.tensor, off + " + a * " + num(cv) + " + b * " + num(cr)) + ");");
        }
      }
    }
    int64_t cwr = C(x.write, 1);
    std::string dto = dtn(x.out_dtype);
    for (int u = 0; u < U; u++) {
      std::string t = "_" + num(u);
      std::string woff = affine(x.write, its[u]);
      o.l("if (ok" + t + ") {");
      o.ind++;
      if (raw) {
        int k = x.nodes[x.result].acc;
        o.l("u32 O[" + num(WR) + "][" + num(W) + "];");
        o.l("#pragma unroll");
        o.l("for (int b = 0; b < " + num(WR) + "; ++b)");
        o.l("#pragma unroll");
        o.l("for (int a = 0; a < " + num(W) + "; ++a) O[b][a] = " +
            std::string(kind[k] == 'A' ? "L" + num(k) + t + "[b][a]" : "L" + num(k) + t + "[a][b]") + ";");
        o.l("#pragma unroll");
        o.l("for (int b = 0; b < " + num(WR) + "; ++b) fop::vstore_raw<" + num(es(x.write.tensor)) + ", " +
            num(W) + ", " + num(L.store_cb[0]) + ", " + spol() + ">(" +
            ptr(x.write.tensor, woff + " + b * " + num(cwr)) + ", O[b]);");
      } else {
        for (size_t k = 0; k < L.loads.size(); k++) {
          if (!wpv[k]) continue;
          bool A = kind[k] == 'A';
          int n_in = A ? W : WR, n_out = A ? WR : W;
          std::string nm = "L" + num(k) + t;
          o.l("float " + nm + "[" + num(n_out) + "][" + num(n_in) + "];");
          o.l("#pragma unroll");
          o.l("for (int q = 0; q < " + num(n_out) + "; ++q) fop::cvt_words<" +
              std::string(dtn(d.t[L.loads[k].tensor].dtype)) + ", " + num(n_in) + ">(" + nm + "[q], W" + nm + "[q]);");
        }
        DagCtx c;
        c.tag = t;
        c.ev = "a";
        c.load_varies = [&](int k) { return kind[k] != 'S'; };
        c.load = [&, t](int k, const std::string& e) {
          std::string nm = "L" + num(k) + t;
          switch (kind[k]) {
            case 'A': return nm + "[b][" + e + "]";
            case 'S': return nm;
            default: return nm + "[" + e + "][b]";
          }
        };
        c.fwd = [&](int, const std::string&) { return std::string("0.f"); };
        c.scalar = [&](int) { return std::string("0.f"); };
        auto var = varies(x, c);
        emit_nodes(o, x, var, false, c);
        o.l("float O[" + num(WR) + "][" + num(W) + "];");
        o.l("#pragma unroll");
        o.l("for (int b = 0; b < " + num(WR) + "; ++b) {");
        o.ind++;
        Sink sk;
        sk.scalar = [&](const std::string& v) { o.l("O[b][a] = " + v + ";"); };
        sk.pair = [&](const std::string& v, const std::string& p) {
          o.l("fop::upk(" + v + ", O[b][2 * " + p + "], O[b][2 * " + p + " + 1]);");
        };
        emit_elems(o, x, var, c, W, sk);
        o.ind--;
        o.l("}");
        o.l("#pragma unroll");
        o.l("for (int b = 0; b < " + num(WR) + "; ++b) fop::vstore<" + dto + ", " + num(W) + ", " +
            num(L.store_cb[0]) + ", " + spol() + ">(" + ptr(x.write.tensor, woff + " + b * " + num(cwr)) +
            ", O[b]);");
      }
      o.ind--;
      o.l("}");
    }
    o.ind--;
    o.l("}");
    footer();
  }

  // ------------------------------------------------------------ TRANSPOSE, software-pipelined
  // The register transpose with the NEXT grid-stride iteration's tile loads
  // issued before the current tiles are converted and stored (FOP_TR_PIPE=1):
  // the thread's loads never drain between iterations.  Two register sets
  // (current / next) of raw words; same tiles, same arithmetic, same bits.
  bool transpose_pipe_ok() const {
    const XStmt& x = L.stmts[0];
    if (x.move || !geometry_knob(L, "FOP_TR_PIPE", 0)) return false;
    for (const auto& a : L.loads) {
      const int64_t cv = C(a, 0), cr = C(a, 1);
      if (cv == 1 || cr == 1) {
        if ((cv == 1 ? L.width : L.read_width) * es(a.tensor) < 4) return false;   // raw words need >= 4 B
      } else if (!(cv == 0 && cr == 0)) {
        return false;   // gathers: not pipelined
      }
    }
    return true;
  }
  void gen_transpose_pipe() {
    const int W = L.width, WR = L.read_width;
    const int U = std::max(1, L.unroll);
    const int64_t NTV = L.kl[0].extent / W, NTR = L.kl[1].extent / WR;
    const int64_t TVH = (NTV + L.gv - 1) / L.gv;
    const int64_t TRH = (NTR + (int64_t)L.gr * U - 1) / ((int64_t)L.gr * U);
    const int64_t STRIDE = L.grid * L.block;
    const XStmt& x = L.stmts[0];
    header("TRANSPOSE (register tiles W x WR, U per thread, next iteration's loads in flight)", 1);
    const int NO = (int)L.kl.size() - 2;   // outer kernel loops
    std::vector<char> kind(L.loads.size(), 'S');
    std::vector<int> wpv(L.loads.size(), 0), n_in(L.loads.size(), 0), n_out(L.loads.size(), 0);
    for (size_t k = 0; k < L.loads.size(); k++) {
      const int64_t cv = C(L.loads[k], 0), cr = C(L.loads[k], 1);
      if (cv == 1 || cr == 1) {
        kind[k] = cv == 1 ? 'A' : 'B';
        n_in[k] = cv == 1 ? W : WR;
        n_out[k] = cv == 1 ? WR : W;
        wpv[k] = n_in[k] * es(L.loads[k].tensor) / 4;
      }
    }
    // state of one fetched iteration: iv, outer iterators, per u: ir, ok, the raw words
    for (const std::string S : {"_c", "_n"}) {
      o.l("idx_t iv" + S + " = 0;");
      for (int q = 0; q < NO; q++) o.l("idx_t i" + num(q + 2) + S + " = 0;");
      for (int u = 0; u < U; u++) {
        o.l("idx_t ir_" + num(u) + S + " = 0; bool ok_" + num(u) + S + " = false;");
        for (size_t k = 0; k < L.loads.size(); k++)
          if (wpv[k]) o.l("u32 WL" + num(k) + "_" + num(u) + S + "[" + num(n_out[k]) + "][" + num(wpv[k]) + "];");
      }
    }
    auto fetch = [&](const std::string& g, const std::string& S) {
      o.l("{");
      o.ind++;
      o.l("idx_t t = " + g + ";");
      o.l("const idx_t tv_lo = t % " + num(L.gv) + "u; t /= " + num(L.gv) + "u;");
      o.l("const idx_t tr_lo = t % " + num(L.gr) + "u; t /= " + num(L.gr) + "u;");
      o.l("const idx_t tv_hi = t % " + num(TVH) + "u; t /= " + num(TVH) + "u;");
      if (NO > 0) o.l("const idx_t tr_hi = t % " + num(TRH) + "u; t /= " + num(TRH) + "u;");
      else o.l("const idx_t tr_hi = t;");
      o.l("const idx_t tv = tv_hi * " + num(L.gv) + "u + tv_lo;");
      o.l("const bool okv = " + g + " < (idx_t)" + num(L.work) + "ull && tv < " + num(NTV) + "u;");
      o.l("iv" + S + " = tv * " + num(W) + "u;");
      for (int q = 0; q < NO; q++) {
        if (q == NO - 1) o.l("i" + num(q + 2) + S + " = t;");
        else o.l("i" + num(q + 2) + S + " = t % " + num(L.kl[q + 2].extent) + "u; t /= " + num(L.kl[q + 2].extent) + "u;");
      }
      for (int u = 0; u < U; u++) {
        const std::string us = "_" + num(u) + S;
        o.l("{ const idx_t tr = tr_hi * " + num((int64_t)L.gr * U) + "u + " + num((int64_t)u * L.gr) + "u + tr_lo;");
        o.l("  ok" + us + " = okv && tr < " + num(NTR) + "u; ir" + us + " = tr * " + num(WR) + "u; }");
        std::vector<std::pair<int, std::string>> its = {{0, "iv" + S}, {1, "ir" + us}};
        for (int q = 0; q < NO; q++) its.push_back({q + 2, "i" + num(q + 2) + S});
        for (size_t k = 0; k < L.loads.size(); k++) {
          if (!wpv[k]) continue;
          const Affine& a = L.loads[k];
          const bool A = kind[k] == 'A';
          const int cb = A ? L.load_cb[k] : L.load_cb_r[k];
          const int64_t step = A ? C(a, 1) : C(a, 0);
          const std::string vl = A ? "b" : "a";
          o.l("#pragma unroll");
          o.l("for (int " + vl + " = 0; " + vl + " < " + num(n_out[k]) + "; ++" + vl + ") if (ok" + us +
              ") fop::vload_words<" + std::string(dtn(d.t[a.tensor].dtype)) + ", " + num(n_in[k]) + ", " + num(cb) +
              ", " + pol(a, false) + ">(WL" + num(k) + us + "[" + vl + "], " +
              ptr(a.tensor, affine(a, its) + " + " + vl + " * " + num(step)) + ");");
        }
      }
      o.ind--;
      o.l("}");
    };
    o.l("const idx_t tid = (idx_t)blockIdx.x * " + num(L.block) + "u + threadIdx.x;");
    fetch("tid", "_c");
    o.l("#pragma unroll 1");
    o.l("for (idx_t g = tid; g < (idx_t)" + num(L.work) + "ull; g += (idx_t)" + num(STRIDE) + "ull) {");
    o.ind++;
    fetch("(g + (idx_t)" + num(STRIDE) + "ull)", "_n");
    int64_t cwr = C(x.write, 1);
    std::string dto = dtn(x.out_dtype);
    for (int u = 0; u < U; u++) {
      const std::string t = "_" + num(u) + "_c";
      std::vector<std::pair<int, std::string>> its = {{0, "iv_c"}, {1, "ir" + t}};
      for (int q = 0; q < NO; q++) its.push_back({q + 2, "i" + num(q + 2) + "_c"});
      o.l("if (ok" + t + ") {");
      o.ind++;
      for (size_t k = 0; k < L.loads.size(); k++) {
        const std::string nm = "L" + num(k) + t;
        if (wpv[k]) {
          o.l("float " + nm + "[" + num(n_out[k]) + "][" + num(n_in[k]) + "];");
          o.l("#pragma unroll");
          o.l("for (int q = 0; q < " + num(n_out[k]) + "; ++q) fop::cvt_words<" +
              std::string(dtn(d.t[L.loads[k].tensor].dtype)) + ", " + num(n_in[k]) + ">(" + nm + "[q], W" + nm + "[q]);");
        } else {   // a scalar (constant over the tile)
          o.l("const float " + nm + " = fop::sload<" + std::string(dtn(d.t[L.loads[k].tensor].dtype)) + ", " +
              pol(L.loads[k], true) + ">(" + ptr(L.loads[k].tensor, affine(L.loads[k], its)) + ");");
        }
      }
      DagCtx c;
      c.tag = t;
      c.ev = "a";
      c.load_varies = [&](int k) { return kind[k] != 'S'; };
      c.load = [&, t](int k, const std::string& e) {
        std::string nm = "L" + num(k) + t;
        switch (kind[k]) {
          case 'A': return nm + "[b][" + e + "]";
          case 'S': return nm;
          default: return nm + "[" + e + "][b]";
        }
      };
      c.fwd = [&](int, const std::string&) { return std::string("0.f"); };
      c.scalar = [&](int) { return std::string("0.f"); };
      auto var = varies(x, c);
      emit_nodes(o, x, var, false, c);
      o.l("float O[" + num(WR) + "][" + num(W) + "];");
      o.l("#pragma unroll");
      o.l("for (int b = 0; b < " + num(WR) + "; ++b) {");
      o.ind++;
      Sink sk;
      sk.scalar = [&](const std::string& v) { o.l("O[b][a] = " + v + ";"); };
      sk.pair = [&](const std::string& v, const std::string& p) {
        o.l("fop::upk(" + v + ", O[b][2 * " + p + "], O[b][2 * " + p + " + 1]);");
      };
      emit_elems(o, x, var, c, W, sk);
      o.ind--;
      o.l("}");
      o.l("#pragma unroll");
      o.l("for (int b = 0; b < " + num(WR) + "; ++b) fop::vstore<" + dto + ", " + num(W) + ", " + num(L.store_cb[0]) +
          ", " + spol() + ">(" + ptr(x.write.tensor, affine(x.write, its) + " + b * " + num(cwr)) + ", O[b]);");
      o.ind--;
      o.l("}");
    }
    // the next iteration becomes the current one
    o.l("iv_c = iv_n;");
    for (int q = 0; q < NO; q++) o.l("i" + num(q + 2) + "_c = i" + num(q + 2) + "_n;");
    for (int u = 0; u < U; u++) {
      o.l("ir_" + num(u) + "_c = ir_" + num(u) + "_n; ok_" + num(u) + "_c = ok_" + num(u) + "_n;");
      for (size_t k = 0; k < L.loads.size(); k++)
        if (wpv[k])
          o.l("#pragma unroll\nfor (int q = 0; q < " + num(n_out[k]) + "; ++q)\n#pragma unroll\nfor (int w = 0; w < " +
              num(wpv[k]) + "; ++w) WL" + num(k) + "_" + num(u) + "_c[q][w] = WL" + num(k) + "_" + num(u) + "_n[q][w];");
    }
    o.ind--;
    o.l("}");
    footer();
  }

  // ------------------------------------------------------------ TRANSPOSE via shared memory
  // For d_r rows too short or odd to carry vectors (a 7x7 plane: 49
  // elements, 98 B rows) whose d_v rows are adjacent in the load tensor: a
  // tile of TV whole rows is ONE contiguous chunk of TV*E[d_r] elements.
  // Phase 1: the CTA copies it into shared memory with 16 B vector loads.
  // Phase 2: each thread reads W elements down a column (one per row, fixed
  // d_r index), evaluates the statement and stores a W-vector along d_v;
  // consecutive lanes take consecutive d_v chunks, so a warp's stores are
  // contiguous.  Several CTAs per SM overlap one's loads with another's
  // read-out.
  void gen_transpose_smem() {
    if (L.tr_smem == 2) {
      gen_transpose_smem_out();
      return;
    }
    const XStmt& x = L.stmts[0];
    const int W = L.width;
    const int64_t TV = L.tr_tv, ER = L.kl[1].extent, NVB = L.kl[0].extent / TV;
    const Affine& ta = L.loads[L.trans_load];
    const int esi = es(ta.tensor), eso = es(x.write.tensor);
    const int64_t tile_bytes = TV * ER * esi, nvec = tile_bytes / 16, nj = TV / W, nout = ER * nj;
    const bool raw = x.move && esi == eso;
    const std::string dti = dtn(d.t[ta.tensor].dtype), dto = dtn(x.out_dtype);
    header("TRANSPOSE via shared memory (flat tile of TV rows x E[d_r] in, vectors along d_v out)", 1);
    o.l("__shared__ __align__(16) unsigned char fop_tile[" + num(tile_bytes) + "];");
    for (size_t k = 0; k < L.loads.size(); k++) {   // constants (eligibility: no loop in the access)
      if ((int)k == L.trans_load) continue;
      const Affine& a = L.loads[k];
      o.l("const float L" + num(k) + " = fop::sload<" + std::string(dtn(d.t[a.tensor].dtype)) + ", " + pol(a, true) +
          ">(" + ptr(a.tensor, affine(a, {})) + ");");
    }
    o.l("#pragma unroll 1");
    o.l("for (idx_t g = blockIdx.x; g < (idx_t)" + num(L.work) + "ull; g += gridDim.x) {");
    o.ind++;
    o.l("[[maybe_unused]] idx_t t = g;");
    o.l("const idx_t vb = t % " + num(NVB) + "u; t /= " + num(NVB) + "u;");
    std::vector<std::pair<int, std::string>> outer;
    decompose("t", 2, (int)L.kl.size(), "", outer);
    std::vector<std::pair<int, std::string>> in_its = {{0, "vb * " + num(TV) + "u"}};
    in_its.insert(in_its.end(), outer.begin(), outer.end());
    o.l("const char* src = " + ptr(ta.tensor, affine(ta, in_its)) + ";");
    o.l("__syncthreads();   // the previous tile is read out");
    o.l("#pragma unroll 4");
    o.l("for (unsigned q = threadIdx.x; q < " + num(nvec) + "u; q += " + num(L.block) + "u) {");
    o.l("  u32 w[4];");
    o.l("  fop::ldraw<16, " + pol(ta, false) + ">(w, src + q * 16u);");
    o.l("  *reinterpret_cast<uint4*>(fop_tile + q * 16u) = make_uint4(w[0], w[1], w[2], w[3]);");
    o.l("}");
    o.l("__syncthreads();");
    o.l("#pragma unroll 2");
    o.l("for (unsigned q = threadIdx.x; q < " + num(nout) + "u; q += " + num(L.block) + "u) {");
    o.ind++;
    o.l("const unsigned j = q % " + num(nj) + "u, r = q / " + num(nj) + "u;");
    std::vector<std::pair<int, std::string>> out_its = {{0, "(vb * " + num(TV) + "u + j * " + num(W) + "u)"},
                                                        {1, "r"}};
    out_its.insert(out_its.end(), outer.begin(), outer.end());
    std::string dst = ptr(x.write.tensor, affine(x.write, out_its));
    std::string cell = "fop_tile + ((j * " + num(W) + "u + e) * " + num(ER) + "u + r) * " + num(esi) + "u";
    if (raw) {
      o.l("u32 O[" + num(W) + "];");
      o.l("#pragma unroll");
      o.l("for (int e = 0; e < " + num(W) + "; ++e) O[e] = " +
          std::string(esi == 2 ? "*reinterpret_cast<const u16*>(" : "*reinterpret_cast<const u32*>(") + cell + ");");
      o.l("fop::vstore_raw<" + num(eso) + ", " + num(W) + ", " + num(L.store_cb[0]) + ", " + spol() + ">(" + dst +
          ", O);");
    } else {
      std::string lt = "L" + num(L.trans_load);
      o.l("float " + lt + "[" + num(W) + "];");
      o.l("#pragma unroll");
      std::string rd = d.t[ta.tensor].dtype == FOP_F16    ? "fop::h2f(*reinterpret_cast<const u16*>(" + cell + "))"
                       : d.t[ta.tensor].dtype == FOP_BF16 ? "fop::b2f(*reinterpret_cast<const u16*>(" + cell + "))"
                                                          : "*reinterpret_cast<const float*>(" + cell + ")";
      o.l("for (int e = 0; e < " + num(W) + "; ++e) " + lt + "[e] = " + rd + ";");
      DagCtx c;
      c.tag = "";
      c.ev = "e";
      const int tl = L.trans_load;
      c.load_varies = [tl](int k) { return k == tl; };
      c.load = [tl](int k, const std::string& e) { return "L" + num(k) + (k == tl ? "[" + e + "]" : std::string()); };
      c.fwd = [&](int, const std::string&) { return std::string("0.f"); };
      c.scalar = [&](int) { return std::string("0.f"); };
      auto var = varies(x, c);
      emit_nodes(o, x, var, false, c);
      o.l("float O[" + num(W) + "];");
      Sink sk;
      sk.scalar = [&](const std::string& v) { o.l("O[e] = " + v + ";"); };
      sk.pair = [&](const std::string& v, const std::string& pp) {
        o.l("fop::upk(" + v + ", O[2 * " + pp + "], O[2 * " + pp + " + 1]);");
      };
      emit_elems(o, x, var, c, W, sk);
      o.l("fop::vstore<" + dto + ", " + num(W) + ", " + num(L.store_cb[0]) + ", " + spol() + ">(" + dst + ", O);");
    }
    (void)dti;
    o.ind--;
    o.l("}");
    o.ind--;
    o.l("}");
    footer();
  }

  // The mirror of gen_transpose_smem: d_v rows too short or odd to carry
  // store vectors (an input layer's C = 3, NHWC -> NCHW of a 7x7 plane) while
  // the output rows are adjacent, so a tile of TR output rows (d_r positions)
  // x all of d_v is ONE contiguous chunk of the output.  Phase 1 loads the E[d_v]
  // input rows of the tile with vectors along d_r into shared memory [v][r];
  // phase 2 writes the flat output chunk with 16 B vectors, each element read
  // from shared memory at (v, r) = (f % E[d_v], f / E[d_v]).
  void gen_transpose_smem_out() {
    const XStmt& x = L.stmts[0];
    const int64_t TR = L.tr_tv, EV = L.kl[0].extent, ER = L.kl[1].extent, NRB = ER / TR;
    const Affine& ta = L.loads[L.trans_load];
    const int esi = es(ta.tensor), eso = es(x.write.tensor);
    const int WR = L.read_width, OW = 16 / eso;
    const int64_t nin = EV * (TR / WR), nout = TR * EV / OW;
    const bool raw = x.move && esi == eso;
    header("TRANSPOSE via shared memory (vectors along d_r in, flat tile of TR output rows x E[d_v] out)", 1);
    o.l("__shared__ __align__(16) unsigned char fop_tile[" + num(TR * EV * esi) + "];");
    for (size_t k = 0; k < L.loads.size(); k++) {
      if ((int)k == L.trans_load) continue;
      const Affine& a = L.loads[k];
      o.l("const float L" + num(k) + " = fop::sload<" + std::string(dtn(d.t[a.tensor].dtype)) + ", " + pol(a, true) +
          ">(" + ptr(a.tensor, affine(a, {})) + ");");
    }
    o.l("#pragma unroll 1");
    o.l("for (idx_t g = blockIdx.x; g < (idx_t)" + num(L.work) + "ull; g += gridDim.x) {");
    o.ind++;
    o.l("[[maybe_unused]] idx_t t = g;");
    o.l("const idx_t rb = t % " + num(NRB) + "u; t /= " + num(NRB) + "u;");
    std::vector<std::pair<int, std::string>> outer;
    decompose("t", 2, (int)L.kl.size(), "", outer);
    std::vector<std::pair<int, std::string>> in_its = {{0, "v"}, {1, "(rb * " + num(TR) + "u + rc * " + num(WR) + "u)"}};
    in_its.insert(in_its.end(), outer.begin(), outer.end());
    // Tile orientation.  d_v-major (OM = 0): the input vectors land as 16 B
    // shared stores, the read-out gathers element (f mod E[d_v], f div E[d_v])
    // with lanes 8 tile rows apart — few banks when E[d_v] is long.  Output-
    // major (OM = 1, long E[d_v] such as C = 255): the tile IS the flat output
    // chunk; lanes take consecutive d_v positions (32 different input rows of
    // the same d_r vector) and scatter each vector's WR elements into
    // consecutive 2/4-byte cells — lane-contiguous, conflict-free — and the
    // read-out is a straight 16 B vector per thread.
    const bool OM = L.tr_om != 0;
    o.l("__syncthreads();   // the previous tile is written out");
    o.l("#pragma unroll 4");
    o.l("for (unsigned q = threadIdx.x; q < " + num(nin) + "u; q += " + num(L.block) + "u) {");
    o.ind++;
    if (OM) o.l("const unsigned v = q % " + num(EV) + "u, rc = q / " + num(EV) + "u;");
    else o.l("const unsigned rc = q % " + num(TR / WR) + "u, v = q / " + num(TR / WR) + "u;");
    o.l("u32 w[" + num(WR * esi / 4) + "];");
    o.l("fop::vload_words<" + std::string(dtn(d.t[ta.tensor].dtype)) + ", " + num(WR) + ", " +
        num(L.load_cb_r[L.trans_load]) + ", " + pol(ta, false) + ">(w, " + ptr(ta.tensor, affine(ta, in_its)) + ");");
    o.l("#pragma unroll");
    if (OM && esi == 2)
      o.l("for (int i = 0; i < " + num(WR) + "; ++i) reinterpret_cast<u16*>(fop_tile)[(rc * " + num(WR) + "u + i) * " +
          num(EV) + "u + v] = (u16)(w[i >> 1] >> ((i & 1) * 16));");
    else if (OM)
      o.l("for (int i = 0; i < " + num(WR) + "; ++i) reinterpret_cast<u32*>(fop_tile)[(rc * " + num(WR) + "u + i) * " +
          num(EV) + "u + v] = w[i];");
    else
      o.l("for (int c = 0; c < " + num(WR * esi / 4) + "; ++c) reinterpret_cast<u32*>(fop_tile + (v * " + num(TR) +
          "u + rc * " + num(WR) + "u) * " + num(esi) + "u)[c] = w[c];");
    o.ind--;
    o.l("}");
    o.l("__syncthreads();");
    std::vector<std::pair<int, std::string>> out_its = {{1, "rb * " + num(TR) + "u"}};
    out_its.insert(out_its.end(), outer.begin(), outer.end());
    o.l("char* dst = " + ptr(x.write.tensor, affine(x.write, out_its)) + ";");
    o.l("#pragma unroll 2");
    o.l("for (unsigned q = threadIdx.x; q < " + num(nout) + "u; q += " + num(L.block) + "u) {");
    o.ind++;
    std::string cell = "fop_tile + (((q * " + num(OW) + "u + e) % " + num(EV) + "u) * " + num(TR) + "u + (q * " +
                       num(OW) + "u + e) / " + num(EV) + "u) * " + num(esi) + "u";
    if (OM) {   // the thread's OW output elements: 16 B shared loads (8 or 4 B when the thread's
                // input bytes are fewer, e.g. 4 bf16 read out under 4 f32 stores — fuzz seed 51)
      const int nw = OW * esi / 4;
      const int cw = nw % 4 == 0 ? 4 : nw % 2 == 0 ? 2 : 1;   // words per shared load
      const std::string ty = cw == 4 ? "uint4" : cw == 2 ? "uint2" : "u32";
      o.l("u32 tw_[" + num(nw) + "];");
      o.l("#pragma unroll");
      o.l("for (int c = 0; c < " + num(nw / cw) + "; ++c) reinterpret_cast<" + ty + "*>(tw_)[c] = "
          "reinterpret_cast<const " + ty + "*>(fop_tile + q * " + num(OW * esi) + "u)[c];");
    }
    auto elem_bits = [&](const std::string& castty) {   // raw element e (u16 or u32 bits)
      if (!OM) return "*reinterpret_cast<const " + castty + "*>(" + cell + ")";
      return esi == 2 ? std::string("(u16)(tw_[e >> 1] >> ((e & 1) * 16))") : std::string("tw_[e]");
    };
    if (raw) {
      o.l("u32 O[" + num(OW) + "];");
      o.l("#pragma unroll");
      o.l("for (int e = 0; e < " + num(OW) + "; ++e) O[e] = " + elem_bits(esi == 2 ? "u16" : "u32") + ";");
      o.l("fop::vstore_raw<" + num(eso) + ", " + num(OW) + ", 16, " + spol() + ">(dst + q * 16u, O);");
    } else {
      std::string lt = "L" + num(L.trans_load);
      o.l("float " + lt + "[" + num(OW) + "];");
      o.l("#pragma unroll");
      std::string rd = d.t[ta.tensor].dtype == FOP_F16    ? "fop::h2f(" + elem_bits("u16") + ")"
                       : d.t[ta.tensor].dtype == FOP_BF16 ? "fop::b2f(" + elem_bits("u16") + ")"
                                                          : "__uint_as_float(" + elem_bits("u32") + ")";
      o.l("for (int e = 0; e < " + num(OW) + "; ++e) " + lt + "[e] = " + rd + ";");
      DagCtx c;
      c.tag = "";
      c.ev = "e";
      const int tl = L.trans_load;
      c.load_varies = [tl](int k) { return k == tl; };
      c.load = [tl](int k, const std::string& e) { return "L" + num(k) + (k == tl ? "[" + e + "]" : std::string()); };
      c.fwd = [&](int, const std::string&) { return std::string("0.f"); };
      c.scalar = [&](int) { return std::string("0.f"); };
      auto var = varies(x, c);
      emit_nodes(o, x, var, false, c);
      o.l("float O[" + num(OW) + "];");
      Sink sk;
      sk.scalar = [&](const std::string& v) { o.l("O[e] = " + v + ";"); };
      sk.pair = [&](const std::string& v, const std::string& pp) {
        o.l("fop::upk(" + v + ", O[2 * " + pp + "], O[2 * " + pp + " + 1]);");
      };
      emit_elems(o, x, var, c, OW, sk);
      o.l("fop::vstore<" + std::string(dtn(x.out_dtype)) + ", " + num(OW) + ", 16, " + spol() + ">(dst + q * 16u, O);");
    }
    o.ind--;
    o.l("}");
    o.ind--;
    o.l("}");
    footer();
  }

  // ------------------------------------------------------------ TRANSPOSE via TMA
  // 64x64 tiles of 16-bit data.  Per CTA (128 threads = two 64-thread tile
  // groups): a pipeline of S smem stages, each holding two 8 KB input tiles
  // loaded by cp.async.bulk.tensor (128B swizzle) and completed on an mbarrier;
  // each thread transposes one 8x8 sub-tile through registers (8 LDS.128 ->
  // compute -> 8 STS.128 into a swizzled output tile); one thread stores both
  // output tiles with cp.async.bulk.tensor and refills the stage.  Sub-tiles
  // are assigned along diagonals (ca = t, cb = t + d) so every quarter-warp
  // LDS.128/STS.128 touches 8 distinct 16 B bank groups of the swizzle.
  void gen_transpose_tma() {
    const XStmt& x = L.stmts[0];
    const int S = L.tma_stages, R = L.tma_rank;
    const int64_t NP = L.work;   // tile pairs
    bool raw = x.move;
    const int ktr = L.trans_load;
    std::string dti = dtn(d.t[L.loads[ktr].tensor].dtype), dto = dtn(x.out_dtype);
    o.l("// generated by libfop (planner + codegen); skeleton: TRANSPOSE via TMA (64x64 tiles, " + num(S) +
        "-stage mbarrier pipeline)");
    if (const char* g = std::getenv("FOP_GELU_NR"); g && *g == '1') o.l("#define FOP_GELU_NR 1");
    o.l("#include \"fop_device.cuh\"");
    o.l("typedef " + idx + " idx_t;");
    const int NW = L.block / 32;
    o.l("extern \"C\" __global__ void __launch_bounds__(" + num(L.block) + ", " + num(std::max(1, L.minblocks)) + ") " +
        L.name + "(const FopArgs args, const __grid_constant__ fop::TmaDesc tin, const __grid_constant__ fop::TmaDesc tout) {");
    o.ind++;
    o.l("extern __shared__ __align__(1024) unsigned char smem_raw[];");
    o.l("unsigned char* smem = (unsigned char*)(((unsigned long long)smem_raw + 1023ull) & ~1023ull);");
    o.l("const unsigned lane = threadIdx.x & 31u, wid = threadIdx.x >> 5;");
    o.l("// per warp: S input stages (8 KB tiles) + 2 output tiles, own mbarriers: warps never wait for each other");
    o.l("unsigned char* sin = smem + wid * " + num((S + 2) * 8192) + "u;");
    o.l("unsigned char* sout = sin + " + num(S * 8192) + ";");
    o.l("u64* full = (u64*)(smem + " + num(NW * (S + 2) * 8192) + ") + wid * " + num(S) + "u;");
    o.l("const u64 fop_zero = (u64)args.zero;  (void)fop_zero;");
    if ((geometry_knob(L, "FOP_PDL_EMIT", 0) & 1) && geometry_knob(L, "FOP_PDL_POS", 1) == 0)
      o.l("fop::pdl_trigger();");
    for (int t = 0; t < d.ntensors; t++) {
      bool used = false;
      for (size_t k = 0; k < L.loads.size(); k++) used |= (int)k != ktr && L.loads[k].tensor == t;
      if (used) o.l("const char* __restrict__ T" + num(t) + " = args.p[" + num(t) + "];");
    }
    // constant (scalar) loads
    for (size_t k = 0; k < L.loads.size(); k++) {
      if ((int)k == ktr) continue;
      const Affine& a = L.loads[k];
      o.l("const float L" + num(k) + " = fop::sload<" + std::string(dtn(d.t[a.tensor].dtype)) + ", fop::LD_CACHED>(" +
          ptr(a.tensor, num(a.base)) + ");");
    }
    // tile -> coordinates (elements): tv fastest, then tr, then outer kloops
    o.l("auto coords = [&](idx_t tile, int* ci, int* co) {");
    o.l("  const int tv = (int)(tile % " + num(L.tma_ntv) + "u); tile /= " + num(L.tma_ntv) + "u;");
    o.l("  const int tr = (int)(tile % " + num(L.tma_ntr) + "u); tile /= " + num(L.tma_ntr) + "u;");
    o.l("  ci[0] = tr * 64; ci[1] = tv * 64; co[0] = tv * 64; co[1] = tr * 64;");
    for (int q = 2; q < R; q++) {
      if (q == R - 1) o.l("  ci[" + num(q) + "] = co[" + num(q) + "] = (int)tile;");
      else o.l("  ci[" + num(q) + "] = co[" + num(q) + "] = (int)(tile % " + num(L.kl[q].extent) + "u); tile /= " +
               num(L.kl[q].extent) + "u;");
    }
    o.l("};");
    const int64_t T = L.tma_tiles;
    o.l("const idx_t first = (idx_t)blockIdx.x * " + num(NW) + "u + wid, tstride = (idx_t)gridDim.x * " + num(NW) + "u;");
    o.l("auto issue = [&](idx_t t, int s) {   // tile t into stage s");
    o.l("  int ci[5], co[5];");
    o.l("  coords(t, ci, co);");
    o.l("  fop::mbar_expect_tx(&full[s], 8192u);");
    o.l("  fop::tma_load(sin + s * 8192, &tin, &full[s], " + num(R) + ", ci);");
    o.l("};");
    o.l("if (lane == 0) {");
    o.l("  for (int s = 0; s < " + num(S) + "; ++s) fop::mbar_init(&full[s], 1);");
    o.l("  fop::fence_mbar_init();");
    o.l("  for (int s = 0; s < " + num(S) + "; ++s) {");
    o.l("    const idx_t t = first + (idx_t)s * tstride;");
    o.l("    if (t < " + num(T) + "u) issue(t, s);");
    o.l("  }");
    o.l("}");
    o.l("__syncwarp();");
    o.l("#pragma unroll 1");
    o.l("for (unsigned k = 0;; ++k) {");
    o.ind++;
    o.l("const idx_t tile = first + (idx_t)k * tstride;");
    o.l("if (tile >= " + num(T) + "u) break;");
    o.l("const int s = (int)(k % " + num(S) + "u);");
    o.l("const unsigned ph = (k / " + num(S) + "u) & 1u;");
    o.l("const int ob = (int)(k & 1u);");
    o.l("if (lane == 0) fop::bulk_wait_read<1>();   // this warp's store of step k-2 has left buffer ob");
    o.l("__syncwarp();");
    o.l("fop::mbar_wait(&full[s], ph);");
    o.l("const u32 ib = fop::smem_u32(sin + s * 8192), obase = fop::smem_u32(sout + ob * 8192);");
    o.l("#pragma unroll");
    o.l("for (int pass = 0; pass < 2; ++pass) {   // 64 sub-tiles, 2 per lane; quarter-warp = one diagonal");
    o.ind++;
    o.l("const unsigned tau = lane + 32u * pass;");
    o.l("const unsigned ca = tau & 7u, cb = ((tau & 7u) + (tau >> 3)) & 7u;");
    o.l("u32 w[8][4];");
    o.l("#pragma unroll");
    o.l("for (int i = 0; i < 8; ++i) fop::lds128(w[i], ib + (8u * ca + i) * 128u + ((cb ^ (unsigned)i) << 4));");
    if (raw) {
      // out row j (R = 8cb + j), chunk ca holds in[i][j] for i = 0..7
      o.l("#pragma unroll");
      o.l("for (int j = 0; j < 8; ++j) {");
      o.l("  u32 h[8];");
      o.l("  #pragma unroll");
      o.l("  for (int i = 0; i < 8; ++i) h[i] = (w[i][j >> 1] >> ((j & 1) * 16)) & 0xffffu;");
      o.l("  fop::sts128(obase + (8u * cb + j) * 128u + ((ca ^ (unsigned)j) << 4), h[0] | (h[1] << 16), h[2] | (h[3] << 16),"
          " h[4] | (h[5] << 16), h[6] | (h[7] << 16));");
      o.l("}");
    } else {
      o.l("float X[8][8];   // X[i][j]: V = 8ca+i, R = 8cb+j");
      o.l("#pragma unroll");
      o.l("for (int i = 0; i < 8; ++i) fop::cvt_words<" + dti + ", 8>(X[i], w[i]);");
      DagCtx c;
      c.tag = "";
      c.ev = "i";
      c.load_varies = [&](int k) { return k == ktr; };
      c.load = [&](int k, const std::string& e) { return k == ktr ? "X[" + e + "][j]" : "L" + num(k); };
      c.fwd = [&](int, const std::string&) { return std::string("0.f"); };
      c.scalar = [&](int) { return std::string("0.f"); };
      auto var = varies(x, c);
      emit_nodes(o, x, var, false, c);
      o.l("#pragma unroll");
      o.l("for (int j = 0; j < 8; ++j) {");
      o.ind++;
      o.l("float O[8];");
      Sink sk;
      sk.scalar = [&](const std::string& v) { o.l("O[i] = " + v + ";"); };
      sk.pair = [&](const std::string& v, const std::string& p) {
        o.l("fop::upk(" + v + ", O[2 * " + p + "], O[2 * " + p + " + 1]);");
      };
      emit_elems(o, x, var, c, 8, sk);
      std::string pack = x.out_dtype == FOP_BF16 ? "fop::f2b2" : "fop::f2h2";
      o.l("fop::sts128(obase + (8u * cb + j) * 128u + ((ca ^ (unsigned)j) << 4), " + pack + "(O[0], O[1]), " + pack +
          "(O[2], O[3]), " + pack + "(O[4], O[5]), " + pack + "(O[6], O[7]));");
      o.ind--;
      o.l("}");
    }
    o.ind--;
    o.l("}");
    o.l("fop::fence_async_smem();   // generic-proxy smem writes -> visible to the TMA store");
    o.l("__syncwarp();");
    o.l("if (lane == 0) {");
    o.l("  int ci[5], co[5];");
    o.l("  coords(tile, ci, co);");
    o.l("  fop::tma_store(&tout, sout + ob * 8192, " + num(R) + ", co);");
    o.l("  fop::bulk_commit();");
    o.l("  const idx_t tn = tile + (idx_t)" + num(S) + "u * tstride;");
    o.l("  if (tn < " + num(T) + "u) issue(tn, s);   // every lane has finished reading stage s");
    o.l("}");
    o.ind--;
    o.l("}");
    o.l("if (lane == 0) fop::bulk_wait<0>();");
    footer();
    (void)NP;
  }

  // ------------------------------------------------------------ ROW_REDUCE
  void gen_row() {
    const int W = L.width;
    const int64_t NVD = L.kl[0].extent / W;
    // G warps per row (few long rows): LN lanes across the row's vectors, the
    // G warp partials of a reduction combined in a fixed order through shared
    // memory, the row loop uniform across the block (it synchronises)
    const bool PEEL = L.row_peel != 0;   // per-row shift to the first aligned element (geometry)
    auto row_variant_acc = [&](const Affine& a) {
      for (size_t k = 1; k < L.kl.size(); k++)
        if (C(a, (int)k) != 0) return true;
      return false;
    };
    const int G = std::max(1, L.row_g);
    // Q CTAs per row (a thread-block cluster; few long rows): the row's lanes
    // span the cluster, block partials are combined through distributed
    // shared memory in rank order, identically in every CTA
    const int Q = std::max(1, L.row_q);
    // P rows per warp (short rows): 32/P lanes per row, group butterflies
    const int P = std::max(1, L.row_p);
    const int64_t LNB = 32 * (int64_t)G / P;   // lanes of one row inside a block
    const int64_t LN = LNB * Q;                // lanes of one row
    // the row loop synchronises (block-uniform trip count), or its shuffles
    // span several rows (P > 1: warp-uniform trip count, per-row validity)
    const bool MULTI = G > 1 || Q > 1 || P > 1;
    const int K = (int)((NVD + LN - 1) / LN);
    int64_t NRO = 1;
    for (int k = 1; k < L.nsplit; k++) NRO *= L.kl[k].extent;
    // split mode (geometry: few vectors, long outer reduction loops): lane =
    // (sub, v), v = lane % NVDP over the vectors, the SPL subgroups take the
    // outer reduction iterations sub, sub + SPL, ... (runtime loop)
    const int64_t SPL = L.row_split;
    const int64_t NVDP = SPL ? LN / SPL : 0;
    const bool jguard = NVD % LN != 0 || MULTI || SPL;
    int64_t rows = L.work;
    const int64_t WSTRIDE = L.grid * L.block / LN;
    // forwarded rows live in registers when they fit (<= 64 values per lane);
    // longer rows are re-read by the lane that stored them (same thread, same
    // address: program order makes the store visible; L2 serves the re-read)
    const bool regmode = NRO * K * W + (PEEL ? 1 : 0) <= 64 && !SPL;
    for (auto& x : L.stmts)
      if (x.kind == FOP_ASSIGN && x.fwd && !regmode && !x.store)
        fail(FOP_E_UNSUPPORTED, "ROW_REDUCE: a long forwarded row must be stored to be re-read");
    // outer reduction iterations: unrolled at compile time while the row can
    // stay in registers, a runtime loop otherwise (no per-vector register
    // arrays are indexed then: no hoisting, prefetch or register forwarding)
    const bool rt_ro = NRO > 64 || SPL;
    const int64_t NRO_E = rt_ro ? 1 : NRO;
    const int NP = (int)(NRO_E * K);   // vectors per lane per row held in registers
    // per-load treatment: hoisted (independent of the row: e.g. a bias, loaded
    // once per warp), prefetched (streaming vector of the first phase, loaded
    // one row ahead so the reductions overlap the next row's HBM latency), or
    // plain
    std::vector<char> mode(L.loads.size(), 'L');
    std::vector<bool> used0(L.loads.size(), false);
    for (auto& n : L.stmts[0].nodes)
      if (n.op == FOP_OP_LOAD) used0[n.acc] = true;
    for (size_t k = 0; k < L.loads.size(); k++) {
      const Affine& a = L.loads[k];
      bool row_inv = true;
      for (size_t q = L.nsplit; q < L.kl.size(); q++) row_inv &= C(a, (int)q) == 0;
      int64_t cv = C(a, 0);
      int es_k = es(a.tensor);
      if (rt_ro) continue;
      if (PEEL && cv != 0) continue;   // vector positions move with each row's shift
      if (L.row_hoist && row_inv && regmode && (cv == 0 || cv == 1) && !written_here(a.tensor)) mode[k] = 'H';
      else if (L.row_prefetch && used0[k] && cv == 1 && W * es_k >= 4 && L.load_cb[k] >= 4 &&
               NP * W * es_k / 4 <= 32 && !written_here(a.tensor))
        mode[k] = 'P';
    }
    auto ro_its = [&](int64_t ro, const std::vector<std::pair<int, std::string>>& base) {
      std::vector<std::pair<int, std::string>> its = base;
      int64_t rem = ro;
      for (int k = 1; k < L.nsplit; k++) {
        its.push_back({k, num(rem % L.kl[k].extent) + "u"});
        rem /= L.kl[k].extent;
      }
      return its;
    };
    auto lane_guard = [&](int kk) {
      return NVD % LN != 0 ? "if (lane + " + num(LN * kk) + "u < " + num(NVD) + "u) " : std::string("");
    };
    header(P > 1 ? "ROW_REDUCE (" + std::to_string(P) + " rows per warp, " + std::to_string(32 / P) +
                       " lanes across each row's vectors, group butterfly)"
           : G == 1 ? "ROW_REDUCE (one warp per row, lanes across d_v vectors, butterfly)"
                  : "ROW_REDUCE (" + std::to_string(G) + " warps per row, butterfly + fixed-order shared-memory combine)", 1);
    if (Q > 1) o.l("const idx_t lane = threadIdx.x % " + num(LNB) + "u + fop::cluster_ctarank() * " + num(LNB) + "u;");
    else o.l("const idx_t lane = threadIdx.x % " + num(LN) + "u;");
    if (SPL) o.l("const idx_t vl_ = lane % " + num(NVDP) + "u, sub_ = lane / " + num(NVDP) + "u;");
    if (G > 1) {
      o.l("const idx_t grp = threadIdx.x / " + num(LNB) + "u;");
      for (auto& x : L.stmts)
        if (x.kind == FOP_REDUCE) o.l("__shared__ float RS" + num(x.stmt) + "[" + num(L.block / 32) + "];");
    }
    if (Q > 1)
      for (auto& x : L.stmts)
        if (x.kind == FOP_REDUCE) o.l("__shared__ float RQ" + num(x.stmt) + ";");
    // hoisted row-invariant loads
    for (size_t k = 0; k < L.loads.size(); k++) {
      if (mode[k] != 'H') continue;
      const Affine& a = L.loads[k];
      std::string dt = dtn(d.t[a.tensor].dtype);
      bool vec = C(a, 0) == 1;
      o.l("float H" + num(k) + "[" + num(NP) + "]" + (vec ? "[" + num(W) + "]" : "") + ";");
      for (int64_t ro = 0; ro < NRO; ro++)
        for (int kk = 0; kk < K; kk++) {
          auto its = ro_its(ro, {});
          its.push_back({0, "((lane + " + num(LN * kk) + "u) * " + num(W) + "u)"});
          std::string off = affine(a, its);
          std::string dst = "H" + num(k) + "[" + num(ro * K + kk) + "]";
          if (vec)
            o.l(lane_guard(kk) + "fop::vload<" + dt + ", " + num(W) + ", " + num(L.load_cb[k]) + ", " +
                pol(a, true) + ">(" + dst + ", " + ptr(a.tensor, off) + ");");
          else
            o.l(dst + " = fop::sload<" + dt + ", " + pol(a, true) + ">(" + ptr(a.tensor, off) + ");");
        }
    }
    // prefetch of the first row's streaming loads
    // prefetch depth D = L.row_prefetch: rows row + WSTRIDE .. row + D*WSTRIDE in
    // flight while `row` is processed (ring P, P_1 .. P_{D-1}; D = 1 default)
    const int PD = std::max(1, L.row_prefetch);
    auto pslot = [&](size_t k, int dd) { return "P" + num(k) + (dd ? "_" + num(dd) : std::string("")); };
    auto emit_prefetch = [&](const std::string& rowvar, const std::string& tag, int slot) {
      bool any = false;
      for (size_t k = 0; k < L.loads.size(); k++) any |= mode[k] == 'P';
      if (!any) return;
      o.l("if (" + rowvar + " < (idx_t)" + num(rows) + "ull) {");
      o.ind++;
      o.l("idx_t pr = " + rowvar + ";");
      std::vector<std::pair<int, std::string>> pits;
      decompose("pr", L.nsplit, (int)L.kl.size(), tag, pits);
      for (size_t k = 0; k < L.loads.size(); k++) {
        if (mode[k] != 'P') continue;
        const Affine& a = L.loads[k];
        int wpv = W * es(a.tensor) / 4;
        for (int64_t ro = 0; ro < NRO; ro++)
          for (int kk = 0; kk < K; kk++) {
            auto its = ro_its(ro, pits);
            its.push_back({0, "((lane + " + num(LN * kk) + "u) * " + num(W) + "u)"});
            o.l(lane_guard(kk) + "fop::vload_words<" + std::string(dtn(d.t[a.tensor].dtype)) + ", " + num(W) +
                ", " + num(L.load_cb[k]) + ", " + pol(a, false) + ">(&" + pslot(k, slot) + "[" +
                num((ro * K + kk) * wpv) + "], " + ptr(a.tensor, affine(a, its)) + ");");
          }
      }
      o.ind--;
      o.l("}");
    };
    for (size_t k = 0; k < L.loads.size(); k++)
      if (mode[k] == 'P')
        for (int dd = 0; dd < PD; dd++) o.l("u32 " + pslot(k, dd) + "[" + num(NP * W * es(L.loads[k].tensor) / 4) + "];");
    o.l("idx_t row = ((idx_t)blockIdx.x * " + num(L.block) + "u + threadIdx.x) / " + num(LN) + "u;");
    emit_prefetch("row", "_p", 0);
    for (int dd = 1; dd < PD; dd++)
      emit_prefetch("row + (idx_t)" + num(WSTRIDE * dd) + "ull", "_p" + num(dd), dd);
    o.l("#pragma unroll 1");
    if (MULTI) {   // block-uniform trip count: every group (and every CTA of the cluster) reaches the barriers
      o.l("for (idx_t rb_ = ((idx_t)blockIdx.x * " + num(L.block) + "u) / " + num(LN) + "u; rb_ < (idx_t)" + num(rows) +
          "ull; rb_ += (idx_t)" + num(WSTRIDE) + "ull, row += (idx_t)" + num(WSTRIDE) + "ull) {");
      o.ind++;
      o.l("const bool rv = row < (idx_t)" + num(rows) + "ull;");
    } else {
      o.l("for (; row < (idx_t)" + num(rows) + "ull; row += (idx_t)" + num(WSTRIDE) + "ull) {");
      o.ind++;
    }
    for (size_t k = 0; k < L.loads.size(); k++)
      if (mode[k] == 'P') {
        int n = NP * W * es(L.loads[k].tensor) / 4;
        o.l("u32 Q" + num(k) + "[" + num(n) + "];");
        o.l("#pragma unroll");
        o.l("for (int i = 0; i < " + num(n) + "; ++i) Q" + num(k) + "[i] = P" + num(k) + "[i];");
        for (int dd = 0; dd + 1 < PD; dd++) {
          o.l("#pragma unroll");
          o.l("for (int i = 0; i < " + num(n) + "; ++i) " + pslot(k, dd) + "[i] = " + pslot(k, dd + 1) + "[i];");
        }
      }
    emit_prefetch("row + (idx_t)" + num(WSTRIDE * PD) + "ull", "_n", PD - 1);
    o.l("idx_t rr = row;");
    std::vector<std::pair<int, std::string>> rits;
    decompose("rr", L.nsplit, (int)L.kl.size(), "", rits);
    if (PEEL) {   // this row's shift to its first W-aligned element, full vectors, scalar head + tail
      // the shift follows the row-variant vectorised accesses (geometry checked
      // they agree modulo W); row-invariant vectors are read element-wise
      auto row_variant = [&](const Affine& a) {
        for (size_t k = 1; k < L.kl.size(); k++)
          if (C(a, (int)k) != 0) return true;
        return false;
      };
      const Affine* ref = nullptr;
      for (auto& a : L.loads)
        if (!ref && C(a, 0) == 1 && row_variant(a)) ref = &a;
      for (auto& x : L.stmts)
        if (!ref && C(x.write, 0) == 1 && row_variant(x.write)) ref = &x.write;
      const int64_t EVr = L.kl[0].extent;
      o.l("const unsigned pe_s = (" + num(W) + "u - (unsigned)(" + affine(*ref, rits) + " % " + num(W) + "u)) % " +
          num(W) + "u;");
      o.l("const unsigned pe_n = (" + num(EVr) + "u - pe_s) / " + num(W) + "u;");
      o.l("const unsigned pe_t = " + num(EVr) + "u - pe_n * " + num(W) + "u;");
    }
    auto load_varies_e = [&](int k) { return C(L.loads[k], 0) != 0; };
    for (size_t si = 0; si < L.stmts.size(); si++) {
      const XStmt& x = L.stmts[si];
      bool red = x.kind == FOP_REDUCE;
      o.l("// statement " + num(x.stmt) + (red ? " (REDUCE)" : " (ASSIGN)"));
      // Sums with many sequential terms per lane (long outer reduction loops
      // over few vectors) use compensated (Kahan) accumulation: the error of
      // a plain running sum grows with the count (R16's bound assumes a
      // short per-lane chain), Kahan's stays ~2u * sum|t| whatever the length.
      // integer reductions (R30): exact wrap-around, no Kahan, no packed fp32 pairs
      const bool ired = red && x.out_dtype == FOP_I32;
      const bool kahan = red && !ired && x.redop == FOP_RED_SUM && (SPL ? (NRO + SPL - 1) / SPL : NRO) * K * W > 128;
      const std::string RADD = ired ? "fop::iadd(" : "__fadd_rn(", RMAX = ired ? "fop::imax(" : "fop::op_max(";
      if (red) {
        o.l(std::string("float acc") + num(x.stmt) + " = " +
            (x.redop == FOP_RED_MAX ? (ired ? "__int_as_float(0x80000000)" : "__uint_as_float(0xff800000u)")
                                    : (ired ? "__int_as_float(0)" : "0.f")) + ";");
        if (x.redop == FOP_RED_SUM && !ired) o.l("u64 acc" + num(x.stmt) + "p = fop::pk1(0.f);");
        if (kahan) o.l("float acc" + num(x.stmt) + "c = 0.f; u64 acc" + num(x.stmt) + "cp = fop::pk1(0.f);");
      }
      if (x.kind == FOP_ASSIGN && x.fwd && regmode)
        o.l("float F" + num(x.stmt) + "[" + num(NRO * K * W + (PEEL ? 1 : 0)) + "];");
      for (int64_t ro = 0; ro < NRO_E; ro++) {
        // decomposition of ro over the outer reduction kloops (compile time;
        // at run time, inside the kk block, for the runtime loop)
        std::vector<std::pair<int, std::string>> its = rits;
        if (!rt_ro) {
          int64_t rem = ro;
          for (int k = 1; k < L.nsplit; k++) {
            its.push_back({k, num(rem % L.kl[k].extent) + "u"});
            rem /= L.kl[k].extent;
          }
        }
        for (int kk = 0; kk < K + (PEEL ? 1 : 0); kk++) {
          // PEEL: kk == K is the row's head + tail elements, one per lane, scalar
          const bool scal = PEEL && kk == K;
          const int Wb = scal ? 1 : W;
          std::string t = "_" + num(si) + "_" + num(ro) + "_" + num(kk);
          o.l("{");
          o.ind++;
          if (SPL) {
            o.l("[[maybe_unused]] const idx_t iv = vl_ * " + num(W) + "u;");
            o.l(std::string("if (") + (MULTI ? "rv && " : "") + "vl_ < " + num(NVD) + "u) {");
          } else {
            if (scal) {
              o.l("[[maybe_unused]] const idx_t iv = lane < pe_s ? lane : pe_n * " + num(W) + "u + lane;");
              o.l(std::string("if (") + (MULTI ? "rv && " : "") + "lane < pe_t) {");
            } else if (PEEL) {
              o.l("[[maybe_unused]] const idx_t iv = pe_s + (lane + " + num(LN * kk) + "u) * " + num(W) + "u;");
              o.l(std::string("if (") + (MULTI ? "rv && " : "") + "lane + " + num(LN * kk) + "u < pe_n) {");
            } else {
              o.l("[[maybe_unused]] const idx_t iv = (lane + " + num(LN * kk) + "u) * " + num(W) + "u;");
              if (jguard)
                o.l(std::string("if (") + (MULTI ? "rv && " : "") + "lane + " + num(LN * kk) + "u < " + num(NVD) + "u) {");
            }
          }
          auto its2 = its;
          if (rt_ro) {
            // the runtime loop over the outer reduction iterations runs
            // INSIDE the lane's (loop-invariant) guard, unrolled, so the loads
            // of several iterations are in flight per lane; per lane the
            // terms are accumulated vector by vector (a fixed order)
            o.l("#pragma unroll " + num(std::max(1, geometry_knob(L, "FOP_ROW_ROU", 8))));
            if (SPL) o.l("for (idx_t ro_ = sub_; ro_ < " + num(NRO) + "u; ro_ += " + num(SPL) + "u) {");
            else o.l("for (idx_t ro_ = 0; ro_ < " + num(NRO) + "u; ++ro_) {");
            o.ind++;
            o.l("idx_t rq_ = ro_;");
            decompose("rq_", 1, L.nsplit, "_r" + num(si), its2);
          }
          its2.push_back({0, "iv"});
          // loads used by this statement
          std::vector<bool> used(L.loads.size(), false);
          for (auto& n : x.nodes)
            if (n.op == FOP_OP_LOAD) used[n.acc] = true;
          for (size_t k = 0; k < L.loads.size(); k++) {
            if (!used[k]) continue;
            const Affine& a = L.loads[k];
            int64_t cv = C(a, 0);
            std::string off = affine(a, its2);
            std::string nm = "L" + num(k);
            std::string dt = dtn(d.t[a.tensor].dtype);
            int64_t vi = ro * K + kk;
            if (mode[k] == 'H') {
              if (cv == 0) o.l("const float " + nm + " = H" + num(k) + "[" + num(vi) + "];");
              else o.l("const float* " + nm + " = H" + num(k) + "[" + num(vi) + "];");
            } else if (mode[k] == 'P') {
              int wpv = W * es(a.tensor) / 4;
              o.l("float " + nm + "[" + num(W) + "];");
              o.l("fop::cvt_words<" + dt + ", " + num(W) + ">(" + nm + ", &Q" + num(k) + "[" + num(vi * wpv) + "]);");
            } else if (cv == 0) {
              o.l("const float " + nm + " = fop::sload<" + dt + ", " + pol(a, true) + ">(" + ptr(a.tensor, off) + ");");
            } else if (cv == 1 && PEEL && !scal && !row_variant_acc(a) && L.load_cb[k] >= 4) {
              // a row-invariant vector under the per-row shift: the two aligned
              // vectors around the window [iv, iv + W), then the window picked by
              // a switch on pe_s (uniform across the warp: one row per warp group)
              const int64_t EVr = L.kl[0].extent;
              auto its_a = its2;
              its_a.back().second = "(iv - pe_s)";
              const std::string pa = ptr(a.tensor, affine(a, its_a));
              o.l("float " + nm + "[" + num(W) + "];");
              o.l("{");
              o.l("  float A_[" + num(2 * W) + "];");
              o.l("  fop::vload<" + dt + ", " + num(W) + ", " + num(L.load_cb[k]) + ", " + pol(a, false) + ">(A_, " + pa + ");");
              o.l("  if (pe_s != 0u) {");
              o.l("    if (iv - pe_s + " + num(2 * W) + "u <= " + num(EVr) + "u) fop::vload<" + dt + ", " + num(W) + ", " +
                  num(L.load_cb[k]) + ", " + pol(a, false) + ">(A_ + " + num(W) + ", " + pa + " + " + num(W * es(a.tensor)) + ");");
              o.l("    else");
              o.l("      for (int e = 0; e < " + num(W) + "; ++e) A_[" + num(W) + " + e] = iv - pe_s + " + num(W) +
                  "u + e < " + num(EVr) + "u ? fop::sload<" + dt + ", " + pol(a, false) + ">(" + pa + " + (" +
                  num(W) + " + e) * " + num(es(a.tensor)) + ") : 0.f;");
              o.l("  }");
              o.l("  switch (pe_s) {");
              for (int sh = 0; sh < W; sh++) {
                std::string cs = "    case " + num(sh) + "u:";
                for (int e = 0; e < W; e++) cs += " " + nm + "[" + num(e) + "] = A_[" + num(e + sh) + "];";
                o.l(cs + " break;");
              }
              o.l("  }");
              o.l("}");
            } else if (cv == 1) {
              o.l("float " + nm + "[" + num(Wb) + "];");
              o.l("fop::vload<" + dt + ", " + num(Wb) + ", " + num(scal ? es(a.tensor) : L.load_cb[k]) + ", " +
                  pol(a, false) + ">(" + nm + ", " + ptr(a.tensor, off) + ");");
            } else {
              o.l("float " + nm + "[" + num(Wb) + "];");
              o.l("for (int e = 0; e < " + num(Wb) + "; ++e) " + nm + "[e] = fop::sload<" + dt + ", " +
                  pol(a, false) + ">(" + ptr(a.tensor, off + " + e * " + num(cv)) + ");");
            }
          }
          if (!regmode) {  // re-read forwarded rows from their stored tensor
            std::vector<bool> fw(L.stmts.size(), false);
            for (auto& n : x.nodes)
              if (n.op == X_FWD) fw[n.src] = true;
            for (size_t s2 = 0; s2 < L.stmts.size(); s2++) {
              if (!fw[s2]) continue;
              const XStmt& pr = L.stmts[s2];
              std::string off = affine(pr.write, its2);
              int64_t cw = C(pr.write, 0);
              std::string nm = "FW" + num(pr.stmt);
              std::string dt = dtn(pr.out_dtype);
              o.l("float " + nm + "[" + num(Wb) + "];");
              if (cw == 1)
                o.l("fop::vload<" + dt + ", " + num(Wb) + ", " + num(scal ? esize(pr.out_dtype) : L.store_cb[s2]) +
                    ", fop::LD_COHERENT>(" + nm + ", " + ptr(pr.write.tensor, off) + ");");
              else
                o.l("for (int e = 0; e < " + num(Wb) + "; ++e) " + nm + "[e] = fop::sload<" + dt +
                    ", fop::LD_COHERENT>(" + ptr(pr.write.tensor, off + " + e * " + num(cw)) + ");");
            }
          }
          DagCtx c;
          c.tag = "";
          c.load_varies = load_varies_e;
          c.load = [&](int k, const std::string& e) {
            return C(L.loads[k], 0) != 0 ? "L" + num(k) + "[" + e + "]" : "L" + num(k);
          };
          int64_t base_idx = (ro * K + kk) * W;   // scal: K * W, the slot after the row's vectors
          c.fwd = [&, base_idx](int s, const std::string& e) {
            return regmode ? "F" + num(L.stmts[s].stmt) + "[" + num(base_idx) + " + " + e + "]"
                           : "FW" + num(L.stmts[s].stmt) + "[" + e + "]";
          };
          c.scalar = [&](int s) { return "S" + num(L.stmts[s].stmt); };
          auto var = varies(x, c);
          emit_nodes(o, x, var, false, c);
          if (!red) o.l("float R[" + num(Wb) + "];");
          std::string A = "acc" + num(x.stmt);
          Sink sk;
          if (red) {
            bool mx = x.redop == FOP_RED_MAX;
            sk.scalar = [&, A, mx, RADD, RMAX](const std::string& v) {
              o.l(A + " = " + (mx ? RMAX : RADD) + A + ", " + v + ");");
            };
            if (kahan) {   // y = v - c; t = s + y; c = (t - s) - y; s = t
              sk.scalar = [&, A](const std::string& v) {
                o.l("{ const float y_ = __fsub_rn(" + v + ", " + A + "c); const float t_ = __fadd_rn(" + A + ", y_); " + A +
                    "c = __fsub_rn(__fsub_rn(t_, " + A + "), y_); " + A + " = t_; }");
              };
              sk.pair = [&, A](const std::string& v, const std::string&) {
                o.l("{ const u64 y_ = fop::sub2(" + v + ", " + A + "cp); const u64 t_ = fop::add2(" + A + "p, y_); " + A +
                    "cp = fop::sub2(fop::sub2(t_, " + A + "p), y_); " + A + "p = t_; }");
              };
              sk.pair_fma = [&, A](const std::string& a, const std::string& b, const std::string&) {
                o.l("{ const u64 y_ = fop::sub2(fop::mul2(" + a + ", " + b + "), " + A + "cp); const u64 t_ = fop::add2(" + A +
                    "p, y_); " + A + "cp = fop::sub2(fop::sub2(t_, " + A + "p), y_); " + A + "p = t_; }");
              };
            } else if (!mx && !ired) {
              sk.pair = [&, A](const std::string& v, const std::string&) { o.l(A + "p = fop::add2(" + A + "p, " + v + ");"); };
              sk.pair_fma = [&, A](const std::string& a, const std::string& b, const std::string&) {
                o.l(A + "p = fop::fma2(" + a + ", " + b + ", " + A + "p);");
              };
            }
          } else {
            std::string F = "F" + num(x.stmt) + "[" + num(base_idx) + " + ";
            bool keep = x.fwd && regmode;
            std::string dto = dtn(x.out_dtype);
            sk.scalar = [&, F, keep, dto](const std::string& v) {
              o.l("R[e] = " + v + ";");
              if (keep) o.l(F + "e] = fop::round_to<" + dto + ">(" + v + ");");
            };
            sk.pair = [&, F, keep, dto](const std::string& v, const std::string& p) {
              o.l("fop::upk(" + v + ", R[2 * " + p + "], R[2 * " + p + " + 1]);");
              if (keep)
                o.l("fop::round2<" + dto + ">(R[2 * " + p + "], R[2 * " + p + " + 1], " + F + "2 * " + p + "], " + F +
                    "2 * " + p + " + 1]);");
            };
          }
          emit_elems(o, x, var, c, Wb, sk);
          if (!red && x.store) {
            std::string off = affine(x.write, its2);
            int64_t cw = C(x.write, 0);
            std::string dt = dtn(x.out_dtype);
            if (cw == 1)
              o.l("fop::vstore<" + dt + ", " + num(Wb) + ", " + num(scal ? esize(x.out_dtype) : L.store_cb[si]) + ", " +
                  spol() + ">(" + ptr(x.write.tensor, off) + ", R);");
            else
              o.l("for (int e = 0; e < " + num(Wb) + "; ++e) fop::sstore<" + dt + ">(" +
                  ptr(x.write.tensor, off + " + e * " + num(cw)) + ", R[e]);");
          }
          if (rt_ro) {
            o.ind--;
            o.l("}");
          }
          if (jguard || PEEL) o.l("}");
          o.ind--;
          o.l("}");
        }
      }
      if (red) {
        std::string a = "acc" + num(x.stmt);
        if (kahan)   // each running sum minus its compensation, then combined
          o.l(a + " = __fadd_rn(__fsub_rn(" + a + ", " + a + "c), __fadd_rn(__fsub_rn(fop::lo(" + a + "p), fop::lo(" + a +
              "cp)), __fsub_rn(fop::hi(" + a + "p), fop::hi(" + a + "cp))));");
        else if (x.redop == FOP_RED_SUM && !ired)
          o.l(a + " = __fadd_rn(" + a + ", __fadd_rn(fop::lo(" + a + "p), fop::hi(" + a + "p)));");
        const std::string I = ired ? "i" : "";
        if (P > 1)
          o.l(a + " = " + std::string(x.redop == FOP_RED_MAX ? "fop::group_" + I + "max<" : "fop::group_" + I + "sum<") +
              num(LN) + ">(" + a + ");");
        else
          o.l(a + " = " + std::string(x.redop == FOP_RED_MAX ? "fop::warp_" + I + "max(" : "fop::warp_" + I + "sum(") + a +
              ");");
        if (G > 1) {   // the row's G warp partials, combined in warp order
          std::string rs = "RS" + num(x.stmt);
          o.l("if ((threadIdx.x & 31u) == 0u) " + rs + "[threadIdx.x >> 5] = " + a + ";");
          o.l("__syncthreads();");
          o.l(a + " = " + rs + "[grp * " + num(G) + "u];");
          o.l("#pragma unroll");
          o.l("for (int g_ = 1; g_ < " + num(G) + "; ++g_) " + a + " = " +
              (x.redop == FOP_RED_MAX ? RMAX : RADD) + a + ", " + rs + "[grp * " + num(G) + "u + g_]);");
          o.l("__syncthreads();");
        }
        if (Q > 1) {   // the cluster's Q block partials, read from every CTA's shared memory in rank order
          std::string rq = "RQ" + num(x.stmt);
          o.l("if (threadIdx.x == 0u) " + rq + " = " + a + ";");
          o.l("fop::cluster_sync();");
          o.l(a + " = fop::ld_dsmem(&" + rq + ", 0u);");
          o.l("#pragma unroll");
          o.l("for (unsigned q_ = 1; q_ < " + num(Q) + "u; ++q_) " + a + " = " +
              (x.redop == FOP_RED_MAX ? RMAX : RADD) + a + ", fop::ld_dsmem(&" + rq + ", q_));");
          o.l("fop::cluster_sync();");
        }
        std::string res = fin_expr(o, x, a, "");
        if (x.fwd) o.l("const float S" + num(x.stmt) + " = fop::round_to<" + dtn(x.out_dtype) + ">(" + res + ");");
        if (x.store)
          o.l(std::string(MULTI ? "if (rv && lane == 0) " : "if (lane == 0) ") + "fop::sstore<" + std::string(dtn(x.out_dtype)) + ">(" +
              ptr(x.write.tensor, affine(x.write, rits)) + ", " + res + ");");
      }
    }
    o.ind--;
    o.l("}");
    footer();
  }

  // ------------------------------------------------------------ COL_REDUCE
  void gen_col() {
    const int W = L.width, U = L.unroll;
    const XStmt& x = L.stmts[0];
    const int64_t EV0 = L.kl[0].extent;
    const int64_t FP = L.col_fold;   // > 0: P-row groups of dense odd rows, read as [R/P, P*E] (geometry.cpp)
    const int64_t NVD = L.col_shift ? (EV0 + W - 1) / W : FP ? FP * EV0 / W : EV0 / W;   // col_shift: a partial last vector
    const int64_t SVN = (NVD + L.gv - 1) / L.gv;
    int64_t slabs = SVN;
    for (int k = 1; k < L.nsplit; k++) slabs *= L.kl[k].extent;
    const int64_t ROWS = L.work;
    const int64_t NCH = L.nchunks;
    const int64_t RPC = (ROWS + NCH - 1) / NCH;
    const int SW = L.gv * W;
    // workspace address of byte `rel` of THIS launch's region (tuning candidates and the
    // narrow variant each own a region starting at their ws_off): checked at generation
    const auto wsa = [&](int64_t rel) {
      if (rel < 0 || rel >= (int64_t)L.ws_bytes)
        fail(FOP_E_INVALID, "internal: COL_REDUCE workspace offset outside the launch's region");
      return num((int64_t)L.ws_off + rel) + "ull";
    };
    bool isMax = x.redop == FOP_RED_MAX;
    const bool ired = x.out_dtype == FOP_I32;   // integer reduction (R30): exact, any order
    std::string init = isMax ? (ired ? "__int_as_float(0x80000000)" : "__uint_as_float(0xff800000u)")
                             : (ired ? "__int_as_float(0)" : "0.f");
    auto comb = [&](const std::string& a, const std::string& b) {
      if (ired) return (isMax ? "fop::imax(" : "fop::iadd(") + a + ", " + b + ")";
      return isMax ? "fop::op_max(" + a + ", " + b + ")" : "__fadd_rn(" + a + ", " + b + ")";
    };
    header("COL_REDUCE (slab of gv x W columns, row chunks, fixed-order trees)", 1);
    o.l("__shared__ float red[" + num(L.block * W) + "];");
    o.l("__shared__ unsigned last_flag;");
    o.l("(void)last_flag;   // (used by multi-chunk finalizes only)");
    if (FP) o.l("__shared__ unsigned fold_flag;");
    o.l("const unsigned tid = threadIdx.x, cv = tid % " + num(L.gv) + "u, rl = tid / " + num(L.gv) + "u;");
    o.l("const idx_t slab = blockIdx.x % " + num(slabs) + "u, chunk = blockIdx.x / " + num(slabs) + "u;");
    // peer exchange: the slab's run counter, read in the epilogue (FOP_PEER_EP=0, default) or at kernel
    // start (1: volatile load, measured 4 us slower on cfg4b; 2: ld.global.cg)
    const int peer_ep = L.peer ? geometry_knob(L, "FOP_PEER_EP", 0) : 0;
    if (peer_ep)
      o.l(std::string("const unsigned xep0_ = ") + (peer_ep == 1 ? "((volatile const unsigned*)" : "__ldcg((const unsigned*)") +
          "(args.peer[args.rank] + " + num((int64_t)L.peer_off) + "ull + " +
          num((int64_t)peer_layout(L, p.opts.peer_world).epoch) + "ull)" + (peer_ep == 1 ? ")[slab];" : " + slab);"));
    o.l("idx_t sr = slab;");
    o.l("const idx_t sv = sr % " + num(SVN) + "u; sr /= " + num(SVN) + "u;");
    std::vector<std::pair<int, std::string>> cits;
    if (L.nsplit > 1) decompose("sr", 1, L.nsplit, "", cits);
    o.l("const idx_t j = sv * " + num(L.gv) + "u + cv;");
    o.l("const bool okc = j < " + num(NVD) + "u;");
    o.l("const idx_t iv = j * " + num(W) + "u;");
    cits.push_back({0, "iv"});
    // Row assignment.  Interleaved (default): chunk c takes rows
    // (k*NCH + c)*gr + rl, so the whole grid sweeps the matrix front to back
    // together (measured +3% over contiguous chunks, tools/probes/col_probe.cu);
    // contiguous: chunk c owns rows [c*RPC, (c+1)*RPC).  Both are fixed
    // assignments, so the summation order is fixed run to run.
    const bool il = L.col_il && NCH > 1;
    // FOP_COL_FIN=3: the slab's last chunk block streams no rows — it only waits for the others'
    // flag words and combines them, so the combine starts as soon as the slowest partial lands
    const bool pure_fin = L.col_fin == 3 && NCH > 2;
    const int64_t NCS = pure_fin ? NCH - 1 : NCH;   // chunks that stream rows
    const int64_t RSTEP = il ? NCS * (int64_t)L.gr : (int64_t)L.gr;   // between the U rows of a batch
    if (il) {
      o.l("const idx_t r0 = chunk * " + num(L.gr) + "u;");
      o.l(std::string("const idx_t r1 = ") + (pure_fin ? "chunk == " + num(NCH - 1) + "u ? 0u : " : "") + num(ROWS) +
          "u;");
    } else {
      o.l("const idx_t r0 = chunk * " + num(RPC) + "u;");
      o.l("const idx_t r1 = (r0 + " + num(RPC) + "u < " + num(ROWS) + "u) ? r0 + " + num(RPC) + "u : " + num(ROWS) +
          "u;");
    }
    const bool packed = !isMax && !ired && W % 2 == 0 && g_packed;
    // rows one lane accumulates in sequence; a long chain is summed with
    // compensation (Kahan), as in ROW_REDUCE
    const int64_t chain = (ROWS + NCS * (int64_t)L.gr - 1) / (NCS * (int64_t)L.gr);
    const bool kahan = !isMax && !ired && chain > 128;
    o.l("float acc[" + num(W) + "];");
    o.l("#pragma unroll");
    o.l("for (int e = 0; e < " + num(W) + "; ++e) acc[e] = " + init + ";");
    if (kahan) {
      o.l("float accc[" + num(W) + "];");
      o.l("#pragma unroll");
      o.l("for (int e = 0; e < " + num(W) + "; ++e) accc[e] = 0.f;");
    }
    if (packed) {
      o.l("u64 accp[" + num(W / 2) + "];");
      o.l("#pragma unroll");
      o.l("for (int p = 0; p < " + num(W / 2) + "; ++p) accp[p] = fop::pk1(0.f);");
      if (kahan) {
        o.l("u64 acccp[" + num(W / 2) + "];");
        o.l("#pragma unroll");
        o.l("for (int p = 0; p < " + num(W / 2) + "; ++p) acccp[p] = fop::pk1(0.f);");
      }
    }
    // Software pipeline (default): the U row loads of batch i+1 are issued as
    // raw words before batch i is converted and accumulated, so HBM requests
    // stay in flight across the accumulation instead of draining each batch.
    bool pipe = L.col_pipe && !FP;
    std::vector<int> wpv(L.loads.size(), 0);
    for (size_t k = 0; k < L.loads.size(); k++) {
      int64_t cv = C(L.loads[k], 0);
      int eb = es(L.loads[k].tensor);
      if (cv == 1 && W * eb >= 4 && L.load_cb[k] >= 4 && !written_here(L.loads[k].tensor)) wpv[k] = W * eb / 4;
      else if (cv != 0) pipe = false;
    }
    const int64_t BSTEP = RSTEP * U;
    // col_shift with the second chunk taken from the neighbouring lane (FOP_COL_SHFL=1, ablation): every
    // row's own chunk is loaded first, the whole batch in flight, then each row's window is assembled by
    // a shuffle inside the row's gv-lane segment; only the segment's last lane and a lane whose neighbour
    // has no vector load a second chunk.  Measured 1.7-3.4 TB/s on [65536,1001] f16 vs 3.2-3.9 for two
    // chunk loads per lane (the per-row window registers cost occupancy): off by default
    const bool shfl = L.col_shift && !pipe && L.gv > 1 && geometry_knob(L, "FOP_COL_SHFL", 0);
    if (shfl)
      o.l("const unsigned smask_ = " + std::string(L.gv == 32 ? "0xffffffffu" : "(" + num((1u << L.gv) - 1) +
          "u << ((threadIdx.x & 31u) & ~" + num(L.gv - 1) + "u))") + ";");
    auto batch_loads = [&](const std::string& rbase, const std::string& buf, const std::string& tg) {
      for (int u = 0; u < U; u++) {
        std::string t = tg + num(u);
        o.l("{");
        o.ind++;
        o.l("const idx_t rr = " + rbase + " + " + num(RSTEP * u) + "u;");
        o.l(FP ? "idx_t q = rr * " + num(FP) + "u;" : "idx_t q = rr;");   // fold: the group's first row
        std::vector<std::pair<int, std::string>> bits = cits;
        decompose("q", L.nsplit, (int)L.kl.size(), t, bits);
        for (size_t k = 0; k < L.loads.size(); k++) {
          if (!wpv[k]) continue;
          const Affine& a = L.loads[k];
          if (shfl) {
            const int esk = es(a.tensor);
            const std::string B = buf + num(k) + "_" + num(u), X = "X" + num(k) + "_" + num(u) + tg,
                              M = "M" + num(k) + "_" + num(u) + tg;
            const int64_t span = tensor_bytes(a.tensor) / esk;
            auto elementwise = [&](const std::string& dst, const std::string& from) {
              if (esk == 2)
                return "for (int e = 0; e < " + num(W) + "; ++e) if (" + from + " + e < (idx_t)" + num(span) + "ull) " +
                       dst + "[e >> 1] |= (u32)fop::ld16<" + pol(a, false) + ">(T" + num(a.tensor) + " + (u64)(" + from +
                       " + e) * 2u) << ((e & 1) * 16);";
              return "for (int e = 0; e < " + num(W) + "; ++e) if (" + from + " + e < (idx_t)" + num(span) +
                     "ull) fop::ldraw<4, " + pol(a, false) + ">(" + dst + " + e, T" + num(a.tensor) + " + (u64)(" + from +
                     " + e) * 4u);";
            };
            o.l("{");
            o.l("  const idx_t o_ = " + affine(a, bits) + ";");
            o.l("  " + M + " = (unsigned)(((u64)T" + num(a.tensor) + " + (u64)o_ * " + num(esk) + "u) & 15u) / " +
                num(esk) + "u;");
            o.l("  const idx_t a_ = o_ - " + M + ";");
            o.l("  #pragma unroll");
            o.l("  for (int w_ = 0; w_ < 4; ++w_) { " + B + "[w_] = 0u; " + X + "[w_] = 0u; }");
            o.l("  if (rr < r1) {");
            o.l("    if (a_ + " + num(W) + "u <= (idx_t)" + num(span) + "ull) fop::ldraw<16, " + pol(a, false) + ">(" + B +
                ", T" + num(a.tensor) + " + (u64)a_ * " + num(esk) + "u);");
            o.l("    else " + elementwise(B, "a_"));
            o.l("    if (" + M + " != 0u && (cv == " + num(L.gv - 1) + "u || j + 1u >= " + num(NVD) + "u)) {");
            o.l("      if (a_ + " + num(2 * W) + "u <= (idx_t)" + num(span) + "ull) fop::ldraw<16, " + pol(a, false) + ">(" +
                X + ", T" + num(a.tensor) + " + (u64)(a_ + " + num(W) + "u) * " + num(esk) + "u);");
            o.l("      else " + elementwise(X, "a_ + " + num(W) + "u"));
            o.l("    }");
            o.l("  }");
            o.l("}");
            continue;
          }
          if (L.col_shift) {
            // the row's W elements from the two aligned 16 B chunks around them,
            // funnel-shifted by the row's misalignment m_ (elements); a second
            // chunk past the tensor's end is read element-wise
            const int esk = es(a.tensor), epw = 4 / esk;
            const std::string B = buf + num(k) + "_" + num(u);
            const int64_t span = tensor_bytes(a.tensor) / esk;
            o.l("{");
            o.l("  const idx_t o_ = " + affine(a, bits) + ";");
            o.l("  const unsigned m_ = (unsigned)(((u64)T" + num(a.tensor) + " + (u64)o_ * " + num(esk) + "u) & 15u) / " +
                num(esk) + "u;");
            o.l("  const idx_t a_ = o_ - m_;");
            // (the second chunk could come from the next lane's first by a shuffle:
            // measured slower, 2978 vs 3888 GB/s on [65536,1001] — the shuffle waits
            // for each row's load, serialising the batch's latency)
            o.l("  u32 V_[8] = {0u, 0u, 0u, 0u, 0u, 0u, 0u, 0u};");
            o.l("  if (okc && rr < r1) {");
            // (the last row's last window may end past the tensor: read only its elements)
            o.l("    if (a_ + " + num(W) + "u <= (idx_t)" + num(span) + "ull) fop::ldraw<16, " + pol(a, false) +
                ">(V_, T" + num(a.tensor) + " + (u64)a_ * " + num(esk) + "u);");
            if (esk == 2)
              o.l("    else for (int e = 0; e < " + num(W) + "; ++e) if (a_ + e < (idx_t)" + num(span) +
                  "ull) V_[e >> 1] |= (u32)fop::ld16<" + pol(a, false) + ">(T" + num(a.tensor) + " + (u64)(a_ + e) * 2u) << "
                  "((e & 1) * 16);");
            else
              o.l("    else for (int e = 0; e < " + num(W) + "; ++e) if (a_ + e < (idx_t)" + num(span) + "ull) fop::ldraw<4, " +
                  pol(a, false) + ">(V_ + e, T" + num(a.tensor) + " + (u64)(a_ + e) * 4u);");
            o.l("    if (m_ != 0u) {");
            o.l("      if (a_ + " + num(2 * W) + "u <= (idx_t)" + num(span) + "ull) fop::ldraw<16, " + pol(a, false) +
                ">(V_ + 4, T" + num(a.tensor) + " + (u64)(a_ + " + num(W) + "u) * " + num(esk) + "u);");
            if (esk == 2)
              o.l("      else for (int e = 0; e < " + num(W) + "; ++e) if (a_ + " + num(W) + "u + e < (idx_t)" + num(span) +
                  "ull) V_[4 + (e >> 1)] |= (u32)fop::ld16<" + pol(a, false) + ">(T" + num(a.tensor) + " + (u64)(a_ + " +
                  num(W) + "u + e) * 2u) << ((e & 1) * 16);");
            else
              o.l("      else for (int e = 0; e < " + num(W) + "; ++e) if (a_ + " + num(W) + "u + e < (idx_t)" + num(span) +
                  "ull) fop::ldraw<4, " + pol(a, false) + ">(V_ + 4 + e, T" + num(a.tensor) + " + (u64)(a_ + " + num(W) +
                  "u + e) * 4u);");
            o.l("    }");
            o.l("  }");
            o.l("  const unsigned t_ = m_ / " + num(epw) + "u, s_ = (m_ % " + num(epw) + "u) * " + num(esk * 8) + "u;");
            o.l("  #pragma unroll");
            o.l("  for (int q = 0; q < 4; ++q) {   // word q of the window: V_[t_ + q .. t_ + q + 1] >> s_");
            o.l("    const u32 lo_ = t_ == 0u ? V_[q] : t_ == 1u ? V_[q + 1] : t_ == 2u ? V_[q + 2] : V_[q + 3];");
            o.l("    const u32 hi_ = t_ == 0u ? V_[q + 1] : t_ == 1u ? V_[q + 2] : t_ == 2u ? V_[q + 3] : V_[q + 4];");
            o.l("    " + B + "[q] = __funnelshift_r(lo_, hi_, s_);");
            o.l("  }");
            o.l("}");
            continue;
          }
          o.l("if (okc && rr < r1) fop::vload_words<" + std::string(dtn(d.t[a.tensor].dtype)) + ", " + num(W) + ", " +
              num(L.load_cb[k]) + ", " + pol(a, false) + ">(" + buf + num(k) + "_" + num(u) + ", " +
              ptr(a.tensor, affine(a, bits)) + ");");
        }
        o.ind--;
        o.l("}");
      }
    };
    if (pipe) {
      for (int u = 0; u < U; u++)
        for (size_t k = 0; k < L.loads.size(); k++)
          if (wpv[k]) o.l("u32 A" + num(k) + "_" + num(u) + "[" + num(wpv[k]) + "];");
      batch_loads("(r0 + rl)", "A", "_a");
    }
    o.l("#pragma unroll 1");
    o.l("for (idx_t r = r0 + rl; r < r1; r += " + num(BSTEP) + "u) {");
    o.ind++;
    if (pipe) {
      for (int u = 0; u < U; u++)
        for (size_t k = 0; k < L.loads.size(); k++)
          if (wpv[k]) o.l("u32 B" + num(k) + "_" + num(u) + "[" + num(wpv[k]) + "];");
      batch_loads("(r + " + num(BSTEP) + "u)", "B", "_b");
    } else {
      // the batch's vector loads stay raw words (half the registers of fp32
      // for 16-bit data) until they are accumulated
      for (int u = 0; u < U; u++)
        for (size_t k = 0; k < L.loads.size(); k++)
          if (wpv[k]) o.l("u32 A" + num(k) + "_" + num(u) + "[" + num(wpv[k]) + "];");
      if (shfl)
        for (int u = 0; u < U; u++)
          for (size_t k = 0; k < L.loads.size(); k++)
            if (wpv[k]) o.l("unsigned M" + num(k) + "_" + num(u) + "_a; u32 X" + num(k) + "_" + num(u) + "_a[4];");
      batch_loads("r", "A", "_a");
      if (shfl) {   // the batch is in flight: now each row's window (its own chunk + the neighbour's)
        for (int u = 0; u < U; u++)
          for (size_t k = 0; k < L.loads.size(); k++) {
            if (!wpv[k]) continue;
            const int esk = es(L.loads[k].tensor), epw = 4 / esk;
            const std::string A = "A" + num(k) + "_" + num(u), M = "M" + num(k) + "_" + num(u) + "_a",
                              X = "X" + num(k) + "_" + num(u) + "_a";
            o.l("{");
            o.l("  u32 V_[8];");
            o.l("  #pragma unroll");
            o.l("  for (int w_ = 0; w_ < 4; ++w_) { V_[w_] = " + A + "[w_]; V_[4 + w_] = __shfl_down_sync(smask_, " + A +
                "[w_], 1, " + num(L.gv) + "); }");
            o.l("  if (cv == " + num(L.gv - 1) + "u || j + 1u >= " + num(NVD) + "u) {");
            o.l("    #pragma unroll");
            o.l("    for (int w_ = 0; w_ < 4; ++w_) V_[4 + w_] = " + X + "[w_];");
            o.l("  }");
            o.l("  const unsigned t_ = " + M + " / " + num(epw) + "u, s_ = (" + M + " % " + num(epw) + "u) * " +
                num(esk * 8) + "u;");
            o.l("  #pragma unroll");
            o.l("  for (int q = 0; q < 4; ++q) {");
            o.l("    const u32 lo_ = t_ == 0u ? V_[q] : t_ == 1u ? V_[q + 1] : t_ == 2u ? V_[q + 2] : V_[q + 3];");
            o.l("    const u32 hi_ = t_ == 0u ? V_[q + 1] : t_ == 1u ? V_[q + 2] : t_ == 2u ? V_[q + 3] : V_[q + 4];");
            o.l("    " + A + "[q] = __funnelshift_r(lo_, hi_, s_);");
            o.l("  }");
            o.l("}");
          }
      }
    }
    std::vector<std::vector<std::pair<int, std::string>>> its(U);
    for (int u = 0; u < U; u++) {
      std::string t = "_" + num(u);
      o.l("const idx_t rr" + t + " = r + " + num(RSTEP * u) + "u;");
      o.l("const bool ok" + t + " = okc && rr" + t + " < r1;");
      o.l("idx_t q" + t + " = rr" + t + (FP ? " * " + num(FP) + "u;" : ";"));
      its[u] = cits;
      decompose("q" + t, L.nsplit, (int)L.kl.size(), t, its[u]);
      for (size_t k = 0; k < L.loads.size(); k++) {
        if (wpv[k]) continue;   // converted inside the accumulation below
        const Affine& a = L.loads[k];
        int64_t cv = C(a, 0);
        std::string off = affine(a, its[u]);
        std::string nm = "L" + num(k) + t;
        std::string dt = dtn(d.t[a.tensor].dtype);
        if (cv == 0) {
          o.l("float " + nm + " = 0.f;");
          o.l("if (ok" + t + ") " + nm + " = fop::sload<" + dt + ", " + pol(a, true) + ">(" + ptr(a.tensor, off) + ");");
        } else {
          o.l("float " + nm + "[" + num(W) + "];");
          if (cv == 1)
            o.l("if (ok" + t + ") fop::vload<" + dt + ", " + num(W) + ", " + num(L.load_cb[k]) + ", " +
                pol(a, false) + ">(" + nm + ", " + ptr(a.tensor, off) + ");");
          else
            o.l("if (ok" + t + ") for (int e = 0; e < " + num(W) + "; ++e) " + nm + "[e] = fop::sload<" + dt + ", " +
                pol(a, false) + ">(" + ptr(a.tensor, off + " + e * " + num(cv)) + ");");
        }
      }
    }
    for (int u = 0; u < U; u++) {
      std::string t = "_" + num(u);
      DagCtx c;
      c.tag = t;
      c.load_varies = [&](int k) { return C(L.loads[k], 0) != 0; };
      c.load = [&, t](int k, const std::string& e) {
        return C(L.loads[k], 0) != 0 ? "L" + num(k) + t + "[" + e + "]" : "L" + num(k) + t;
      };
      c.fwd = [&](int, const std::string&) { return std::string("0.f"); };
      c.scalar = [&](int) { return std::string("0.f"); };
      auto var = varies(x, c);
      o.l("if (ok" + t + ") {");
      o.ind++;
      for (size_t k = 0; k < L.loads.size(); k++)
        if (wpv[k]) {   // raw words -> fp32 only here, so one row's values are live at a time
          o.l("float L" + num(k) + t + "[" + num(W) + "];");
          o.l("fop::cvt_words<" + std::string(dtn(d.t[L.loads[k].tensor].dtype)) + ", " + num(W) + ">(L" + num(k) + t +
              ", A" + num(k) + t + ");");
        }
      emit_nodes(o, x, var, false, c);
      Sink sk;
      sk.scalar = [&](const std::string& v) { o.l("acc[e] = " + comb("acc[e]", v) + ";"); };
      if (packed) {
        sk.pair = [&](const std::string& v, const std::string& p) { o.l("accp[" + p + "] = fop::add2(accp[" + p + "], " + v + ");"); };
        sk.pair_fma = [&](const std::string& a, const std::string& b, const std::string& p) {
          o.l("accp[" + p + "] = fop::fma2(" + a + ", " + b + ", accp[" + p + "]);");
        };
      }
      if (kahan) {   // y = v - c; t = s + y; c = (t - s) - y; s = t
        sk.scalar = [&](const std::string& v) {
          o.l("{ const float y_ = __fsub_rn(" + v + ", accc[e]); const float t_ = __fadd_rn(acc[e], y_); accc[e] = "
              "__fsub_rn(__fsub_rn(t_, acc[e]), y_); acc[e] = t_; }");
        };
        if (packed) {
          auto kp = [&](const std::string& v, const std::string& p) {
            o.l("{ const u64 y_ = fop::sub2(" + v + ", acccp[" + p + "]); const u64 t_ = fop::add2(accp[" + p + "], y_); acccp[" +
                p + "] = fop::sub2(fop::sub2(t_, accp[" + p + "]), y_); accp[" + p + "] = t_; }");
          };
          sk.pair = kp;
          sk.pair_fma = [&, kp](const std::string& a, const std::string& b, const std::string& p) {
            kp("fop::mul2(" + a + ", " + b + ")", p);
          };
        }
      }
      emit_elems(o, x, var, c, W, sk);
      o.ind--;
      o.l("}");
    }
    if (pipe) {  // batch i+1 becomes the current batch
      for (int u = 0; u < U; u++)
        for (size_t k = 0; k < L.loads.size(); k++)
          if (wpv[k])
            o.l("#pragma unroll\nfor (int i = 0; i < " + num(wpv[k]) + "; ++i) A" + num(k) + "_" + num(u) + "[i] = B" +
                num(k) + "_" + num(u) + "[i];");
    }
    o.ind--;
    o.l("}");
    if (kahan) {   // running sums minus their compensations
      o.l("#pragma unroll");
      o.l("for (int e = 0; e < " + num(W) + "; ++e) acc[e] = __fsub_rn(acc[e], accc[e]);");
      if (packed) {
        o.l("#pragma unroll");
        o.l("for (int p = 0; p < " + num(W / 2) + "; ++p) accp[p] = fop::sub2(accp[p], acccp[p]);");
      }
    }
    if (packed) {  // pairs of partial sums back to one accumulator per column
      o.l("#pragma unroll");
      o.l("for (int p = 0; p < " + num(W / 2) + "; ++p) { float a0_, a1_; fop::upk(accp[p], a0_, a1_); "
          "acc[2 * p] = __fadd_rn(acc[2 * p], a0_); acc[2 * p + 1] = __fadd_rn(acc[2 * p + 1], a1_); }");
    }
    // Block combine over the row lanes, fixed order (deterministic): xor
    // butterflies over the row lanes that share a warp, then one thread per
    // (column, element) adds the NG warp-group results in order; the block's
    // sums end in red[0 .. SW).
    const int RPW = L.gv < 32 ? 32 / L.gv : 1;   // row lanes per warp
    const int NG = L.gr / RPW;                    // row groups (one per warp when gv < 32)
    auto tree = [&]() {
      if (RPW > 1) {
        o.l("#pragma unroll");
        o.l("for (int e = 0; e < " + num(W) + "; ++e) {");
        for (int m = L.gv; m < 32; m *= 2)
          o.l("  acc[e] = " + comb("acc[e]", "__shfl_xor_sync(0xffffffffu, acc[e], " + num(m) + ")") + ";");
        o.l("}");
      }
      if (NG == 1) {
        o.l("if (rl == 0u) {");
        o.l("  #pragma unroll");
        o.l("  for (int e = 0; e < " + num(W) + "; ++e) red[cv * " + num(W) + "u + e] = acc[e];");
        o.l("}");
        o.l("__syncthreads();");
        return;
      }
      o.l("if (rl % " + num(RPW) + "u == 0u) {");
      o.l("  #pragma unroll");
      o.l("  for (int e = 0; e < " + num(W) + "; ++e) red[(rl / " + num(RPW) + "u) * " + num(SW) + "u + cv * " + num(W) +
          "u + e] = acc[e];");
      o.l("}");
      o.l("__syncthreads();");
      o.l("for (unsigned t_ = tid; t_ < " + num(SW) + "u; t_ += " + num(L.block) + "u) {");
      o.l("  float s_ = red[t_];");
      o.l("  #pragma unroll");
      o.l("  for (int g = 1; g < " + num(NG) + "; ++g) s_ = " + comb("s_", "red[g * " + num(SW) + "u + t_]") + ";");
      o.l("  red[t_] = s_;");
      o.l("}");
      o.l("__syncthreads();");
    };
    tree();
    // Cross-GPU combine (opts.peer_world >= 1, fop.h peer groups; SURVEY
    // §8(e)).  The block holding this rank's slab sums in red[0 .. SW)
    // pushes each sum, packed with the run's epoch into one 64-bit word
    // (single-copy atomic, so the epoch doubles as the arrival flag: no
    // separate flag, fence or release round trip), into slot
    // [parity][rank][slab][e] of every rank's exchange buffer (NVLink stores
    // into peer memory), then polls its own buffer until every rank's words
    // carry this epoch and sums the world contributions in rank order — the
    // same order on every rank, so all ranks store identical bits.  The epoch
    // is a per-slab run counter kept in the local buffer (read at kernel
    // start); the two parities let a rank run ahead by one run without
    // overwriting words a slower rank has not read yet (it cannot get
    // further: its next wait needs that rank's next push).
    auto exchange = [&]() {
      if (!L.peer) return;
      const int PW = p.opts.peer_world;
      const PeerLayout pl = peer_layout(L, PW);
      const int64_t S = L.peer_slabs;
      const int NP = PW * SW;                         // words this block receives
      const int K = (NP + L.block - 1) / L.block;     // per thread
      const unsigned long long lim =
          (unsigned long long)(p.opts.peer_timeout_ms > 0 ? p.opts.peer_timeout_ms : 10000) * 1000000ull;
      const std::string base = num((int64_t)L.peer_off);
      const int spins = geometry_knob(L, "FOP_PEER_SPIN", 64);
      o.l("{");
      o.ind++;
      o.l("__shared__ float xv_[" + num(NP) + "];");
      if (!geometry_knob(L, "FOP_PEER_EP", 0)) {
        // one thread reads the run counter and shares it: thread 0 writes the
        // next value below, and a warp still to read the global counter would
        // see it (the epoch would be off by one on that warp only)
        o.l("__shared__ unsigned xeps_;");
        o.l("if (tid == 0u) xeps_ = ((volatile const unsigned*)(args.peer[args.rank] + " + base + "ull + " +
            num((int64_t)pl.epoch) + "ull))[slab];");
        o.l("__syncthreads();");
        o.l("const unsigned xep0_ = xeps_;");
      }
      o.l("const unsigned xe_ = xep0_ + 1u, xp_ = xe_ & 1u;");
      o.l("const u64* const xb_ = (const u64*)(args.peer[args.rank] + " + base + "ull);");
      o.l("if (tid == 0u) ((volatile unsigned*)(args.peer[args.rank] + " + base + "ull + " + num((int64_t)pl.epoch) +
          "ull))[slab] = xe_;");
      o.l("for (unsigned i_ = tid; i_ < " + num(NP) + "u; i_ += " + num(L.block) + "u) {");
      o.l("  const unsigned q_ = i_ / " + num(SW) + "u, e_ = i_ % " + num(SW) + "u;");
      o.l("  u64* d_ = (u64*)(args.peer[q_] + " + base + "ull) + ((xp_ * " + num(PW) + "u + args.rank) * " + num(S) +
          "ull + slab) * " + num(SW) + "u + e_;");
      o.l("  fop::st_relaxed_sys_u64(d_, ((u64)xe_ << 32) | __float_as_uint(red[e_]));");
      o.l("}");
      o.l("int xok_ = 1;");
      o.l("u64 xw_[" + num(K) + "];");
      o.l("#pragma unroll");
      o.l("for (int k = 0; k < " + num(K) + "; ++k) {   // every word requested before the first is checked");
      o.l("  const unsigned i_ = tid + k * " + num(L.block) + "u;");
      o.l("  if (i_ < " + num(NP) + "u) xw_[k] = fop::ld_relaxed_sys_u64(xb_ + ((xp_ * " + num(PW) + "u + i_ / " +
          num(SW) + "u) * " + num(S) + "ull + slab) * " + num(SW) + "u + i_ % " + num(SW) + "u);");
      o.l("}");
      o.l("#pragma unroll");
      o.l("for (int k = 0; k < " + num(K) + "; ++k) {");
      o.l("  const unsigned i_ = tid + k * " + num(L.block) + "u;");
      o.l("  if (i_ < " + num(NP) + "u) {");
      o.l("    const u64* a_ = xb_ + ((xp_ * " + num(PW) + "u + i_ / " + num(SW) + "u) * " + num(S) + "ull + slab) * " +
          num(SW) + "u + i_ % " + num(SW) + "u;");
      o.l("    if ((unsigned)(xw_[k] >> 32) != xe_ && !fop::wait_word(a_, xe_, xw_[k], " + std::to_string(lim) + "ull, " +
          num(spins) + ")) {");
      o.l("      xok_ = 0;");
      o.l("      atomicExch((unsigned*)(args.peer[args.rank] + " + num((int64_t)(p.peer_bytes - 16)) + "ull), 1u);");
      o.l("    }");
      o.l("    xv_[i_] = __uint_as_float((unsigned)xw_[k]);");
      o.l("  }");
      o.l("}");
      o.l("xok_ = __syncthreads_and(xok_);");
      o.l("if (rl == 0u) {");
      o.l("  #pragma unroll");
      o.l("  for (int e = 0; e < " + num(W) + "; ++e) {");
      o.l("    float s_ = " + init + ";");
      o.l("    for (unsigned q_ = 0; q_ < " + num(PW) + "u; ++q_) s_ = " +
          comb("s_", "xv_[q_ * " + num(SW) + "u + cv * " + num(W) + "u + e]") + ";");
      o.l("    red[cv * " + num(W) + "u + e] = xok_ ? s_ : __int_as_float(0x7fc00000);");
      o.l("  }");
      o.l("}");
      o.ind--;
      o.l("}");
    };
    auto final_store = [&]() {
      o.l("if (rl == 0u && okc) {");
      o.ind++;
      o.l("float res[" + num(W) + "];");
      o.l("#pragma unroll");
      o.l("for (int e = 0; e < " + num(W) + "; ++e) {");
      o.ind++;
      o.l("const float a_ = red[cv * " + num(W) + "u + e];");
      std::string r = fin_expr(o, x, "a_", "");
      o.l("res[e] = " + r + ";");
      o.ind--;
      o.l("}");
      std::string off = affine(x.write, cits);
      int64_t cw = C(x.write, 0);
      std::string dt = dtn(x.out_dtype);
      if (cw == 1 && L.store_cb[0] && L.col_shift && EV0 % W) {   // the last vector is partial
        o.l("if (iv + " + num(W) + "u <= " + num(EV0) + "u) fop::vstore<" + dt + ", " + num(W) + ", " +
            num(L.store_cb[0]) + ", fop::ST_DEFAULT>(" + ptr(x.write.tensor, off) + ", res);");
        o.l("else for (int e = 0; e < " + num(W) + "; ++e) if (iv + e < " + num(EV0) + "u) fop::sstore<" + dt + ">(" +
            ptr(x.write.tensor, off + " + e") + ", res[e]);");
      } else if (cw == 1 && L.store_cb[0])
        o.l("fop::vstore<" + dt + ", " + num(W) + ", " + num(L.store_cb[0]) + ", fop::ST_DEFAULT>(" +
            ptr(x.write.tensor, off) + ", res);");
      else
        o.l("for (int e = 0; e < " + num(W) + "; ++e) fop::sstore<" + dt + ">(" +
            ptr(x.write.tensor, off + " + e * " + num(cw)) + ", res[e]);");
      o.ind--;
      o.l("}");
    };
    // fold (col_fold = P): the slab's sums of wide columns iv + e go to F in
    // the workspace; the last slab to arrive adds, for each output column c,
    // F[g * E + c] over the P group rows g in order (fixed, deterministic) and
    // stores the E results element-wise
    auto fold_store = [&]() {
      const size_t FB = ((size_t)FP * (size_t)EV0 * sizeof(float) + 255) & ~size_t(255);
      o.l("{");
      o.ind++;
      // (fold_off is relative to the launch's own workspace region, which starts at
      // ws_off: tuning candidates and the narrow variant each have a region of their own)
      o.l("float* F_ = (float*)(args.ws + " + wsa((int64_t)L.fold_off) + ");");
      o.l("unsigned* fc_ = (unsigned*)(args.ws + " + wsa((int64_t)(L.fold_off + FB)) + ");");
      o.l("if (rl == 0u && okc) {");
      o.l("  #pragma unroll");
      o.l("  for (int e = 0; e < " + num(W) + "; ++e) F_[iv + e] = red[cv * " + num(W) + "u + e];");
      o.l("}");
      if (!L.col_acqrel) o.l("__threadfence();");
      o.l("__syncthreads();");
      o.l(std::string("if (tid == 0u) fold_flag = (") + (L.col_acqrel ? "fop::atom_add_acq_rel_gpu" : "atomicAdd") +
          "(fc_, 1u) == " + num(SVN - 1) + "u);");
      o.l("__syncthreads();");
      o.l("if (fold_flag) {");
      o.ind++;
      if (!L.col_acqrel) o.l("__threadfence();");
      o.l("for (unsigned c_ = tid; c_ < " + num(EV0) + "u; c_ += " + num(L.block) + "u) {");
      o.ind++;
      o.l("float a_ = " + init + ";");
      o.l("#pragma unroll");
      o.l("for (int g = 0; g < " + num(FP) + "; ++g) a_ = " + comb("a_", "__ldcg(&F_[g * " + num(EV0) + "u + c_])") + ";");
      // the R mod P rows after the last whole group, element-wise, in row order
      const int64_t RT = L.kl[1].extent, R0 = RT - RT % FP;
      if (R0 < RT) {
        o.l("#pragma unroll 1");
        o.l("for (unsigned tr_ = " + num(R0) + "u; tr_ < " + num(RT) + "u; ++tr_) {");
        o.ind++;
        const std::vector<std::pair<int, std::string>> tits = {{0, "(idx_t)c_"}, {1, "(idx_t)tr_"}};
        for (size_t k = 0; k < L.loads.size(); k++) {
          const Affine& a = L.loads[k];
          o.l("float L" + num(k) + "_t[1];");
          o.l("L" + num(k) + "_t[0] = fop::sload<" + std::string(dtn(d.t[a.tensor].dtype)) + ", " + pol(a, true) + ">(" +
              ptr(a.tensor, affine(a, tits)) + ");");
        }
        DagCtx tc;
        tc.tag = "_t";
        tc.load_varies = [](int) { return true; };
        tc.load = [&](int k, const std::string& e) { return "L" + num(k) + "_t[" + e + "]"; };
        tc.fwd = [&](int, const std::string&) { return std::string("0.f"); };
        tc.scalar = [&](int) { return std::string("0.f"); };
        auto tvar = varies(x, tc);
        emit_nodes(o, x, tvar, false, tc);
        Sink tsk;
        tsk.scalar = [&](const std::string& v) { o.l("a_ = " + comb("a_", v) + ";"); };
        emit_elems(o, x, tvar, tc, 1, tsk);
        o.ind--;
        o.l("}");
      }
      std::string r = fin_expr(o, x, "a_", "");
      std::vector<std::pair<int, std::string>> fc = {{0, "(idx_t)c_"}};
      o.l("fop::sstore<" + std::string(dtn(x.out_dtype)) + ">(" + ptr(x.write.tensor, affine(x.write, fc)) + ", " + r + ");");
      o.ind--;
      o.l("}");
      o.l("if (tid == 0u) *fc_ = 0u;");
      o.ind--;
      o.l("}");
      o.ind--;
      o.l("}");
    };
    if (NCH == 1) {
      exchange();
      if (FP) fold_store();
      else final_store();
    } else if (L.col_fin) {
      // Flag-word finalize (FOP_COL_FIN=1/2, ablations; 0 = the default below):
      // chunk blocks store their SW slab sums as 64-bit words (1 << 32 | fp32
      // bits) — one single-copy-atomic store carries the value and its arrival,
      // so no fence orders it — and ONE block per slab polls the words, adds
      // them in chunk order (deterministic) and clears them (the workspace is
      // zero again for the next run).  1: the slab's last chunk block (the last
      // dispatched) is that block, no atomic at all; 2: the last block to
      // arrive at a relaxed arrival counter (no fence before it).  Measured on
      // cfg4b: 27.2 us (1) vs 25.3 us for the fence + counter scheme — the
      // designated block is not the last to finish, so its poll loop sits on
      // the critical path (profiles/r02/sweep_r02_colfin.log).
      const int FM = L.col_fin == 3 ? 1 : L.col_fin;   // 3: mode 1 with a pure finalizer (no rows of its own)
      const std::string OWN = FM == 1 ? "c == " + num(NCH - 1) + "u" : "false";
      o.l("u64* partw = (u64*)(args.ws + " + wsa(0) + ");");
      o.l(std::string("if (rl == 0u") + (FM == 1 ? " && chunk != " + num(NCH - 1) + "u" : "") + ") {");
      o.l("  #pragma unroll");
      o.l("  for (int e = 0; e < " + num(W) + "; ++e) fop::st_relaxed_gpu_u64(&partw[(chunk * " + num(slabs) +
          "u + slab) * " + num(SW) + "u + cv * " + num(W) + "u + e], (1ull << 32) | __float_as_uint(red[cv * " + num(W) +
          "u + e]));");
      o.l("}");
      if (FM == 2) {
        size_t words = ((size_t)NCH * (size_t)slabs * (size_t)SW * 8 + 255) & ~size_t(255);
        o.l("unsigned* cnt = (unsigned*)(args.ws + " + wsa((int64_t)words) + ");");
        o.l("__syncthreads();");
        o.l("if (tid == 0u) last_flag = (atomicAdd(&cnt[slab], 1u) == " + num(NCH - 1) + "u);");
        o.l("__syncthreads();");
        o.l("if (last_flag) {");
      } else {
        o.l("if (chunk == " + num(NCH - 1) + "u) {");
      }
      o.ind++;
      o.l("#pragma unroll");
      o.l("for (int e = 0; e < " + num(W) + "; ++e) acc[e] = " + init + ";");
      const int64_t MAXIT = (NCH + L.gr - 1) / L.gr;
      const std::string NW_ = FM == 1 ? num(NCH - 1) : num(NCH);   // chunks whose words are read
      // every word this thread combines is requested before the first is
      // checked (one round trip); missing ones are re-polled as a batch
      o.l("u64 pw_[" + num(MAXIT) + "][" + num(W) + "];");
      o.l("#pragma unroll");
      o.l("for (int it = 0; it < " + num(MAXIT) + "; ++it) {");
      o.l("  const idx_t c = rl + it * " + num(L.gr) + "u;");
      o.l("  #pragma unroll");
      o.l("  for (int e = 0; e < " + num(W) + "; ++e) pw_[it][e] = c < " + NW_ +
          "u ? fop::ld_relaxed_gpu_u64(&partw[(c * " + num(slabs) + "u + slab) * " + num(SW) + "u + cv * " + num(W) +
          "u + e]) : 0ull;");
      o.l("}");
      o.l("unsigned long long t0_ = 0;");
      o.l("for (unsigned ns_ = 32u;;) {");
      o.l("  bool all_ = true;");
      o.l("  #pragma unroll");
      o.l("  for (int it = 0; it < " + num(MAXIT) + "; ++it)");
      o.l("    #pragma unroll");
      o.l("    for (int e = 0; e < " + num(W) + "; ++e) all_ &= rl + it * " + num(L.gr) + "u >= " + NW_ +
          "u || (unsigned)(pw_[it][e] >> 32) != 0u;");
      o.l("  if (all_) break;");
      o.l("  unsigned long long t_ = 0;");
      o.l("  asm volatile(\"mov.u64 %0, %%globaltimer;\" : \"=l\"(t_));");
      o.l("  if (t0_ == 0ull) t0_ = t_;");
      o.l("  else if (t_ - t0_ > 4000000000ull) break;   // a word that never arrives: NaN, not a hang");
      if (!geometry_knob(L, "FOP_COL_SPIN", 0)) o.l("  __nanosleep(ns_);");   // (1: spin without sleeping)
      o.l("  if (ns_ < 256u) ns_ *= 2u;");
      o.l("  #pragma unroll");
      o.l("  for (int it = 0; it < " + num(MAXIT) + "; ++it) {");
      o.l("    const idx_t c = rl + it * " + num(L.gr) + "u;");
      o.l("    #pragma unroll");
      o.l("    for (int e = 0; e < " + num(W) + "; ++e)");
      o.l("      if (c < " + NW_ + "u && (unsigned)(pw_[it][e] >> 32) == 0u) pw_[it][e] = "
          "fop::ld_relaxed_gpu_u64(&partw[(c * " + num(slabs) + "u + slab) * " + num(SW) + "u + cv * " + num(W) + "u + e]);");
      o.l("  }");
      o.l("}");
      o.l("#pragma unroll");
      o.l("for (int it = 0; it < " + num(MAXIT) + "; ++it) {");
      o.l("  const idx_t c = rl + it * " + num(L.gr) + "u;");
      o.l("  if (c < " + num(NCH) + "u) {");
      o.l("    #pragma unroll");
      o.l("    for (int e = 0; e < " + num(W) + "; ++e) {");
      o.l("      const float v_ = " + OWN + " ? red[cv * " + num(W) + "u + e] : ((unsigned)(pw_[it][e] >> 32) "
          "? __uint_as_float((unsigned)pw_[it][e]) : __int_as_float(0x7fc00000));");
      o.l("      acc[e] = " + comb("acc[e]", "v_") + ";");
      o.l("    }");
      o.l("  }");
      o.l("}");
      o.l("__syncthreads();   // every thread has read red[] before the tree reuses it");
      tree();
      exchange();
      final_store();
      o.l("for (int it = 0; it < " + num(MAXIT) + "; ++it) {   // leave the words zero for the next run");
      o.l("  const idx_t c = rl + it * " + num(L.gr) + "u;");
      o.l("  if (c < " + NW_ + "u) {");
      o.l("    #pragma unroll");
      o.l("    for (int e = 0; e < " + num(W) + "; ++e) fop::st_relaxed_gpu_u64(&partw[(c * " + num(slabs) + "u + slab) * " +
          num(SW) + "u + cv * " + num(W) + "u + e], 0ull);");
      o.l("  }");
      o.l("}");
      if (FM == 2) o.l("if (tid == 0u) cnt[slab] = 0u;");
      o.ind--;
      o.l("}");
    } else {
      size_t part = (size_t)NCH * (size_t)slabs * (size_t)SW * sizeof(float);
      part = (part + 255) & ~size_t(255);
      o.l("float* part = (float*)(args.ws + " + wsa(0) + ");");
      o.l("unsigned* cnt = (unsigned*)(args.ws + " + wsa((int64_t)part) + ");");
      o.l("if (rl == 0u) {");
      o.l("  #pragma unroll");
      o.l("  for (int e = 0; e < " + num(W) + "; ++e) part[(chunk * " + num(slabs) + "u + slab) * " + num(SW) +
          "u + cv * " + num(W) + "u + e] = red[cv * " + num(W) + "u + e];");
      o.l("}");
      // arrival: membar.gl in every thread + relaxed atomic (default), or one
      // acq_rel atomic after the barrier (FOP_COL_ACQREL=1, default)
      const bool acqrel = L.col_acqrel;
      if (!acqrel) o.l("__threadfence();");
      o.l("__syncthreads();");
      o.l(std::string("if (tid == 0u) last_flag = (") + (acqrel ? "fop::atom_add_acq_rel_gpu" : "atomicAdd") +
          "(&cnt[slab], 1u) == " + num(NCH - 1) + "u);");
      o.l("__syncthreads();");
      o.l("if (last_flag) {");
      o.ind++;
      if (!acqrel) o.l("__threadfence();");
      o.l("#pragma unroll");
      o.l("for (int e = 0; e < " + num(W) + "; ++e) acc[e] = " + init + ";");
      // every partial this thread combines is requested before the first is
      // used (one L2 round trip instead of one per chunk), then combined in
      // chunk order
      const int64_t MAXIT = (NCH + L.gr - 1) / L.gr;
      const bool v4 = W % 4 == 0 && MAXIT <= 8;
      if (v4) {
        o.l("float pv_[" + num(MAXIT) + "][" + num(W) + "];");
        o.l("#pragma unroll");
        o.l("for (int it = 0; it < " + num(MAXIT) + "; ++it) {");
        o.l("  const idx_t c = rl + it * " + num(L.gr) + "u;");
        o.l("  if (c < " + num(NCH) + "u) {");
        o.l("    const float* p_ = &part[(c * " + num(slabs) + "u + slab) * " + num(SW) + "u + cv * " + num(W) + "u];");
        o.l("    #pragma unroll");
        o.l("    for (int q = 0; q < " + num(W / 4) + "; ++q) asm volatile(\"ld.global.cg.v4.f32 {%0,%1,%2,%3}, [%4];\" : "
            "\"=f\"(pv_[it][4 * q]), \"=f\"(pv_[it][4 * q + 1]), \"=f\"(pv_[it][4 * q + 2]), \"=f\"(pv_[it][4 * q + 3]) : "
            "\"l\"(p_ + 4 * q));");
        o.l("  }");
        o.l("}");
        o.l("#pragma unroll");
        o.l("for (int it = 0; it < " + num(MAXIT) + "; ++it)");
        o.l("  if (rl + it * " + num(L.gr) + "u < " + num(NCH) + "u) {");
        o.l("    #pragma unroll");
        o.l("    for (int e = 0; e < " + num(W) + "; ++e) acc[e] = " + comb("acc[e]", "pv_[it][e]") + ";");
        o.l("  }");
      } else {
        o.l("for (idx_t c = rl; c < " + num(NCH) + "u; c += " + num(L.gr) + "u) {");
        o.l("  #pragma unroll");
        o.l("  for (int e = 0; e < " + num(W) + "; ++e) { float v_; const float* p_ = &part[(c * " + num(slabs) +
            "u + slab) * " + num(SW) + "u + cv * " + num(W) +
            "u + e]; asm volatile(\"ld.global.cg.f32 %0, [%1];\" : \"=f\"(v_) : \"l\"(p_)); acc[e] = " +
            comb("acc[e]", "v_") + "; }");
        o.l("}");
      }
      o.l("__syncthreads();");
      tree();
      exchange();
      if (FP) fold_store();
      else final_store();
      o.l("if (tid == 0u) cnt[slab] = 0u;");
      o.ind--;
      o.l("}");
    }
    footer();
  }
};

const char* class_name(int c) {
  switch (c) {
    case FOP_CLASS_TRANSPOSE: return "transpose";
    case FOP_CLASS_ROW_REDUCE: return "row_reduce";
    case FOP_CLASS_COL_REDUCE: return "col_reduce";
    default: return "ew";
  }
}

}  // namespace

std::string generate(const Plan& p, Launch& L, int launch_index) {
  {
    const char* e = std::getenv("FOP_PACKED");   // 0: scalar fp32 DAG evaluation (ablation)
    g_packed = !(e && *e == '0');
    g_approx16 = false;                           // set per statement by decide_fast()
    g_out_f16 = false;
    g_int = false;
  }
  Gen g(p, L);
  // 32-bit index arithmetic when every offset and work index fits
  int64_t maxv = L.work + L.grid * L.block * 8;
  for (int t = 0; t < p.desc.ntensors; t++) {
    int64_t span = 1;
    for (int r = 0; r < p.desc.t[t].rank; r++) span += (p.desc.t[t].shape[r] - 1) * p.desc.t[t].stride[r];
    maxv = std::max(maxv, span + 64);
  }
  g.idx = maxv < (int64_t(1) << 31) ? "unsigned" : "unsigned long long";
  L.name = std::string("fop_") + class_name(L.kclass) + (L.tma ? "_tma" : (L.tr_smem ? "_smem" : "")) + "_k" + std::to_string(launch_index) +
           (L.scalar_variant ? "_narrow" : "") + L.name_suffix;
  switch (L.kclass) {
    case FOP_CLASS_TRANSPOSE:
      if (L.tma) g.gen_transpose_tma();
      else if (L.tr_smem) g.gen_transpose_smem();
      else if (g.transpose_pipe_ok()) g.gen_transpose_pipe();
      else g.gen_transpose();
      break;
    case FOP_CLASS_ROW_REDUCE: g.gen_row(); break;
    case FOP_CLASS_COL_REDUCE: g.gen_col(); break;
    default:
      if (!L.seq.empty()) g.gen_ew_seq();
      else g.gen_ew();
  }
  L.src = g.o.s.str();
  return L.src;
}

}  // namespace fop
