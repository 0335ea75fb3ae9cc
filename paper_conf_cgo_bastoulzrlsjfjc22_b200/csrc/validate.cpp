// validate.cpp — row a1 (descriptor intake & validation) and the affine form
// of accesses used by row a2.
//
// The descriptor follows the paper's problem statement: statements over
// tensors with box iteration domains D_S(p) (§III-A) and
// access functions that are "either a constant or an affine form where only
// one loop iterator is present with coefficient 1".
#include <cmath>
#include <cstring>
#include <string>

#include "fop_internal.h"

namespace fop {

static std::string where(int s) { return "statement " + std::to_string(s) + ": "; }

Affine affine_of(const fop_desc& d, const fop_access& a) {
  Affine f;
  f.tensor = a.tensor;
  const fop_tensor& t = d.t[a.tensor];
  for (int r = 0; r < t.rank; r++) {
    f.base += t.stride[r] * a.offset[r];
    if (a.loop[r] >= 0) f.coef[a.loop[r]] += t.stride[r];
  }
  return f;
}

static bool in_stmt(const fop_stmt& st, int loop) {
  for (int k = 0; k < st.nloops; k++)
    if (st.loop[k] == loop) return true;
  return false;
}

bool empty_domain(const fop_desc& d, const fop_stmt& st) {
  for (int k = 0; k < st.nloops; k++)
    if (st.loop[k] >= 0 && st.loop[k] < FOP_MAX_LOOPS && d.extent[st.loop[k]] == 0) return true;
  return false;
}

static void check_access(const fop_desc& d, const fop_stmt& st, const fop_access& a, int s) {
  if (a.tensor < 0 || a.tensor >= d.ntensors) fail(FOP_E_INVALID, where(s) + "access tensor out of range");
  const fop_tensor& t = d.t[a.tensor];
  const bool empty = empty_domain(d, st);   // an empty box domain accesses nothing
  for (int r = 0; r < t.rank; r++) {
    int64_t lo = a.offset[r], hi = a.offset[r];
    if (a.loop[r] >= 0) {
      if (a.loop[r] >= d.nloops || !in_stmt(st, a.loop[r]))
        fail(FOP_E_INVALID, where(s) + "access uses a loop the statement does not iterate");
      hi += d.extent[a.loop[r]] - 1;
    } else if (a.loop[r] != -1) {
      fail(FOP_E_INVALID, where(s) + "access loop id must be >= 0 or -1");
    }
    if (!empty && (lo < 0 || hi >= t.shape[r]))
      fail(FOP_E_INVALID, where(s) + "access index range leaves the tensor (dim " + std::to_string(r) + ")");
  }
  for (int r = t.rank; r < FOP_MAX_RANK; r++)
    if (a.loop[r] != -1 && a.loop[r] != 0 && r >= t.rank) {
      // entries beyond the rank are ignored; tolerate zero-filled structs
    }
}

static void check_dag(const fop_node* n, int nn, int nacc, bool fin, int s) {
  int maxn = fin ? FOP_MAX_FIN : FOP_MAX_NODES;
  if (nn < 1 || nn > maxn) fail(FOP_E_INVALID, where(s) + "bad node count");
  for (int i = 0; i < nn; i++) {
    const fop_node& q = n[i];
    if (q.op < 0 || q.op >= FOP_OP__COUNT) fail(FOP_E_INVALID, where(s) + "unknown opcode");
    switch (q.op) {
      case FOP_OP_LOAD:
        if (fin || q.a < 1 || q.a >= nacc) fail(FOP_E_INVALID, where(s) + "LOAD must name a read access (1..nacc-1)");
        break;
      case FOP_OP_CONST:
        break;
      case FOP_OP_ACC:
        if (!fin) fail(FOP_E_INVALID, where(s) + "ACC is only allowed in a finalize DAG");
        break;
      case FOP_OP_ADD: case FOP_OP_SUB: case FOP_OP_MUL: case FOP_OP_DIV:
      case FOP_OP_MAX: case FOP_OP_MIN:
        if (q.b < 0 || q.b >= i) fail(FOP_E_INVALID, where(s) + "operand b is not an earlier node");
        [[fallthrough]];
      default:
        if (q.a < 0 || q.a >= i) fail(FOP_E_INVALID, where(s) + "operand a is not an earlier node");
        if (q.op == FOP_OP_CAST && (q.cvt < FOP_F32 || q.cvt > FOP_BF16))
          fail(FOP_E_INVALID, where(s) + "CAST target must be f32/f16/bf16");
    }
  }
}

void validate(const fop_desc& d) {
  if (d.nloops < 1 || d.nloops > FOP_MAX_LOOPS) fail(FOP_E_INVALID, "nloops must be 1..8");
  for (int l = 0; l < d.nloops; l++)
    if (d.extent[l] < 0) fail(FOP_E_INVALID, "loop " + std::to_string(l) + " has extent < 0");
  if (d.ntensors < 1 || d.ntensors > FOP_MAX_TENSORS) fail(FOP_E_INVALID, "ntensors must be 1..16");
  for (int i = 0; i < d.ntensors; i++) {
    const fop_tensor& t = d.t[i];
    std::string w = "tensor " + std::to_string(i) + ": ";
    if (t.rank < 0 || t.rank > FOP_MAX_RANK) fail(FOP_E_INVALID, w + "rank must be 0..8");
    if (t.dtype < FOP_F32 || t.dtype > FOP_I32) fail(FOP_E_INVALID, w + "unknown dtype");
    if (t.role < FOP_IN || t.role > FOP_TEMP) fail(FOP_E_INVALID, w + "unknown role");
    for (int r = 0; r < t.rank; r++) {
      if (t.shape[r] < 0) fail(FOP_E_INVALID, w + "shape must be >= 0");
      if (t.stride[r] < 0) fail(FOP_E_UNSUPPORTED, w + "negative strides are not supported");
    }
  }
  if (d.nstmts < 1 || d.nstmts > FOP_MAX_STMTS) fail(FOP_E_INVALID, "nstmts must be 1..8");
  for (int s = 0; s < d.nstmts; s++) {
    const fop_stmt& st = d.s[s];
    if (st.kind != FOP_ASSIGN && st.kind != FOP_REDUCE) fail(FOP_E_INVALID, where(s) + "unknown kind");
    if (st.kind == FOP_REDUCE && st.reduce_op != FOP_RED_SUM && st.reduce_op != FOP_RED_MAX)
      fail(FOP_E_INVALID, where(s) + "unknown reduce op");
    if (st.nloops < 1 || st.nloops > FOP_MAX_LOOPS) fail(FOP_E_INVALID, where(s) + "nloops must be 1..8");
    for (int k = 0; k < st.nloops; k++) {
      if (st.loop[k] < 0 || st.loop[k] >= d.nloops) fail(FOP_E_INVALID, where(s) + "loop id out of range");
      for (int q = 0; q < k; q++)
        if (st.loop[q] == st.loop[k]) fail(FOP_E_INVALID, where(s) + "loop listed twice");
    }
    if (st.nacc < 1 || st.nacc > FOP_MAX_ACC) fail(FOP_E_INVALID, where(s) + "nacc must be 1..8");
    for (int a = 0; a < st.nacc; a++) check_access(d, st, st.acc[a], s);
    check_dag(st.node, st.nnodes, st.nacc, false, s);
    if (st.kind == FOP_REDUCE) {
      if (st.nfin < 0 || st.nfin > FOP_MAX_FIN) fail(FOP_E_INVALID, where(s) + "bad finalize count");
      if (st.nfin > 0) check_dag(st.fin, st.nfin, 0, true, s);
    } else if (st.nfin != 0) {
      fail(FOP_E_INVALID, where(s) + "finalize DAG on an ASSIGN statement");
    }
    const fop_tensor& wt = d.t[st.acc[0].tensor];
    if (wt.role == FOP_IN) fail(FOP_E_INVALID, where(s) + "writes an IN tensor");
    if (st.kind == FOP_REDUCE)
      for (int a = 1; a < st.nacc; a++)
        if (st.acc[a].tensor == st.acc[0].tensor)
          fail(FOP_E_INVALID, where(s) + "a REDUCE statement may not read its own target");

    // Write-injectivity of the target over the domain (a write-write
    // pair is a dependence; within one ASSIGN that is a read-modify-write
    // over the missing loops, Fig. 2's Y — row N2).
    Affine w = affine_of(d, st.acc[0]);
    bool injective = true;   // no loop of extent > 1 leaves the target index unchanged
    bool has_red = false;    // some loop does not appear in the target index
    for (int k = 0; k < st.nloops; k++) {
      if (w.coef[st.loop[k]] == 0) {
        has_red = true;
        if (d.extent[st.loop[k]] > 1) injective = false;
      }
    }
    // distinct loops must not alias: require each loop to index exactly one
    // tensor dim and stride-0 dims to be absent from written tensors
    int uses[FOP_MAX_LOOPS] = {0};
    for (int r = 0; r < wt.rank; r++) {
      if (st.acc[0].loop[r] >= 0) {
        uses[st.acc[0].loop[r]]++;
        if (wt.stride[r] == 0 && wt.shape[r] > 1)
          fail(FOP_E_INVALID, where(s) + "written tensor has a broadcast (stride 0) dim: write-write conflict");
      }
    }
    for (int l = 0; l < d.nloops; l++)
      if (uses[l] > 1) fail(FOP_E_UNSUPPORTED, where(s) + "write access uses one loop in two dims");
    if (st.kind == FOP_ASSIGN && !injective) {
      // In-order read-modify-write (Fig. 2's Y): every iteration of the
      // loops the target ignores updates the same element, in lexicographic
      // order.  Supported when the statement reads its target only through
      // the write access itself (the running value) — then one thread owns
      // each target element and walks those loops sequentially.
      for (int a = 1; a < st.nacc; a++)
        if (st.acc[a].tensor == st.acc[0].tensor && !affine_of(d, st.acc[a]).same(w))
          fail(FOP_E_UNSUPPORTED, where(s) + "read-modify-write statement reads its target at another index");
    }
    if (st.kind == FOP_ASSIGN && injective) {
      // A read of the target at another index makes the statement a
      // recurrence (row N3): supported when the dependence is uniform — the
      // read maps every tensor dim to the same loop as the write, so the
      // distance vector is the constant offset difference.
      for (int a = 1; a < st.nacc; a++) {
        if (st.acc[a].tensor != st.acc[0].tensor) continue;
        for (int r = 0; r < wt.rank; r++)
          if (st.acc[a].loop[r] != st.acc[0].loop[r])
            fail(FOP_E_UNSUPPORTED, where(s) + "reads its target through another index map (non-uniform dependence)");
      }
    }
    if (st.kind == FOP_REDUCE && !has_red)
      fail(FOP_E_UNSUPPORTED, where(s) + "REDUCE statement without a reduction loop (use ASSIGN)");

    // Element types (reading R30).  A pure element move copies any
    // type.  A statement writing an i32 tensor is an INTEGER statement: it reads
    // i32 tensors only and its DAG is + - * max min neg abs relu and integral
    // constants on int32 values, wrapping modulo 2^32 (two's complement).  Any
    // other statement is a float statement and reads no i32 tensor.
    const bool move = st.kind == FOP_ASSIGN && st.nnodes == 1 && st.node[0].op == FOP_OP_LOAD &&
                      d.t[st.acc[st.node[0].a].tensor].dtype == wt.dtype;
    if (!move) {
      const bool integer = wt.dtype == FOP_I32;
      for (int a = 1; a < st.nacc; a++)
        if ((d.t[st.acc[a].tensor].dtype == FOP_I32) != integer)
          fail(FOP_E_INVALID, where(s) + (integer ? "integer statement reads a float tensor"
                                                   : "float statement reads an i32 tensor"));
      auto int_ok = [](const fop_node& q) {
        switch (q.op) {
          case FOP_OP_LOAD: case FOP_OP_ACC: case FOP_OP_ADD: case FOP_OP_SUB: case FOP_OP_MUL:
          case FOP_OP_MAX: case FOP_OP_MIN: case FOP_OP_NEG: case FOP_OP_ABS: case FOP_OP_RELU: return true;
          case FOP_OP_CONST: return q.imm == std::floor(q.imm) && q.imm >= -2147483648.0f && q.imm < 2147483648.0f;
        }
        return false;
      };
      for (int i = 0; i < st.nnodes; i++) {
        if (integer && !int_ok(st.node[i])) fail(FOP_E_INVALID, where(s) + "operation not defined on i32");
        if (!integer && st.node[i].op == FOP_OP_CAST && st.node[i].cvt == FOP_I32)
          fail(FOP_E_INVALID, where(s) + "cast to i32");
      }
      for (int i = 0; st.kind == FOP_REDUCE && i < st.nfin; i++) {
        if (integer && !int_ok(st.fin[i])) fail(FOP_E_INVALID, where(s) + "operation not defined on i32");
        if (!integer && st.fin[i].op == FOP_OP_CAST && st.fin[i].cvt == FOP_I32)
          fail(FOP_E_INVALID, where(s) + "cast to i32");
      }
    }
  }
}

}  // namespace fop
