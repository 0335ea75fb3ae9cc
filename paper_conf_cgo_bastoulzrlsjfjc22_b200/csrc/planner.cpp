// planner.cpp — rows a3 (Algorithm 2 + cost), a4 (vector width, divisibility,
// alignment), a5 (kernel class, mapping, launch plan) and a7 (fusion).
//
// Algorithm 2 (§V) builds, per statement, the influenced
// dimension scenario I_s: the shortest ordered list of innermost dimensions
// that minimises memory transactions, greedily from the innermost
// position outwards with the non-linear cost of P:338:
//     cost = w1|V_w| + w2|V_r| + w3/M + w4|C| + w5 * thread_term
// In the paper the scenarios become an influence constraint tree for isl
// (P:355); here the planner consumes them directly: the innermost loop of the
// best scenario carries the explicit vector type (A13), the following
// ones are mapped to consecutive threads for coalescing (goal (ii)) and
// the vectorised loop is never mapped to threads (the mapping-pass change,
// P:357).  Readings R1-R9 are listed in DESIGN.md §2.
#include <algorithm>
#include <cmath>
#include <cstring>
#include <string>

#include "fop_internal.h"

namespace fop {

// ======================================================================== a3

namespace {
struct Acc2 {
  bool store;
  int64_t stride[FOP_MAX_LOOPS];
};

std::vector<Acc2> stmt_accesses(const fop_desc& d, int s) {
  const fop_stmt& st = d.s[s];
  std::vector<Acc2> A;
  auto push = [&](const fop_access& a, bool store) {
    Affine f = affine_of(d, a);
    Acc2 x;
    x.store = store;
    for (int l = 0; l < FOP_MAX_LOOPS; l++) x.stride[l] = f.coef[l] < 0 ? -f.coef[l] : f.coef[l];
    A.push_back(x);
  };
  push(st.acc[0], true);
  if (st.kind == FOP_REDUCE) push(st.acc[0], false);  // accumulator read (Fig. 2's C)
  for (int a = 1; a < st.nacc; a++) push(st.acc[a], false);
  return A;
}

struct Score {
  double score;
  int64_t M;  // 0 = no non-zero stride
};

Score cost(const fop_desc& d, const std::vector<Acc2>& A, const fop_plan_opts& o, double L,
           int loop, bool innermost) {
  const double* w = o.w;
  int vw = 0, vr = 0;
  int64_t M = 0;
  for (const Acc2& a : A) {
    int64_t s = a.stride[loop];
    if (innermost && (s == 0 || s == 1)) (a.store ? vw : vr)++;          // R3
    if (s != 0 && (M == 0 || s < M)) M = s;                              // R2
  }
  int cn = 0;
  if (M != 0) {
    for (const Acc2& a : A) {
      if (o.readings & FOP_READING_R6_STRIDE1_C) cn += (M == 1 && a.stride[loop] == 1);  // R6
      else cn += (a.stride[loop] == M);
    }
  }
  double invM = M ? 1.0 / (double)M : 0.0;
  double N = (double)d.extent[loop];
  double F = N < L ? 1.0 : 0.0;
  double thread = (o.readings & FOP_READING_R1_THREAD_TERM) ? F * N / L : F * L / N;    // R1
  double sc = w[0] * vw + w[1] * vr + w[2] * invM + w[3] * cn + w[4] * thread;
  return {sc, M};
}

// best(): highest score, then smaller M, then the loop innermost in the input nest (R8)
int best(const fop_desc& d, int s, const std::vector<Acc2>& A, const fop_plan_opts& o, double L,
         const std::vector<int>& chosen, int depth) {
  const fop_stmt& st = d.s[s];
  int bl = -1;
  double bs = 0;
  int64_t bm = 0;
  int bp = -1;
  for (int pos = 0; pos < st.nloops; pos++) {
    int l = st.loop[pos];
    if (std::find(chosen.begin(), chosen.end(), l) != chosen.end()) continue;
    Score c = cost(d, A, o, L, l, depth == st.nloops);
    double m = c.M ? (double)c.M : INFINITY;
    double bmd = bm ? (double)bm : INFINITY;
    bool better = bl < 0 || c.score > bs || (c.score == bs && (m < bmd || (m == bmd && pos > bp)));
    if (better) {
      bl = l;
      bs = c.score;
      bm = c.M;
      bp = pos;
    }
  }
  return bl;
}

// Algorithm 2, lines 4-12 (optionally seeded with the innermost loop, R9)
std::vector<int> algorithm2(const fop_desc& d, int s, const std::vector<Acc2>& A,
                            const fop_plan_opts& o, int seed) {
  const fop_stmt& st = d.s[s];
  std::vector<int> I;  // innermost first while building
  int depth = st.nloops;
  double L = (double)o.thread_limit;   // L_s := L (R4)
  if (seed >= 0) {
    I.push_back(seed);
    L /= (double)d.extent[seed];         // R7
    depth--;
  }
  while ((int)I.size() < 3 && (int)I.size() < st.nloops) {
    int b = best(d, s, A, o, L, I, depth);
    I.push_back(b);                       // I_s := [b, I_s]
    L /= (double)d.extent[b];
    depth--;
  }
  std::reverse(I.begin(), I.end());      // outermost -> innermost
  return I;
}
}  // namespace

Scenarios rank_scenarios(const fop_desc& d, int s, const fop_plan_opts& o) {
  const fop_stmt& st = d.s[s];
  std::vector<Acc2> A = stmt_accesses(d, s);
  Scenarios out;
  struct Cand { double sc; int64_t M; int pos; int loop; };
  std::vector<Cand> c;
  for (int pos = 0; pos < st.nloops; pos++) {
    Score sc = cost(d, A, o, (double)o.thread_limit, st.loop[pos], true);
    out.inner_score[pos] = sc.score;
    c.push_back({sc.score, sc.M, pos, st.loop[pos]});
  }
  std::sort(c.begin(), c.end(), [](const Cand& a, const Cand& b) {
    if (a.sc != b.sc) return a.sc > b.sc;
    double ma = a.M ? (double)a.M : INFINITY, mb = b.M ? (double)b.M : INFINITY;
    if (ma != mb) return ma < mb;
    return a.pos > b.pos;
  });
  int n = std::min<int>((int)c.size(), std::max(1, std::min(o.max_scenarios, FOP_MAX_SCEN)));
  for (int k = 0; k < n; k++) {
    std::vector<int> I = algorithm2(d, s, A, o, c[k].loop);
    out.len[k] = (int)I.size();
    for (int q = 0; q < (int)I.size(); q++) out.loops[k][q] = I[q];
  }
  out.nscen = n;
  return out;
}

// ======================================================================== a5/a7

namespace {

bool same_access(const fop_desc& d, const fop_access& a, const fop_access& b) {
  return affine_of(d, a).same(affine_of(d, b));
}

int writer_before(const fop_desc& d, int s, int tensor) {
  for (int q = s - 1; q >= 0; q--)
    if (d.s[q].acc[0].tensor == tensor) return q;
  return -1;
}

bool reads_tensor(const fop_stmt& st, int t) {
  for (int a = 1; a < st.nacc; a++)
    if (st.acc[a].tensor == t) return true;
  return false;
}

bool loopset_equal(const fop_stmt& a, const fop_stmt& b) {
  if (a.nloops != b.nloops) return false;
  for (int i = 0; i < a.nloops; i++) {
    bool f = false;
    for (int j = 0; j < b.nloops; j++) f |= a.loop[i] == b.loop[j];
    if (!f) return false;
  }
  return true;
}

int innermost(const Plan& p, int s) {
  const Scenarios& sc = p.scen[s];
  return sc.loops[0][sc.len[0] - 1];
}

// A statement is inlined into its consumers (recomputed where used, never
// stored) when it is an ASSIGN to a TEMP tensor, every consumer reads it with
// exactly the producer's write access, and nothing between producer and
// consumers overwrites what the producer reads.  This is the register-level
// form of graph-kernel fusion's "remove intermediate allocations".
std::vector<bool> find_inlined(const fop_desc& d) {
  std::vector<bool> inl(d.nstmts, false);
  for (int p = 0; p < d.nstmts; p++) {
    const fop_stmt& ps = d.s[p];
    int T = ps.acc[0].tensor;
    if (ps.kind != FOP_ASSIGN || d.t[T].role != FOP_TEMP) continue;
    if (reads_tensor(ps, T)) continue;
    bool ok = true;
    int last = -1;
    for (int q = p + 1; q < d.nstmts && ok; q++) {
      const fop_stmt& qs = d.s[q];
      for (int a = 1; a < qs.nacc; a++)
        if (qs.acc[a].tensor == T) {
          if (!same_access(d, qs.acc[a], ps.acc[0])) ok = false;
          last = q;
        }
      if (qs.acc[0].tensor == T) break;  // a later writer ends p's live range
    }
    if (!ok || last < 0) continue;
    for (int q = p + 1; q <= last && ok; q++)
      for (int a = 1; a < ps.nacc; a++)
        if (d.s[q].acc[0].tensor == ps.acc[a].tensor) ok = false;
    inl[p] = ok;
  }
  return inl;
}

struct Group {
  std::vector<int> stmts;
  int kclass = FOP_CLASS_EW;
  int vec = -1;
  bool has_reduce = false;
  bool closed = false;   // a read-modify-write / recurrence launch: nothing joins it
  std::vector<int> seq;  // closed: loops carrying the statement's dependences, outer first
  bool rec = false;
  int scen_pick = 0, fallback = 0, coal = -1;
};

// read-modify-write ASSIGN (Fig. 2's Y): some loop of extent > 1 leaves the target index unchanged
bool is_rmw(const fop_desc& d, int s) {
  const fop_stmt& st = d.s[s];
  if (st.kind != FOP_ASSIGN) return false;
  Affine w = affine_of(d, st.acc[0]);
  for (int k = 0; k < st.nloops; k++)
    if (w.coef[st.loop[k]] == 0 && d.extent[st.loop[k]] > 1) return true;
  return false;
}

// reduction loops of a REDUCE statement: loops its target does not depend on
uint32_t red_loops(const fop_desc& d, int s) {
  Affine w = affine_of(d, d.s[s].acc[0]);
  uint32_t m = 0;
  for (int k = 0; k < d.s[s].nloops; k++)
    if (w.coef[d.s[s].loop[k]] == 0) m |= 1u << d.s[s].loop[k];
  return m;
}

}  // namespace

// ======================================================================== N3

std::vector<Dep> self_dependences(const fop_desc& d, int s) {
  const fop_stmt& st = d.s[s];
  std::vector<Dep> out;
  if (st.kind != FOP_ASSIGN) return out;
  auto lex_positive = [&](const Dep& D) {
    for (int k = 0; k < st.nloops; k++)
      if (D.dist[st.loop[k]] != 0) return D.dist[st.loop[k]] > 0;
    return false;
  };
  auto push = [&](Dep D) {
    for (const Dep& e : out)
      if (std::memcmp(e.dist, D.dist, sizeof D.dist) == 0 && e.anti == D.anti) return;
    out.push_back(D);
  };
  const fop_access& w = st.acc[0];
  if (is_rmw(d, s)) {
    // Fig. 2's Y: the target element is rewritten at every iteration of the
    // loops it ignores, so every lexicographically positive vector over those
    // loops is a dependence; e_i (carried by ignored loop i) and e_i - e_j
    // (i before j) represent them for a permutation test.
    Affine wa = affine_of(d, w);
    std::vector<int> ign;
    for (int k = 0; k < st.nloops; k++)
      if (wa.coef[st.loop[k]] == 0 && d.extent[st.loop[k]] > 1) ign.push_back(st.loop[k]);
    for (size_t i = 0; i < ign.size(); i++) {
      Dep D;
      D.dist[ign[i]] = 1;
      push(D);
    }
    for (size_t i = 0; i < ign.size(); i++)
      for (size_t j = i + 1; j < ign.size(); j++) {
        Dep D;
        D.dist[ign[i]] = 1;
        D.dist[ign[j]] = -1;
        push(D);
      }
    return out;
  }
  const fop_tensor& t = d.t[w.tensor];
  for (int a = 1; a < st.nacc; a++) {
    const fop_access& r = st.acc[a];
    if (r.tensor != w.tensor) continue;
    // written at iteration I, read at J: J_l = I_l + (w.offset - r.offset) on
    // the loop of every tensor dim (validate() guarantees the same loop map)
    Dep D;
    bool meets = true;
    for (int q = 0; q < t.rank; q++) {
      if (w.loop[q] < 0) {
        if (w.offset[q] != r.offset[q]) meets = false;   // constant dims never coincide
        continue;
      }
      D.dist[w.loop[q]] = w.offset[q] - r.offset[q];
    }
    bool zero = true;
    for (int l = 0; l < FOP_MAX_LOOPS; l++)
      if (D.dist[l] != 0) {
        zero = false;
        if (D.dist[l] >= d.extent[l] || -D.dist[l] >= d.extent[l]) meets = false;  // no pair inside the domain
      }
    if (!meets || zero) continue;
    if (!lex_positive(D)) {   // the read comes first: anti dependence from the read to the write
      for (int l = 0; l < FOP_MAX_LOOPS; l++) D.dist[l] = -D.dist[l];
      D.anti = true;
    }
    push(D);
  }
  return out;
}

bool schedule_legal(const std::vector<Dep>& deps, const std::vector<int>& seq, int vec_loop, int nloops,
                    const int* loops) {
  for (const Dep& D : deps) {
    // parallel loops (threads, and the vector lanes) must not carry anything
    for (int k = 0; k < nloops; k++) {
      int l = loops[k];
      bool in_seq = std::find(seq.begin(), seq.end(), l) != seq.end();
      if (!in_seq && D.dist[l] != 0) return false;
    }
    (void)vec_loop;
    // and each thread's sequential order must keep the source first
    int first = 0;
    for (int l : seq)
      if (D.dist[l] != 0) {
        first = D.dist[l] > 0 ? 1 : -1;
        break;
      }
    if (first <= 0) return false;
  }
  return true;
}

// Expand statement s's DAG for a launch: inlined producers are substituted,
// values of earlier statements in the same launch are forwarded.
static int expand(const Plan& p, Launch& L, const std::vector<bool>& inl, int s,
                  const std::vector<int>& in_launch, std::vector<XNode>& out, int node_idx,
                  std::vector<int>& memo, std::vector<int>& pmemo) {
  if (memo[node_idx] >= 0) return memo[node_idx];
  const fop_desc& d = p.desc;
  const fop_stmt& st = d.s[s];
  const fop_node& q = st.node[node_idx];
  XNode x;
  x.op = q.op;
  x.cvt = q.cvt;
  x.imm = q.imm;
  if (q.op == FOP_OP_LOAD) {
    const fop_access& a = st.acc[q.a];
    if (a.tensor == st.acc[0].tensor && is_rmw(d, s)) {  // read-modify-write: running value
      x.op = X_SELF;
      out.push_back(x);
      return memo[node_idx] = (int)out.size() - 1;
    }
    int w = writer_before(d, s, a.tensor);
    if (w >= 0 && inl[w]) {  // inlined producer: substitute its DAG once per consumer
      if (pmemo[w] < 0) {
        std::vector<int> m2(d.s[w].nnodes, -1);
        pmemo[w] = expand(p, L, inl, w, in_launch, out, d.s[w].nnodes - 1, m2, pmemo);
      }
      return memo[node_idx] = pmemo[w];
    }
    if (w >= 0) {
      for (size_t k = 0; k < in_launch.size(); k++)
        if (in_launch[k] == w) {
          x.op = d.s[w].kind == FOP_ASSIGN ? X_FWD : X_SCALAR;
          x.src = (int)k;
          out.push_back(x);
          return memo[node_idx] = (int)out.size() - 1;
        }
    }
    Affine f = affine_of(d, a);
    int idx = -1;
    for (size_t k = 0; k < L.loads.size(); k++)
      if (L.loads[k].same(f)) idx = (int)k;
    if (idx < 0) {
      L.loads.push_back(f);
      idx = (int)L.loads.size() - 1;
    }
    x.acc = idx;
    out.push_back(x);
    return memo[node_idx] = (int)out.size() - 1;
  }
  if (q.op != FOP_OP_CONST && q.op != FOP_OP_ACC) {
    x.a = expand(p, L, inl, s, in_launch, out, q.a, memo, pmemo);
    if (q.op >= FOP_OP_ADD && q.op <= FOP_OP_MIN) x.b = expand(p, L, inl, s, in_launch, out, q.b, memo, pmemo);
  }
  out.push_back(x);
  return memo[node_idx] = (int)out.size() - 1;
}

void plan_launches(Plan& p) {
  const fop_desc& d = p.desc;
  for (int s = 0; s < d.nstmts; s++) p.scen[s] = rank_scenarios(d, s, p.opts);
  std::vector<bool> inl = find_inlined(d);

  // ---- grouping (statement order; a group = one launch)
  std::vector<Group> groups;
  for (int s = 0; s < d.nstmts; s++) {
    if (inl[s] || empty_domain(d, d.s[s])) continue;   // an empty domain executes nothing
    const fop_stmt& st = d.s[s];
    int v = innermost(p, s);
    bool is_red = st.kind == FOP_REDUCE;
    bool row = is_red && (red_loops(d, s) >> v & 1u);
    bool joined = false;
    p.deps[s] = self_dependences(d, s);
    if (!p.deps[s].empty()) {
      // Row N3: the influence tree restricted to permutation
      // schedules whose loop nest, seen from one thread, is
      //     [parallel loops (threads; the coalescing loop innermost),
      //      dependence-carrying loops in a legal order, d_v (vector lanes)].
      // Siblings are the ranked scenarios.  Depth 0 of a scenario is
      // the vector loop: feasible when it carries no dependence (a parallel
      // dimension has zero dependence distance).  Deeper levels
      // must be the innermost sequential loops (any order the permutation
      // test accepts), then parallel loops; a scenario failing there keeps
      // only its vector constraint (the lower-priority looser variant).
      // With no feasible scenario the schedule is the uninfluenced one (P:202,
      // P:289): original order, no explicit vector type.
      const std::vector<Dep>& deps = p.deps[s];
      uint32_t carried = 0;
      for (const Dep& D : deps)
        for (int l = 0; l < FOP_MAX_LOOPS; l++)
          if (D.dist[l] != 0) carried |= 1u << l;
      Group g;
      g.stmts.push_back(s);
      g.kclass = FOP_CLASS_EW;
      g.closed = true;
      g.rec = !is_rmw(d, s);
      std::vector<int> seq0;   // carrying loops, original order (always legal)
      for (int k = 0; k < st.nloops; k++)
        if (carried >> st.loop[k] & 1u) seq0.push_back(st.loop[k]);
      const Scenarios& sc = p.scen[s];
      g.scen_pick = -1;
      for (int k = 0; k < sc.nscen && g.scen_pick < 0; k++) {
        const int m = sc.len[k];
        int vl = sc.loops[k][m - 1];
        if (carried >> vl & 1u) continue;                 // depth 0 infeasible: next sibling
        std::vector<int> inner;                           // scenario-fixed sequential loops, innermost first
        bool full = true;
        int coal = -1;
        for (int q = m - 2; q >= 0 && full; q--) {
          int l = sc.loops[k][q];
          bool cl = carried >> l & 1u;
          if (inner.size() < seq0.size()) {
            if (cl) inner.push_back(l);
            else full = false;                            // a parallel loop cannot sit inside a sequential one
          } else if (cl) {
            full = false;
          } else if (coal < 0) {
            coal = l;
          }
        }
        std::vector<int> order;
        for (int l : seq0)
          if (std::find(inner.begin(), inner.end(), l) == inner.end()) order.push_back(l);
        for (auto it = inner.rbegin(); it != inner.rend(); ++it) order.push_back(*it);
        if (!full || !schedule_legal(deps, order, vl, st.nloops, st.loop)) {
          full = false;                                   // looser variant: vector constraint only
          order = seq0;
          coal = -1;
          for (int q = m - 2; q >= 0 && coal < 0; q--)
            if (!(carried >> sc.loops[k][q] & 1u)) coal = sc.loops[k][q];
        }
        if (!schedule_legal(deps, order, vl, st.nloops, st.loop)) continue;
        g.vec = vl;
        g.seq = order;
        g.coal = coal;
        g.scen_pick = k;
        g.fallback = full ? 0 : 1;
      }
      if (g.scen_pick < 0) {
        g.seq = seq0;
        g.vec = -1;
        for (int k = st.nloops - 1; k >= 0 && g.vec < 0; k--)
          if (!(carried >> st.loop[k] & 1u)) g.vec = st.loop[k];
        g.fallback = g.vec >= 0 ? 2 : 3;
      }
      groups.push_back(g);
      continue;
    }
    if (!groups.empty() && !groups.back().closed) {
      Group& g = groups.back();
      const fop_stmt& g0 = d.s[g.stmts[0]];
      bool ok = g.kclass != FOP_CLASS_COL_REDUCE && g.kclass != FOP_CLASS_TRANSPOSE;
      ok = ok && loopset_equal(g0, st) && v == g.vec;
      if (ok && is_red) {
        ok = row;
        for (int q : g.stmts)
          if (d.s[q].kind == FOP_REDUCE && red_loops(d, q) != red_loops(d, s)) ok = false;
      }
      // reads of tensors produced inside the group must be forwardable
      for (int a = 1; ok && a < st.nacc; a++) {
        int w = writer_before(d, s, st.acc[a].tensor);
        if (w >= 0 && std::find(g.stmts.begin(), g.stmts.end(), w) != g.stmts.end())
          if (!same_access(d, st.acc[a], d.s[w].acc[0])) ok = false;
      }
      // no write to anything the group touches (WAR/WAW inside one launch)
      for (int q : g.stmts) {
        if (!ok) break;
        const fop_stmt& qs = d.s[q];
        for (int a = 0; a < qs.nacc; a++)
          if (qs.acc[a].tensor == st.acc[0].tensor) ok = false;
      }
      if (ok) {
        g.stmts.push_back(s);
        if (is_red) {
          g.has_reduce = true;
          g.kclass = FOP_CLASS_ROW_REDUCE;
        }
        joined = true;
      }
    }
    if (!joined) {
      Group g;
      g.stmts.push_back(s);
      g.vec = v;
      g.has_reduce = is_red;
      g.kclass = is_red ? (row ? FOP_CLASS_ROW_REDUCE : FOP_CLASS_COL_REDUCE) : FOP_CLASS_EW;
      groups.push_back(g);
    }
  }

  // ---- launches: expanded DAGs, load tables, class refinement
  p.launches.clear();
  for (const Group& g : groups) {
    Launch L;
    L.kclass = g.kclass;
    L.main_stmt = g.stmts[0];
    L.vec_loop = g.vec;
    for (int k = 0; k < d.s[L.main_stmt].nloops; k++) L.loops.push_back(d.s[L.main_stmt].loop[k]);
    std::vector<int> in_launch;
    for (int s : g.stmts) {
      L.mask |= 1u << s;
      const fop_stmt& st = d.s[s];
      XStmt x;
      x.stmt = s;
      x.kind = st.kind;
      x.redop = st.reduce_op;
      std::vector<int> memo(st.nnodes, -1), pmemo(d.nstmts, -1);
      // expand from the result only: unreachable nodes (and their loads) vanish
      x.result = expand(p, L, inl, s, in_launch, x.nodes, st.nnodes - 1, memo, pmemo);
      for (int i = 0; i < st.nfin; i++) {
        XNode f;
        f.op = st.fin[i].op;
        f.a = st.fin[i].a;
        f.b = st.fin[i].b;
        f.cvt = st.fin[i].cvt;
        f.imm = st.fin[i].imm;
        x.fin.push_back(f);
      }
      x.write = affine_of(d, st.acc[0]);
      x.out_dtype = d.t[st.acc[0].tensor].dtype;
      x.store = true;
      x.move = st.kind == FOP_ASSIGN && x.nodes[x.result].op == FOP_OP_LOAD &&
               d.t[L.loads[x.nodes[x.result].acc].tensor].dtype == x.out_dtype;
      L.stmts.push_back(x);
      in_launch.push_back(s);
    }
    // forwarded values: consumed by a later statement of the launch
    for (auto& x : L.stmts)
      for (auto& n : x.nodes)
        if (n.op == X_FWD || n.op == X_SCALAR) L.stmts[n.src].fwd = true;
    // TEMP results forwarded inside the launch and not read by later launches need no store
    for (auto& x : L.stmts) {
      int T = x.write.tensor;
      if (d.t[T].role != FOP_TEMP) continue;
      bool later = false;
      int last = -1;
      for (int s : g.stmts) last = std::max(last, s);
      for (int q = last + 1; q < d.nstmts; q++)
        if (reads_tensor(d.s[q], T)) later = true;
      if (!later && x.fwd) x.store = false;
    }

    // TRANSPOSE: single ASSIGN whose largest load is strided along d_v but
    // contiguous along another loop (store-contiguous != load-contiguous)
    if (L.kclass == FOP_CLASS_EW && L.stmts.size() == 1 && L.stmts[0].write.coef[L.vec_loop] == 1) {
      int64_t best_bytes = -1;
      for (size_t k = 0; k < L.loads.size(); k++) {
        const Affine& f = L.loads[k];
        int64_t cv = f.coef[L.vec_loop];
        if (cv == 0 || cv == 1) continue;
        int rl = -1;
        for (int l : L.loops)
          if (l != L.vec_loop && f.coef[l] == 1) rl = l;
        if (rl < 0) continue;
        int64_t bytes = esize(d.t[f.tensor].dtype);
        for (int r = 0; r < d.t[f.tensor].rank; r++) bytes *= d.t[f.tensor].shape[r];
        if (bytes > best_bytes) {
          best_bytes = bytes;
          L.kclass = FOP_CLASS_TRANSPOSE;
          L.read_loop = rl;
          L.trans_load = (int)k;
        }
      }
    }
    // coalescing loop: next loop of the main scenario (goal (ii))
    const Scenarios& sc = p.scen[L.main_stmt];
    L.coal_loop = sc.len[0] >= 2 ? sc.loops[0][sc.len[0] - 2] : -1;
    if (g.closed) {  // read-modify-write / recurrence: dependence-carrying loops run in order inside each thread
      L.kclass = FOP_CLASS_EW;
      L.read_loop = -1;
      L.trans_load = -1;
      L.seq = g.seq;
      L.rec = g.rec;
      L.scen_pick = g.scen_pick;
      L.fallback = g.fallback;
      L.force_w1 = g.fallback >= 2;
      L.coal_loop = g.coal;
      const fop_stmt& st = d.s[L.main_stmt];
      if (g.vec < 0) {
        // fully sequential: a placeholder vector loop of extent 1 (an id the
        // statement does not use, so every access has coefficient 0 on it)
        for (int id = 0; id < FOP_MAX_LOOPS && L.vec_loop < 0; id++) {
          bool used = false;
          for (int k = 0; k < st.nloops; k++) used |= st.loop[k] == id;
          if (!used) L.vec_loop = id;
        }
        if (L.vec_loop < 0) fail(FOP_E_UNSUPPORTED, "fully sequential statement over 8 loops");
        L.virt_vec = true;
      }
      if (L.rec) {
        // reads of the target 1..4 iterations back along the innermost
        // sequential loop come from registers (this thread's last stores)
        L.fwd_dist.assign(L.loads.size(), 0);
        const fop_access& w = st.acc[0];
        const fop_tensor& t = d.t[w.tensor];
        int sl = g.seq.back();
        for (int a = 1; a < st.nacc; a++) {
          const fop_access& r = st.acc[a];
          if (r.tensor != w.tensor) continue;
          int64_t dist[FOP_MAX_LOOPS] = {0};
          bool ok = true;
          for (int q = 0; q < t.rank; q++) {
            if (w.loop[q] < 0) ok = ok && w.offset[q] == r.offset[q];
            else dist[w.loop[q]] = w.offset[q] - r.offset[q];
          }
          for (int l = 0; l < FOP_MAX_LOOPS; l++)
            if (l != sl && dist[l] != 0) ok = false;
          if (!ok || dist[sl] < 1 || dist[sl] > 4) continue;
          Affine f = affine_of(d, r);
          for (size_t k = 0; k < L.loads.size(); k++)
            if (L.loads[k].same(f)) L.fwd_dist[k] = (int)dist[sl];
        }
      }
    }
    p.launches.push_back(L);
  }

  // ---- workspace: TEMP tensors stored by one launch and read by another
  p.temp_off.assign(d.ntensors, -1);
  size_t ws = 0;
  for (auto& L : p.launches)
    for (auto& x : L.stmts) {
      int T = x.write.tensor;
      if (d.t[T].role == FOP_TEMP && x.store && p.temp_off[T] < 0) {
        int64_t span = 1;
        for (int r = 0; r < d.t[T].rank; r++) span += (d.t[T].shape[r] - 1) * d.t[T].stride[r];
        ws = (ws + 255) & ~size_t(255);
        p.temp_off[T] = (int64_t)ws;
        ws += (size_t)span * esize(d.t[T].dtype);
      }
    }
  for (auto& L : p.launches) {
    finalize_launch_geometry(p, L);
    if (L.ws_bytes) {
      ws = (ws + 255) & ~size_t(255);
      L.ws_off = ws;
      ws += L.ws_bytes;
    }
  }
  p.ws_bytes = ws;

  // ---- multi-GPU (opts.peer_world >= 1; fop.h): a REDUCE
  // statement whose reduction loops include the loop split across the peer
  // group combines the ranks' partial results in its COL_REDUCE epilogue.
  // Only the final result may be exchanged: a statement that consumes it in
  // the same operator would read a partial value.
  p.peer_bytes = 0;
  if (p.opts.peer_world >= 1) {
    const int PW = p.opts.peer_world, PL = p.opts.peer_loop;
    if (PW > FOP_MAX_PEERS) fail(FOP_E_INVALID, "peer_world exceeds FOP_MAX_PEERS");
    if (PL < 0 || PL >= d.nloops) fail(FOP_E_INVALID, "peer_loop is not a loop of the operator");
    for (int s = 0; s < d.nstmts; s++) {
      bool iterates = false;
      for (int k = 0; k < d.s[s].nloops; k++) iterates |= d.s[s].loop[k] == PL;
      if (!iterates || empty_domain(d, d.s[s])) continue;
      const int T = d.s[s].acc[0].tensor;
      if (d.s[s].kind != FOP_REDUCE || !(red_loops(d, s) >> PL & 1u)) continue;
      if (inl[s])
        fail(FOP_E_UNSUPPORTED, "statement " + std::to_string(s) + " reduces over the peer loop but is fused into a consumer");
      for (int q = s + 1; q < d.nstmts; q++)
        for (int a = 1; a < d.s[q].nacc; a++)
          if (d.s[q].acc[a].tensor == T)
            fail(FOP_E_UNSUPPORTED, "statement " + std::to_string(q) + " consumes the cross-GPU reduction of statement " +
                                        std::to_string(s) + " inside the same operator");
      Launch* X = nullptr;
      for (auto& L : p.launches)
        if (L.main_stmt == s) X = &L;
      if (!X || X->kclass != FOP_CLASS_COL_REDUCE || X->stmts.size() != 1)
        fail(FOP_E_UNSUPPORTED, "statement " + std::to_string(s) +
                                    ": a reduction over the peer loop must be a COL_REDUCE launch of its own (the "
                                    "vector loop parallel)");
      X->peer = true;
    }
    size_t off = 0;
    for (auto& L : p.launches) {
      if (!L.peer) continue;
      int64_t svn = (L.kl[0].extent / L.width + L.gv - 1) / L.gv;
      for (int k = 1; k < L.nsplit; k++) svn *= L.kl[k].extent;
      L.peer_slabs = svn;
      L.peer_off = off;
      off += peer_layout(L, PW).total;
    }
    p.peer_bytes = off ? off + 16 : 0;   // + error word; no exchanging launch: no buffer
  }
}

}  // namespace fop
