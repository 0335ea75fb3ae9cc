// geometry.cpp — rows a4 (vector width, divisibility, alignment) and a5
// (mapping and launch geometry) for one launch.
//
// a4: the paper's vector dimension must be innermost, of size 2 or 4, with
// accesses "aligned and either constant or contiguous", carried by
// 64/128-bit transactions.  On B200 the width is byte based: the
// narrowest element type among the accesses contiguous along d_v gets a full
// max_vec_bytes vector (16 B = LDG/STG.128, or 32 B = LDG/STG.256 on
// sm_100a); wider types move several chunks.  Divisibility: the vector
// loop's extent must be a multiple of W (halve W otherwise — down to 1, the
// paper's "novec").  Alignment: each access gets the largest chunk
// its base and the other loops' strides keep aligned ("we may mix vector
// types with scalar types"); base pointers are checked at fop_run.
//
// a5: "dimensions marked as vectorized" are not mapped to blocks/threads
// — each thread owns W consecutive iterations of d_v; consecutive
// threads take consecutive vectors, then the next loops of the thread order
// (coalescing, goal (ii) of P:297).  Loops that are contiguous for every
// access are collapsed (a B200 step beyond the paper).
#include <algorithm>
#include <cstdlib>
#include <numeric>
#include <string>

#include "fop_internal.h"

namespace fop {

namespace {

std::vector<const Affine*> all_accesses(const Launch& L) {
  std::vector<const Affine*> v;
  for (const auto& a : L.loads) v.push_back(&a);
  for (const auto& x : L.stmts) v.push_back(&x.write);
  return v;
}

// order a set of loops innermost first
std::vector<int> order_rest(const Plan& p, const Launch& L, std::vector<int> rest) {
  const fop_stmt& st = p.desc.s[L.main_stmt];
  auto pos = [&](int l) {
    for (int k = 0; k < st.nloops; k++)
      if (st.loop[k] == l) return k;
    return -1;
  };
  const Affine& w = L.stmts[0].write;
  if (p.opts.coalesce_order == FOP_ORDER_MEMORY) {
    // memory order of the write; loops the write does not use (the reduction
    // loops of COL) are ordered by the first load instead
    auto key = [&](int l) {
      if (w.coef[l] != 0 || L.loads.empty()) return w.coef[l];
      return L.loads[0].coef[l];
    };
    std::stable_sort(rest.begin(), rest.end(), [&](int a, int b) {
      int64_t ca = key(a), cb = key(b);
      if (ca != cb) return ca < cb;
      return pos(a) > pos(b);
    });
    return rest;
  }
  // FOP_ORDER_PAPER: the best scenario (outer -> inner) gives the innermost
  // loops after d_v; loops outside the scenario follow, innermost first
  std::vector<int> out;
  const Scenarios& sc = p.scen[L.main_stmt];
  for (int q = sc.len[0] - 1; q >= 0; q--) {
    int l = sc.loops[0][q];
    if (std::find(rest.begin(), rest.end(), l) != rest.end()) out.push_back(l);
  }
  for (int k = st.nloops - 1; k >= 0; k--) {
    int l = st.loop[k];
    if (std::find(rest.begin(), rest.end(), l) != rest.end() &&
        std::find(out.begin(), out.end(), l) == out.end())
      out.push_back(l);
  }
  return out;
}

// collapse adjacent loops of a segment: merge l into K iff for every access
// coef(l) == coef(K.members[0]) * K.extent
void collapse_into(const Plan& p, const std::vector<const Affine*>& acc, const std::vector<int>& seg,
                   std::vector<KLoop>& out) {
  for (size_t i = 0; i < seg.size(); i++) {
    int l = seg[i];
    if (i > 0) {
      KLoop& K = out.back();
      bool ok = true;
      for (const Affine* a : acc)
        if (a->coef[l] != a->coef[K.members[0]] * K.extent) ok = false;
      if (ok) {
        K.members.push_back(l);
        K.extent *= p.desc.extent[l];
        continue;
      }
    }
    KLoop K;
    K.members.push_back(l);
    K.extent = p.desc.extent[l];
    out.push_back(K);
  }
}

int64_t pow2_ceil(int64_t x);
int pow2_floor(int64_t x) {
  int r = 1;
  while ((int64_t)r * 2 <= x) r *= 2;
  return r;
}
int64_t pow2_ceil(int64_t x) {
  int64_t r = 1;
  while (r < x) r *= 2;
  return r;
}

// largest power-of-two chunk (bytes) <= cap keeping `a` aligned, given the
// kernel loops other than `vk` (whose steps are multiples of the vector)
int chunk_bytes(const Plan& p, const Launch& L, const Affine& a, int vk, int cap) {
  int es = esize(p.desc.t[a.tensor].dtype);
  int cb = cap;
  auto fits = [&](int64_t elems) { return ((elems * es) % cb) == 0; };
  while (cb > es) {
    bool ok = fits(a.base);
    for (int k = 0; k < (int)L.kl.size() && ok; k++)
      if (k != vk) ok = fits(a.coef[L.kl[k].members[0]]);
    if (ok) break;
    cb /= 2;
  }
  return std::max(cb, es);
}

int64_t coef(const Launch& L, const Affine& a, int k) { return a.coef[L.kl[k].members[0]]; }

}  // namespace

// A geometry knob: the launch's variant overrides first (auto-tuning), then
// the environment (manual sweeps, tools/sweep.py), then the default rule.
int geometry_knob(const Launch& L, const char* name, int dflt) {
  for (const auto& kv : L.knobs)
    if (kv.first == name) return kv.second;
  const char* e = std::getenv(name);
  return e && *e ? std::atoi(e) : dflt;
}

// Candidate geometries the run-time auto-tuner times (the paper's tile sizes
// come from auto-tuners too).  Entry 0 is the default rule.  Chosen
// from the measured sweeps (profiles/sweep_r01_*.log): streaming kernels
// prefer few threads with many vectors in flight, ALU-heavy ones more threads.
std::vector<std::vector<std::pair<std::string, int>>> tuning_variants(const Launch& L, int /*sms*/) {
  typedef std::vector<std::pair<std::string, int>> K;
  std::vector<K> v = {K{}};
  switch (L.kclass) {
    case FOP_CLASS_EW:
      if (!L.seq.empty()) break;
      v.push_back({{"FOP_EW_U", 4}, {"FOP_EW_MINB", 2}, {"FOP_SMEM_TABLES", 0}});
      v.push_back({{"FOP_EW_U", 2}, {"FOP_EW_MINB", 4}, {"FOP_SMEM_TABLES", 0}});
      v.push_back({{"FOP_EW_U", 2}, {"FOP_EW_MINB", 4}});
      v.push_back({{"FOP_EW_U", 1}, {"FOP_EW_MINB", 8}});
      v.push_back({{"FOP_EW_U", 4}, {"FOP_EW_MINB", 3}});
      // 32-byte vectors (LDG/STG.256), 8 warps per SM with 4 vectors in flight each:
      // cfg2 6112 -> 6525 GB/s (profiles/r02/sweep_r02_vec32.log)
      v.push_back({{"FOP_VEC_BYTES", 32}, {"FOP_EW_U", 4}, {"FOP_EW_MINB", 1}});
      v.push_back({{"FOP_VEC_BYTES", 32}, {"FOP_EW_U", 4}, {"FOP_EW_MINB", 2}, {"FOP_BLOCK", 128}});
      break;
    case FOP_CLASS_TRANSPOSE:
      if (L.tma) {   // TMA tiles: 2 warps per CTA x 2 CTAs per SM next to the default 4 x 1,
                     // and the register tiles (ahead where the tuner's cold launch says so)
        v.push_back({{"FOP_TR_TMA_WARPS", 2}, {"FOP_TR_TMA_MINB", 2}});
        v.push_back({{"FOP_TR_TMA", 0}});
        v.push_back({{"FOP_TR_TMA", 0}, {"FOP_BLOCK", 256}, {"FOP_TR_MINB", 1}});
        v.push_back({{"FOP_TR_TMA", 0}, {"FOP_BLOCK", 128}, {"FOP_TR_MINB", 2}});
        break;
      }
      if (L.tr_smem) {
        v.push_back({{"FOP_TR_SMEM_MINB", 2}});
        v.push_back({{"FOP_TR_SMEM_MINB", 6}});
        v.push_back({{"FOP_TR_SMEM_BYTES", 16384}, {"FOP_TR_SMEM_MINB", 8}});
        break;
      }
      v.push_back({{"FOP_BLOCK", 256}, {"FOP_TR_MINB", 1}});                       // round 1's default
      v.push_back({{"FOP_BLOCK", 128}, {"FOP_TR_MINB", 2}});
      v.push_back({{"FOP_BLOCK", 32}, {"FOP_TR_MINB", 8}});
      // round 1's candidates (more warps per SM: f32 data, 2-D transposes, C = 96)
      v.push_back({{"FOP_BLOCK", 256}, {"FOP_TR_U", 1}, {"FOP_TR_MINB", 2}});
      v.push_back({{"FOP_BLOCK", 256}, {"FOP_TR_U", 2}, {"FOP_TR_MINB", 2}});
      v.push_back({{"FOP_BLOCK", 256}, {"FOP_TR_U", 1}, {"FOP_TR_MINB", 3}});
      // 32-byte stores along d_v over 16-byte loads along d_r (cfg3 6088 GB/s at 2 x 128 threads)
      v.push_back({{"FOP_VEC_BYTES", 32}, {"FOP_TR_WR_BYTES", 16}, {"FOP_TR_U", 1}, {"FOP_BLOCK", 128},
                   {"FOP_TR_MINB", 2}});
      break;
    case FOP_CLASS_ROW_REDUCE:
      if (L.row_g > 1) {   // few long rows: neighbouring warps-per-row counts
        v.push_back({{"FOP_ROW_G", L.row_g / 2}});
        if (L.row_g < 32) v.push_back({{"FOP_ROW_G", L.row_g * 2}});
        if (L.row_q > 1) {   // rows spread over clusters: more CTAs per row / more warps per SM
          v.push_back({{"FOP_ROW_Q", 8}, {"FOP_ROW_G", 16}});
          v.push_back({{"FOP_ROW_Q", 8}, {"FOP_ROW_MINB", 4}});
        }
        break;
      }
      v.push_back({{"FOP_ROW_MINB", 2}});
      v.push_back({{"FOP_ROW_MINB", 4}});
      v.push_back({{"FOP_BLOCK", 128}, {"FOP_ROW_MINB", 6}});
      // two rows prefetched per warp at 2 CTAs/SM: BERT LayerNorm 36.4 -> 30.4 us untuned
      // (cfg4a: 23.0 vs 20.9, profiles/r02/sweep_r02_rowpf.log)
      if (L.row_p == 1) v.push_back({{"FOP_ROW_PREFETCH", 2}, {"FOP_ROW_MINB", 2}});
      if (L.row_p > 1) {   // short rows: one vector per lane per row, latency hidden by more warps
        v.push_back({{"FOP_ROW_MINB", 6}});
        v.push_back({{"FOP_ROW_MINB", 8}});
      }
      break;
    default:
      v.push_back({{"FOP_COL_U", 2}, {"FOP_COL_MINB", 8}});
      v.push_back({{"FOP_COL_U", 8}, {"FOP_COL_MINB", 4}});
      v.push_back({{"FOP_COL_U", 4}, {"FOP_COL_MINB", 6}, {"FOP_COL_SLAB_BYTES", 256}});
  }
  return v;
}

static int knob_w_cap(const Launch& L) { return geometry_knob(L, "FOP_SEQ_W", 1 << 20); }

void finalize_launch_geometry(const Plan& p, Launch& L) {
  // variants start as copies of the planned launch: a flag one class sets must
  // not survive into a copy that ends in another class (the narrow variant of a
  // transpose becomes EW with gathers; a stale tma = 1 sent misaligned pointers
  // to cuTensorMapEncodeTiled — fuzz seed 41, tests/fuzz_regressions/)
  L.tma = 0;
  const fop_desc& d = p.desc;
  const fop_plan_opts& o = p.opts;
  auto acc = all_accesses(L);
  int sms = o.sm_count > 0 ? o.sm_count : 148;
  // vector bytes: the planner option, or a tuning candidate's FOP_VEC_BYTES
  // (LDG/STG.256 stores measured +3-7 % on copies, profiles/r02/bw_probe2_r02.log)
  int vbytes = geometry_knob(L, "FOP_VEC_BYTES", o.max_vec_bytes);
  if (vbytes != 4 && vbytes != 8 && vbytes != 16 && vbytes != 32) vbytes = o.max_vec_bytes;
  int vmax = vbytes >= 32 ? 32 : 16;

  // ---- loop order + collapse
  L.kl.clear();
  std::vector<int> rest;
  for (int l : L.loops)
    if (l != L.vec_loop && l != L.read_loop && std::find(L.seq.begin(), L.seq.end(), l) == L.seq.end())
      rest.push_back(l);
  if (L.kclass == FOP_CLASS_EW || L.kclass == FOP_CLASS_TRANSPOSE) {
    std::vector<int> ord = {L.vec_loop};
    if (L.kclass == FOP_CLASS_TRANSPOSE) ord.push_back(L.read_loop);
    for (int l : order_rest(p, L, rest)) ord.push_back(l);
    L.order = ord;
    std::vector<int> seg0 = {ord[0]};
    collapse_into(p, acc, seg0, L.kl);
    std::vector<int> seg1(ord.begin() + 1, ord.end());
    // V never absorbs loops in TRANSPOSE (d_r follows it); in EW it may
    if (L.kclass == FOP_CLASS_EW) {
      L.kl.clear();
      collapse_into(p, acc, ord, L.kl);
      if (L.virt_vec) L.kl[0].extent = 1;   // fully sequential statement (row N3)
    } else {
      // d_v first absorbs the loops that continue it contiguously for every
      // access, wherever they sit in the order (NHWC -> NCHW: w then h is one
      // run on both sides, d_v = hw, not w alone), then d_r absorbs its own
      std::vector<int> vseg = {ord[0]}, others(ord.begin() + 2, ord.end());
      int64_t vext = p.desc.extent[ord[0]];
      for (bool grew = true; grew;) {
        grew = false;
        for (size_t q = 0; q < others.size() && !grew; q++) {
          bool ok = true;
          for (const Affine* a : acc)
            if (a->coef[others[q]] != a->coef[ord[0]] * vext) ok = false;
          if (ok) {
            vseg.push_back(others[q]);
            vext *= p.desc.extent[others[q]];
            others.erase(others.begin() + q);
            grew = true;
          }
        }
      }
      L.kl.clear();
      collapse_into(p, acc, vseg, L.kl);
      seg1.assign(1, ord[1]);
      seg1.insert(seg1.end(), others.begin(), others.end());
      collapse_into(p, acc, seg1, L.kl);
      L.order = vseg;
      L.order.insert(L.order.end(), seg1.begin(), seg1.end());
    }
    L.nsplit = L.kclass == FOP_CLASS_TRANSPOSE ? 2 : 1;
  } else {
    // ROW: [d_v, other reduction loops | parallel loops]
    // COL: [d_v, other parallel loops  | reduction loops]
    const Affine* wp = &L.stmts.back().write;  // a REDUCE target
    for (const auto& x : L.stmts)
      if (x.kind == FOP_REDUCE) wp = &x.write;
    const Affine& w = *wp;
    std::vector<int> red, par;
    for (int l : rest) (w.coef[l] == 0 ? red : par).push_back(l);
    std::vector<int> seg1 = {L.vec_loop}, seg2;
    std::vector<int> first = L.kclass == FOP_CLASS_ROW_REDUCE ? red : par;
    std::vector<int> second = L.kclass == FOP_CLASS_ROW_REDUCE ? par : red;
    for (int l : order_rest(p, L, first)) seg1.push_back(l);
    for (int l : order_rest(p, L, second)) seg2.push_back(l);
    L.order = seg1;
    L.order.insert(L.order.end(), seg2.begin(), seg2.end());
    collapse_into(p, acc, seg1, L.kl);
    L.nsplit = (int)L.kl.size();
    collapse_into(p, acc, seg2, L.kl);
  }

  // ---- EW over an innermost extent no vector divides, under a broadcast along
  // it (bias add over 1001 columns: the bias row blocks the collapse of
  // (c, r), and W must divide E[c]).  When every access is either contiguous
  // across (d_v, next loop) — coef(next) == E[d_v] — or ignores the next loop
  // (a "period" access, e.g. bias[c]), the two loops become one flat loop
  // carrying full-width vectors; period accesses are read per element at
  // c = flat index mod E[d_v] (vector and scalar accesses mixed).
  L.period = 0;
  L.period_load.assign(L.loads.size(), 0);
  if (L.kclass == FOP_CLASS_EW && L.seq.empty() && !L.virt_vec && !L.scalar_variant && !L.force_w1 &&
      L.kl.size() >= 2 && geometry_knob(L, "FOP_EW_PERIOD", 1)) {
    const int64_t E0 = L.kl[0].extent;
    int mes = 16;
    for (const Affine* a : acc)
      if (coef(L, *a, 0) == 1) mes = std::min(mes, esize(d.t[a->tensor].dtype));
    const int Wf = std::max(1, vbytes / mes);
    if (Wf > 1 && E0 % Wf != 0 && E0 >= Wf && (o.force_width <= 0 || o.force_width >= Wf)) {
      bool ok = true;
      int nflat = 0;
      for (size_t k = 0; k < L.loads.size() && ok; k++) {
        const int64_t c0 = coef(L, L.loads[k], 0), c1 = coef(L, L.loads[k], 1);
        if (c0 == 1 && c1 == E0) nflat++;
        else if (c1 == 0 && c0 != 0) L.period_load[k] = 1;   // varies with c only: read at flat mod E[c]
        else if (c1 != 0 || c0 != 0) ok = false;              // (c0 == c1 == 0: a scalar along both, kept)
      }
      for (const auto& x : L.stmts)
        ok &= coef(L, x.write, 0) == 1 && coef(L, x.write, 1) == E0;
      if (ok && nflat + (int)L.stmts.size() > 0) {
        L.period = E0;
        KLoop& K = L.kl[0];
        K.members.insert(K.members.end(), L.kl[1].members.begin(), L.kl[1].members.end());
        K.extent *= L.kl[1].extent;
        L.kl.erase(L.kl.begin() + 1);
      } else {
        L.period_load.assign(L.loads.size(), 0);
      }
    }
  }

  // ---- a4: width
  int min_es = 16;
  bool any_vec = false;
  for (const Affine* a : acc)
    if (coef(L, *a, 0) == 1) {
      min_es = std::min(min_es, esize(d.t[a->tensor].dtype));
      any_vec = true;
    }
  int W = any_vec ? std::max(1, vbytes / min_es) : 1;
  if (o.force_width > 0) W = std::min(W, pow2_floor(o.force_width));
  if (L.scalar_variant || L.force_w1) W = 1;
  if (!L.seq.empty() && any_vec) {
    // sequential launches get one thread per W lanes and nothing else to hide
    // latency with: narrow the vectors (down to 4-byte accesses) until the
    // lanes cover ~128 threads per SM
    int64_t lanes = 1;
    for (const auto& k : L.kl) lanes *= k.extent;
    while (W > 1 && W * min_es > 4 && lanes / W < (int64_t)sms * 128) W /= 2;
    W = std::min(W, knob_w_cap(L));
  }
  int64_t EV = L.kl[0].extent;
  bool tail_ok = L.kclass == FOP_CLASS_EW && L.kl.size() == 1;
  // ROW over rows of odd length / odd pitch (GPT-2's 50257-entry vocabulary,
  // LayerNorm over 1023): keep the full vector width and peel per row — the
  // kernel shifts each row to its first W-aligned element (the same shift for
  // every vectorised access: their offsets agree modulo W), runs W-vectors in
  // between and takes the <= 2(W-1) head/tail elements as scalars
  L.row_peel = 0;
  if (L.kclass == FOP_CLASS_ROW_REDUCE && W > 1 && EV % W != 0 && EV >= 4 * W && L.nsplit == 1 &&
      L.seq.empty() && geometry_knob(L, "FOP_ROW_PEEL", 1)) {
    const Affine* ref = nullptr;
    bool ok = true;
    auto row_invariant = [&](const Affine* a) {
      for (size_t k = 1; k < L.kl.size(); k++)
        if (coef(L, *a, (int)k) != 0) return false;
      return true;
    };
    for (const Affine* a : acc) {
      // row-invariant vectors (LayerNorm's gamma/beta) keep their own
      // positions: loaded element-wise (cached), not part of the congruence
      if (coef(L, *a, 0) != 1 || row_invariant(a)) continue;
      if (!ref) ref = a;
      ok &= ((a->base - ref->base) % W + W) % W == 0;
      for (size_t k = 1; k < L.kl.size(); k++) ok &= ((coef(L, *a, (int)k) - coef(L, *ref, (int)k)) % W + W) % W == 0;
    }
    if (ok && ref) L.row_peel = 1;
  }
  // COL_REDUCE over rows no vector divides (column sums over 1001 columns): keep
  // the full width; each lane loads the two aligned 16 B chunks around its W
  // columns of the row and funnel-shifts them by the row's misalignment (the
  // same for every lane of the row), so the loads stay 16 B vectors whatever
  // the row pitch; the last vector's columns past E[d_v] are never stored.
  L.col_shift = 0;
  if (L.kclass == FOP_CLASS_COL_REDUCE && W > 1 && EV % W != 0 && EV >= W && L.nsplit == 1 && !L.scalar_variant &&
      L.stmts.size() == 1 && geometry_knob(L, "FOP_COL_SHIFT", 1)) {
    bool ok = coef(L, L.stmts[0].write, 0) == 1;
    for (const auto& a : L.loads) {
      const int64_t c0 = coef(L, a, 0);
      ok &= c0 == 0 || (c0 == 1 && W * esize(d.t[a.tensor].dtype) == 16);
    }
    if (ok) L.col_shift = 1;
  }
  // ... and when the rows are dense (pitch E[d_v]), with P = W / gcd(E, W),
  // P consecutive rows are P*E elements: a whole number of aligned W-vectors.
  // Read the first R - R mod P rows as [R/P, P*E] — full-width aligned
  // vectors, no shifts — where lane j's element e always falls on column
  // (j*W + e) mod E (of row (j*W + e) div E inside the group); the last block
  // to finish folds the P*E wide-column sums into the E outputs, P terms each
  // in group-row order, then adds the R mod P remaining rows element-wise
  // (the vector access is kept whole, scalar accesses mixed in).
  L.col_fold = 0;
  if (L.kclass == FOP_CLASS_COL_REDUCE && W > 1 && EV % W != 0 && L.nsplit == 1 && L.kl.size() == 2 &&
      !L.scalar_variant && L.stmts.size() == 1 && p.opts.peer_world < 1 && geometry_knob(L, "FOP_COL_FOLD", 1)) {
    const int64_t P = W / std::gcd<int64_t>(EV, W);
    bool ok = L.kl[1].extent >= P && coef(L, L.stmts[0].write, 0) == 1 && coef(L, L.stmts[0].write, 1) == 0;
    for (const auto& a : L.loads) {
      const int es_a = esize(d.t[a.tensor].dtype);
      ok &= coef(L, a, 0) == 1 && coef(L, a, 1) == EV && W * es_a == 16 && a.base * es_a % 16 == 0;
    }
    if (ok) {
      L.col_fold = (int)P;
      L.col_shift = 0;
    }
  }
  if (tail_ok) {
    if (EV < W) W = pow2_floor(EV);
  } else if (!L.row_peel && !L.col_shift && !L.col_fold) {
    while (W > 1 && EV % W) W /= 2;
  }
  L.width = W;

  if (L.kclass == FOP_CLASS_TRANSPOSE) {
    const Affine& t = L.loads[L.trans_load];
    // read-side vector bytes: the store side's by default; FOP_TR_WR_BYTES sets them
    // apart (32 B loads along d_r under 16 B stores along d_v: an 8 x 16 tile of 16-bit data)
    int wr = std::max(1, std::min<int>(32, geometry_knob(L, "FOP_TR_WR_BYTES", vbytes)) / esize(d.t[t.tensor].dtype));
    if (o.force_width > 0) wr = std::min(wr, pow2_floor(o.force_width));
    if (L.scalar_variant) wr = 1;
    while (wr > 1 && L.kl[1].extent % wr) wr /= 2;
    L.read_width = wr;
    L.tr_smem = 0;
    L.tr_om = 0;
    if (W >= 2 && wr == 1 && !L.scalar_variant && geometry_knob(L, "FOP_TR_SMEM", 1)) {
      // d_r cannot carry vectors (odd extent, e.g. a 7x7 plane: 49), but when
      // consecutive d_v rows are adjacent in the load tensor (coef(d_v) ==
      // E[d_r]) a tile of TV full rows is one flat contiguous chunk: load it
      // with 16 B vectors into shared memory and store vectors along d_v
      // (ResNet stage-4 NCHW [N,2048,7,7] -> NHWC)
      const int64_t ER = L.kl[1].extent, EVx = L.kl[0].extent;
      const Affine& t = L.loads[L.trans_load];
      const int esi = esize(d.t[t.tensor].dtype);
      bool ok = L.stmts.size() == 1 && coef(L, t, 1) == 1 && coef(L, t, 0) == ER && (t.base * esi) % 16 == 0;
      for (size_t k = 2; k < L.kl.size() && ok; k++) ok = (coef(L, t, (int)k) * esi) % 16 == 0;
      for (size_t k = 0; k < L.loads.size() && ok; k++) {
        if ((int)k == L.trans_load) continue;
        for (size_t q = 0; q < L.kl.size(); q++) ok &= coef(L, L.loads[k], (int)q) == 0;   // constants only
      }
      int64_t TV = 0;
      const int64_t cap = std::min<int64_t>(EVx, geometry_knob(L, "FOP_TR_SMEM_BYTES", 32768) / (ER * esi));
      for (int64_t tv = cap - cap % W; ok && tv >= W; tv -= W)
        if (EVx % tv == 0 && (tv * ER * esi) % 16 == 0) {
          TV = tv;
          break;
        }
      if (TV) {
        L.tr_smem = 1;
        L.tr_tv = TV;
      }
    }
    // (a long odd d_v, e.g. C = 255, puts the read-out's consecutive lanes 8
    // tile rows apart, on few shared-memory banks: 1104 GB/s, still above the
    // gathering elementwise kernel's 958 — profiles/odd_variety_r01.log)
    // (FOP_TR_SMEM_OUT=1 takes this path even when d_v could carry store vectors: an ablation/tuning
    // candidate for ordinary transposes such as cfg3)
    if ((W == 1 || geometry_knob(L, "FOP_TR_SMEM_OUT", 0)) && wr >= 2 && !L.scalar_variant &&
        L.kl[0].extent <= geometry_knob(L, "FOP_TR_SMEM_MAXV", 1 << 30) &&
        geometry_knob(L, "FOP_TR_SMEM", 1)) {
      // the mirror case: d_v rows too short/odd for store vectors (an input
      // layer's C = 3; NHWC -> NCHW of a 7x7 plane), but the output rows are
      // adjacent (coef_out(d_r) == E[d_v]): a tile of TR whole output rows is
      // one contiguous chunk of the output, written with 16 B vectors after
      // the input rows were loaded with vectors along d_r
      const int64_t ER = L.kl[1].extent, EVx = L.kl[0].extent;
      const Affine& w = L.stmts[0].write;
      const int eso = esize(L.stmts[0].out_dtype);
      bool ok = L.stmts.size() == 1 && coef(L, w, 0) == 1 && coef(L, w, 1) == EVx && (w.base * eso) % 16 == 0;
      for (size_t k = 2; k < L.kl.size() && ok; k++) ok = (coef(L, w, (int)k) * eso) % 16 == 0;
      for (size_t k = 0; k < L.loads.size() && ok; k++) {
        if ((int)k == L.trans_load) continue;
        for (size_t q = 0; q < L.kl.size(); q++) ok &= coef(L, L.loads[k], (int)q) == 0;   // constants only
      }
      const int esi = esize(d.t[L.loads[L.trans_load].tensor].dtype);
      const int64_t rowb = EVx * std::max(esi, eso);
      const int64_t cap = std::min<int64_t>(ER, geometry_knob(L, "FOP_TR_SMEM_BYTES", 32768) / rowb);
      // output-major tile for long d_v rows (codegen gen_transpose_smem_out): each
      // lane reads one input row's vector, so the vector grows to a full 32 B
      // sector (C = 255: 3.1 -> 5.4 TB/s, profiles/r02/sweep_r02_trsmem.log)
      const bool om = EVx >= 32 && geometry_knob(L, "FOP_TR_SMEM_OM", 1);
      auto pick = [&](int w_) -> int64_t {   // rows per tile for read vectors of w_ elements, 0 = none
        // the input rows are read with whole vectors along d_r: every row start aligned
        if (!ok || w_ < 2 || ER % w_ || chunk_bytes(p, L, L.loads[L.trans_load], 1, w_ * esi) != w_ * esi) return 0;
        for (int64_t tr = cap - cap % w_; tr >= w_; tr -= w_)
          if (ER % tr == 0 && (tr * EVx * eso) % 16 == 0) return tr;
        return 0;
      };
      int64_t TR = 0;
      if (om) {
        const int w32 = std::min<int>(32, geometry_knob(L, "FOP_TR_WR_BYTES", 32)) / esi;
        if ((TR = pick(w32))) wr = L.read_width = w32;
      }
      if (!TR) TR = pick(wr);
      if (TR) {
        L.tr_smem = 2;
        L.tr_tv = TR;
        L.tr_om = om ? 1 : 0;
      }
    }
    if ((W == 1 || wr == 1) && !L.tr_smem) {  // degenerate tile: plain elementwise with gathers
      L.kclass = FOP_CLASS_EW;
      L.read_loop = -1;
      L.trans_load = -1;
      L.read_width = 0;
      finalize_launch_geometry(p, L);
      return;
    }
  }

  // ---- a4: per-access chunks
  // loads may move wider chunks than the stores (FOP_LD_BYTES=32: LDG.256 under
  // STG.128, the copy pattern measured fastest at 0.4-1 GB, profiles/r02/bw_probe3_r02.log)
  const int vmax_ld = geometry_knob(L, "FOP_LD_BYTES", vmax) >= 32 ? 32 : vmax;
  auto vec_cb = [&](const Affine& a, int vk, int w, int cap) {
    int es = esize(d.t[a.tensor].dtype);
    return chunk_bytes(p, L, a, vk, std::min(cap, w * es));
  };
  L.load_cb.assign(L.loads.size(), 0);
  L.load_cb_r.assign(L.loads.size(), 0);
  for (size_t k = 0; k < L.loads.size(); k++) {
    if (coef(L, L.loads[k], 0) == 1 && !L.period_load[k]) L.load_cb[k] = vec_cb(L.loads[k], 0, W, vmax_ld);
    if (L.kclass == FOP_CLASS_TRANSPOSE && coef(L, L.loads[k], 0) != 1 && coef(L, L.loads[k], 1) == 1)
      L.load_cb_r[k] = vec_cb(L.loads[k], 1, L.read_width, 32);
  }
  L.store_cb.assign(L.stmts.size(), 0);
  for (size_t k = 0; k < L.stmts.size(); k++)
    if (coef(L, L.stmts[k].write, 0) == 1) L.store_cb[k] = vec_cb(L.stmts[k].write, 0, W, vmax);
  if (L.col_shift)   // aligned 16 B chunks around each row's window (the base must be 16 B aligned)
    for (size_t k = 0; k < L.loads.size(); k++)
      if (coef(L, L.loads[k], 0) == 1) L.load_cb[k] = 16;
  if (L.col_fold) {   // aligned 16 B vectors of the [R/P, P*E] view; the E outputs are stored element-wise
    for (size_t k = 0; k < L.loads.size(); k++) L.load_cb[k] = 16;
    L.store_cb[0] = 0;
  }
  if (L.row_peel) {   // alignment comes from the per-row shift, not from the static coefficients
    for (size_t k = 0; k < L.loads.size(); k++) {
      if (coef(L, L.loads[k], 0) != 1) continue;
      bool rinv = true;
      for (size_t q = 1; q < L.kl.size(); q++) rinv &= coef(L, L.loads[k], (int)q) == 0;
      const int es_k = esize(d.t[L.loads[k].tensor].dtype);
      // row-invariant (LayerNorm's gamma/beta): two aligned vectors around the
      // shifted window when the base is vector-aligned, element-wise otherwise
      L.load_cb[k] = rinv && L.loads[k].base % W != 0 ? es_k : std::min(vmax, W * es_k);
    }
    for (size_t k = 0; k < L.stmts.size(); k++)
      if (coef(L, L.stmts[k].write, 0) == 1) L.store_cb[k] = std::min(vmax, W * esize(L.stmts[k].out_dtype));
  }
  L.align.assign(d.ntensors, 1);
  for (size_t k = 0; k < L.loads.size(); k++) {
    int t = L.loads[k].tensor;
    L.align[t] = std::max({L.align[t], L.load_cb[k], L.load_cb_r[k], esize(d.t[t].dtype)});
  }
  for (size_t k = 0; k < L.stmts.size(); k++) {
    int t = L.stmts[k].write.tensor;
    L.align[t] = std::max({L.align[t], L.store_cb[k], esize(d.t[t].dtype)});
  }
  if (L.tr_smem == 1) L.align[L.loads[L.trans_load].tensor] = std::max(L.align[L.loads[L.trans_load].tensor], 16);
  if (L.tr_smem == 2) L.align[L.stmts[0].write.tensor] = std::max(L.align[L.stmts[0].write.tensor], 16);

  // ---- a5: launch geometry.  Grid-stride classes launch exactly the blocks
  // that are resident at once (SMs x minblocks, guaranteed by
  // __launch_bounds__(block, minblocks)): one wave, no tail wave.
  // FOP_<CLASS>_U / FOP_<CLASS>_MINB override the defaults (tuning sweeps).
  int64_t prod_rest = 1;
  L.ws_bytes = 0;
  auto knob = [&](const char* name, int dflt) { return geometry_knob(L, name, dflt); };
  L.block = knob("FOP_BLOCK", 256);
  if (L.kclass == FOP_CLASS_EW) {
    for (size_t k = 1; k < L.kl.size(); k++) prod_rest *= L.kl[k].extent;
    int64_t nv = (EV + W - 1) / W;
    L.work = nv * prod_rest;
    // bytes each work item loads; ~128 B of loads in flight per thread at
    // 512-768 threads/SM measured best on B200 (tools/sweep.py)
    int bytes = 0;
    for (size_t k = 0; k < L.loads.size(); k++)
      if (coef(L, L.loads[k], 0) != 0) bytes += W * esize(d.t[L.loads[k].tensor].dtype);
    int u = bytes > 0 ? std::max(1, std::min(8, pow2_floor(std::max(1, 128 / bytes)))) : 4;
    L.unroll = L.seq.empty() ? knob("FOP_EW_U", u) : 1;   // RMW: one target vector per thread
    L.minblocks = knob("FOP_EW_MINB", L.unroll >= 4 ? 2 : 3);
    if (!L.seq.empty()) {
      // one pass over the lanes (a second grid-stride pass would double the
      // sequential chain); small blocks spread the lanes over every SM; the
      // target-independent loads of the innermost sequential loop are kept
      // P iterations ahead (512 B per thread, <= 128 registers; measured on a
      // [64,512,768] f16 time scan: P=16 3.3 TB/s, 64 4.8 TB/s, 128 5.2 TB/s)
      int pbytes = 0;
      const int sl = L.seq.back();
      for (const auto& a : L.loads)
        if (a.tensor != L.stmts[0].write.tensor && a.coef[sl] != 0)
          pbytes += (coef(L, a, 0) != 0 ? W : 1) * esize(d.t[a.tensor].dtype);
      int P = pbytes ? std::max(2, std::min(128, pow2_floor(std::max(1, 512 / pbytes)))) : 1;
      L.seq_prefetch = knob("FOP_SEQ_P", P);
      L.block = knob("FOP_BLOCK", L.work >= (int64_t)sms * 256 ? 256 : (L.work >= (int64_t)sms * 128 ? 128 : 64));
      int64_t need = (L.work + L.block - 1) / L.block;
      L.minblocks = knob("FOP_EW_MINB", (int)std::max<int64_t>(1, std::min<int64_t>(8, (need + sms - 1) / sms)));
      L.grid = std::max<int64_t>(1, need);
    } else {
      int64_t need = (L.work + (int64_t)L.block * L.unroll - 1) / ((int64_t)L.block * L.unroll);
      L.grid = std::max<int64_t>(1, std::min<int64_t>(need, (int64_t)sms * L.minblocks));
    }
  } else if (L.kclass == FOP_CLASS_TRANSPOSE && L.tr_smem) {
    // one tile (TV x E[d_r]) per CTA iteration, several CTAs per SM so one
    // CTA's loads overlap another's shared-memory read-out and stores
    for (size_t k = 2; k < L.kl.size(); k++) prod_rest *= L.kl[k].extent;
    L.block = 256;
    L.unroll = 1;
    L.tma = 0;
    L.minblocks = knob("FOP_TR_SMEM_MINB", 4);
    const int esi = esize(d.t[L.loads[L.trans_load].tensor].dtype);
    if (L.tr_smem == 1) {   // tiles of tr_tv d_v rows
      L.work = (L.kl[0].extent / L.tr_tv) * prod_rest;
      L.smem = (size_t)L.tr_tv * L.kl[1].extent * esi;
    } else {                // tiles of tr_tv d_r positions (output rows)
      L.work = (L.kl[1].extent / L.tr_tv) * prod_rest;
      L.smem = (size_t)L.tr_tv * L.kl[0].extent * esi;
    }
    L.grid = std::max<int64_t>(1, std::min<int64_t>(L.work, (int64_t)sms * L.minblocks));
  } else if (L.kclass == FOP_CLASS_TRANSPOSE) {
    for (size_t k = 2; k < L.kl.size(); k++) prod_rest *= L.kl[k].extent;
    int64_t ntv = EV / W, ntr = L.kl[1].extent / L.read_width;
    int es_out = esize(L.stmts[0].out_dtype);
    int gv = (int)std::min<int64_t>(32, std::max<int64_t>(1, 128 / (W * es_out)));
    gv = std::min(pow2_floor(std::max(1, std::min(32, knob("FOP_TR_GV", gv)))), pow2_floor(ntv));
    L.gv = gv;
    L.gr = 32 / gv;
    int64_t tvh = (ntv + gv - 1) / gv, trh = (ntr + L.gr - 1) / L.gr;
    // U tiles per thread, adjacent along d_r (tr, tr+gr, ...): a warp's loads
    // of consecutive tiles complete the same 128 B lines back to back
    L.unroll = std::max(1, knob("FOP_TR_U", 2));
    trh = (ntr + (int64_t)L.gr * L.unroll - 1) / ((int64_t)L.gr * L.unroll);
    if (knob("FOP_TR_ORDER", 0) == 2) {   // blocked traversal (codegen gen_transpose): whole blocks of BV
      const int64_t BV = std::max(1, knob("FOP_TR_BV", 8));
      tvh = (tvh + BV - 1) / BV * BV;
    }
    L.work = (int64_t)gv * L.gr * tvh * trh * prod_rest;
    // 8 warps per SM (16 at U = 1) in small CTAs: 64-thread CTAs x 4 per SM measured +1.4 % over
    // one 256-thread CTA on cfg3 (6097 vs 6013 GB/s, profiles/r02/sweep_r02_trblock.log) — CTAs
    // retire independently, so the grid's tail is finer
    L.block = knob("FOP_BLOCK", 64);
    L.minblocks = knob("FOP_TR_MINB", std::max(1, (L.unroll >= 2 ? 8 : 16) * 32 / L.block));
    int64_t need = (L.work + L.block - 1) / L.block;
    L.grid = std::max<int64_t>(1, std::min<int64_t>(need, (int64_t)sms * L.minblocks));

    // TMA variant (sm_100a tensor memory accelerator): 64x64 16-bit tiles
    // moved by cp.async.bulk.tensor with 128B swizzle, mbarrier pipeline.
    L.tma = 0;
    const Affine& tl = L.loads[L.trans_load];
    const XStmt& x0 = L.stmts[0];
    // Default for eligible 16-bit transposes since round 2 (2 stages per warp): in the bench suite
    // 6427 vs 6106 GB/s for the register tiles (suite 6299 vs 6166), cold single launch under ncu
    // 122.4 vs 131.8 us; only back-to-back repeats of the same transpose favour the register tiles
    // (5971 vs 6104, profiles/r02/tma_suite_r02.log).  FOP_TR_TMA=0 selects the register path.
    bool ok = knob("FOP_TR_TMA", 1) && !L.scalar_variant && L.stmts.size() == 1 &&
              esize(d.t[tl.tensor].dtype) == 2 && esize(x0.out_dtype) == 2 && L.kl.size() <= 5 &&
              L.kl[0].extent >= 64 && L.kl[1].extent >= 64 && tl.base % 8 == 0 && x0.write.base % 8 == 0;
    for (size_t k = 0; k < L.loads.size() && ok; k++) {
      if ((int)k == L.trans_load) continue;
      for (size_t q = 0; q < L.kl.size(); q++) ok &= coef(L, L.loads[k], (int)q) == 0;   // constants only
    }
    if (ok) {
      int r = (int)L.kl.size();
      // load tensor dims: R (contiguous), V, outer...; store tensor dims: V (contiguous), R, outer...
      int in_order[5], out_order[5];
      in_order[0] = 1;
      in_order[1] = 0;
      out_order[0] = 0;
      out_order[1] = 1;
      for (int q = 2; q < r; q++) in_order[q] = out_order[q] = q;
      for (int q = 0; q < r && ok; q++) {
        int ki = in_order[q], ko = out_order[q];
        L.tma_in_dim[q] = (uint64_t)L.kl[ki].extent;
        L.tma_out_dim[q] = (uint64_t)L.kl[ko].extent;
        int64_t si = coef(L, tl, ki) * 2, so = coef(L, x0.write, ko) * 2;
        if (q == 0) {
          ok &= si == 2 && so == 2;
        } else {
          ok &= si > 0 && so > 0 && si % 16 == 0 && so % 16 == 0 && si < (int64_t(1) << 40) && so < (int64_t(1) << 40);
          L.tma_in_stride[q - 1] = (uint64_t)si;
          L.tma_out_stride[q - 1] = (uint64_t)so;
        }
      }
      if (ok) {
        L.tma = 1;
        L.tma_rank = r;
        L.tma_in_tensor = tl.tensor;
        L.tma_out_tensor = x0.write.tensor;
        L.tma_in_base = tl.base;
        L.tma_out_base = x0.write.base;
        L.tma_stages = std::max(2, std::min(8, knob("FOP_TR_TMA_STAGES", 2)));   // 3+ stages: 5.6-5.8 TB/s in the suite
        L.tma_ntv = (L.kl[0].extent + 63) / 64;
        L.tma_ntr = (L.kl[1].extent + 63) / 64;
        L.tma_tiles = L.tma_ntv * L.tma_ntr * prod_rest;
        // one independent pipeline per warp: S input stages + 2 output tiles of 8 KB
        int nw = std::max(1, std::min(8, knob("FOP_TR_TMA_WARPS", 4)));
        L.minblocks = knob("FOP_TR_TMA_MINB", 1);
        while ((size_t)nw * (L.tma_stages + 2) * 8192 * L.minblocks > 220 * 1024) {
          if (L.tma_stages > 2) L.tma_stages--;
          else if (nw > 1) nw--;
          else break;
        }
        L.block = 32 * nw;
        L.smem = (size_t)nw * (L.tma_stages + 2) * 8192 + 8 * nw * L.tma_stages + 1024;
        L.align[tl.tensor] = std::max(L.align[tl.tensor], 16);      // TMA global address alignment
        L.align[x0.write.tensor] = std::max(L.align[x0.write.tensor], 16);
        int64_t ctas = (L.tma_tiles + nw - 1) / nw;
        L.grid = std::max<int64_t>(1, std::min<int64_t>(ctas, (int64_t)sms * L.minblocks));
        L.work = L.tma_tiles;
      }
    }
  } else if (L.kclass == FOP_CLASS_ROW_REDUCE) {
    int64_t rows = 1;
    for (size_t k = L.nsplit; k < L.kl.size(); k++) rows *= L.kl[k].extent;
    L.work = rows;
    // one warp per row while the rows fill the GPU; few long rows get G warps
    // each (up to 32), until ~16 warps per SM are busy or a lane would hold
    // fewer than 4 vectors of the row (measured: G=16 beats 32 at 2-4
    // vectors per lane, profiles/sweep_r01_rowg.log)
    int64_t nvd = EV / W;
    int64_t nro = 1;
    for (int k = 1; k < L.nsplit; k++) nro *= L.kl[k].extent;
    // few vectors along d_v under long outer reduction loops (per-channel
    // statistics over N,H,W of an NCHW tensor: 7 vectors x 14336 outer
    // iterations): the lanes also split the outer iterations, else most
    // lanes idle and one chain walks the whole row
    const bool split = nvd < 32 && nro * W > 64 && knob("FOP_ROW_SPLIT", 1);
    const int64_t row_vecs = split ? nvd * nro : nvd;
    int G = 1;
    while (G < 32 && rows * G < (int64_t)sms * 16 && 256 * (int64_t)G <= row_vecs) G *= 2;
    // fewer rows than SMs: each row also spreads over a cluster of Q CTAs
    // (several SMs; block partials combined through distributed shared
    // memory), G capped at 8 warps per CTA so the parallelism goes across SMs
    const int64_t lanes_cap = split ? nvd * nro : nvd;   // lanes one row can keep busy
    int Q = 1;
    if (rows < (int64_t)sms) {
      G = std::min(G, 8);
      while (Q < 8 && rows * Q * 2 <= (int64_t)sms * 2 && 32 * (int64_t)G * Q * 2 <= lanes_cap) Q *= 2;
    }
    G = std::max(1, pow2_floor(knob("FOP_ROW_G", G)));
    Q = std::max(1, std::min(8, pow2_floor(knob("FOP_ROW_Q", Q))));
    // short rows (fewer than 16 vectors): P rows share a warp, 32/P lanes
    // each, so the lanes are not left idle by a row of 4-8 vectors
    int P = 1;
    if (G == 1 && Q == 1 && !split && !L.row_peel && knob("FOP_ROW_P", 1))
      while (P < 32 && 32 / (2 * P) >= nvd) P *= 2;
    // FOP_ROW_PFORCE: P rows per warp regardless (e.g. 2 rows of 48 32-byte vectors
    // over 16 lanes each: 32-byte accesses without a ragged lane count)
    if (G == 1 && Q == 1 && !split && !L.row_peel && knob("FOP_ROW_PFORCE", 0) > 1)
      P = std::min(32, pow2_floor(knob("FOP_ROW_PFORCE", 0)));
    L.row_g = G;
    L.row_q = Q;
    L.row_p = P;
    L.row_split = split ? (int)(32 * (int64_t)G * Q / std::min<int64_t>(32 * (int64_t)G * Q, pow2_ceil(nvd))) : 0;
    if (G > 1) L.block = std::max(L.block, 32 * G);
    if (Q > 1) L.block = 32 * G;   // one row per CTA
    // short rows hold one vector per lane per row: more warps hide the
    // latency (profiles/red_variety_r01.log: [1048576,64] f16 3745 -> 5343 GB/s)
    L.minblocks = knob("FOP_ROW_MINB", L.block >= 1024 ? 1 : (L.block >= 512 ? 2 : (P > 1 ? 8 : 3)));
    L.row_prefetch = knob("FOP_ROW_PREFETCH", 1);   // rows in flight ahead of the one processed (0: none)
    L.row_hoist = knob("FOP_ROW_HOIST", 1);
    int64_t gpb = L.block * P / (32 * G);   // rows per block
    int64_t need = (rows + gpb - 1) / gpb;
    // one resident wave walking the rows (default), or FOP_ROW_ONEPASS=1: a block per
    // group of rows, the hardware block scheduler balancing the SMs as blocks retire
    L.grid = std::max<int64_t>(1, knob("FOP_ROW_ONEPASS", 0) ? need : std::min<int64_t>(need, (int64_t)sms * L.minblocks));
    if (Q > 1)   // whole clusters, one row each per pass
      L.grid = std::max<int64_t>(1, std::min<int64_t>({rows, (int64_t)sms * L.minblocks / Q,
                                                       (int64_t)knob("FOP_ROW_CLUSTERS", 1 << 30)})) * Q;
    L.unroll = 1;
  } else {  // COL_REDUCE
    int64_t nvd = L.col_shift ? (EV + W - 1) / W : L.col_fold ? L.col_fold * EV / W : EV / W;   // col_shift: a partial last vector
    const Affine* big = nullptr;
    for (const auto& a : L.loads)
      if (coef(L, a, 0) == 1) big = &a;
    int es_ld = big ? esize(d.t[big->tensor].dtype) : 4;
    int gv = (int)std::min<int64_t>(32, std::max<int64_t>(1, knob("FOP_COL_SLAB_BYTES", 128) / (W * es_ld)));
    gv = std::min(pow2_floor(gv), pow2_floor(nvd));
    L.gv = gv;
    L.gr = L.block / gv;
    int64_t slabs = (nvd + gv - 1) / gv;
    for (int k = 1; k < L.nsplit; k++) slabs *= L.kl[k].extent;
    int64_t rows = 1;
    for (size_t k = L.nsplit; k < L.kl.size(); k++) rows *= L.kl[k].extent;
    if (L.col_fold) rows /= L.col_fold;   // groups of P rows
    L.col_pipe = knob("FOP_COL_PIPE", 0);   // measured: no gain over plain batches (sweep_r01_4)
    L.col_il = knob("FOP_COL_IL", 1);
    // 6 blocks/SM x 4 rows in flight: the column-sum probe and the sweep
    // (profiles/col_probe_r01.log, sweep_r01_col.log) peak at 6-8 blocks/SM
    L.minblocks = knob("FOP_COL_MINB", 6);
    L.unroll = knob("FOP_COL_U", 4);
    int64_t target = (int64_t)sms * L.minblocks;   // one resident wave
    int64_t nch = std::max<int64_t>(1, target / std::max<int64_t>(1, slabs));
    nch = std::min<int64_t>(nch, std::max<int64_t>(1, (rows + L.gr - 1) / L.gr));
    L.nchunks = nch;
    L.work = rows;
    L.grid = slabs * nch;
    // finalize: store + fence + arrival counter + last-arriving block (0, default),
    // or flag words polled by the slab's last chunk block (1) / last arrival (2)
    L.col_fin = L.col_fold ? 0 : knob("FOP_COL_FIN", 0);
    L.col_acqrel = knob("FOP_COL_ACQREL", 1);   // measured: cfg4b 25.07 -> 25.00 us, odd fold 27.36 -> 26.97 (profiles/r02/sweep_r02_acqrel.log)
    if (nch > 1 && L.col_fin) {
      L.ws_bytes = ((size_t)nch * (size_t)slabs * (size_t)(gv * W) * sizeof(unsigned long long) + 255) & ~size_t(255);
      if (L.col_fin == 2) L.ws_bytes += (size_t)slabs * sizeof(unsigned);
      if (L.col_fin == 3 && !L.col_il) L.col_fin = 1;   // the pure finalizer needs interleaved chunks
    } else if (nch > 1) {
      size_t part = (size_t)nch * (size_t)slabs * (size_t)(gv * W) * sizeof(float);
      part = (part + 255) & ~size_t(255);
      L.ws_bytes = part + (size_t)slabs * sizeof(unsigned);
    }
    if (L.col_fold) {   // the wide-column sums and the arrival counter of the fold
      L.fold_off = (L.ws_bytes + 255) & ~size_t(255);
      L.ws_bytes = L.fold_off + (((size_t)L.col_fold * (size_t)EV * sizeof(float) + 255) & ~size_t(255)) + 16;
    }
    L.smem = (size_t)L.block * W * sizeof(float) + 16;
  }
}

}  // namespace fop
