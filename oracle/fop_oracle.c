/*
 * fop_oracle.c — TEST INFRASTRUCTURE ONLY: the parity oracle.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg,
 * --impl reference) may load this library.  It shares no code, header, table
 * or helper with the product path (paper_conf_cgo_bastoulzrlsjfjc22_b200/).
 *
 * What it computes — the plain definition of a fused operator:
 *   1. statements execute in textual order; each iterates its box domain
 *      D_S = { 0 <= i_l < E_l } (§III-A) in lexicographic
 *      order, i.e. the schedule theta of P:119-121;
 *   2. each read access maps the iteration to an element,
 *      idx_r = i_{iter(r)} + off_r or off_r, widened exactly to fp32;
 *   3. the expression DAG is evaluated node by node: + - * / max min neg abs
 *      sqrt relu in fp32 (IEEE, correctly rounded, no contraction: compiled
 *      with -ffp-contract=off); exp log tanh sigmoid gelu in double, rounded
 *      once to fp32 (reading R12);
 *   4. ASSIGN converts the value to the target element type (RNE, overflow to
 *      inf) and stores it — a read-modify-write statement such as Fig. 2's Y
 *       therefore sees its own earlier stores, strictly in order;
 *      REDUCE overwrites each target element with the sum (or max) over the
 *      statement's remaining loops, accumulated in double, rounded once to
 *      fp32, then the finalize DAG (fp32) and the conversion (readings R16,
 *      R19);
 *   5. later statements read the stored (rounded) values (reading R17).
 *   6. an INTEGER statement (its target is i32, reading R30) evaluates its
 *      DAG on int32 values: every i32 load, constant and + - * max min neg
 *      abs relu result is computed in int64 and reduced modulo 2^32 to the
 *      two's-complement int32 range (wrap-around); REDUCE sums modulo 2^32
 *      (wrapping after every term), MAX keeps the maximum.  Float statements never read i32 tensors, and integer
 *      statements never read float tensors, except a pure element move.
 * No blocking, no reordering, no threads.
 */
#include "fop_oracle.h"

#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

/* ---------------------------------------------------------------------- */
/* Element conversions, written out bit by bit (IEEE 754 binary16/bfloat16). */

float orc_f16_to_f32(uint16_t h) {
  uint32_t sign = (uint32_t)(h & 0x8000u) << 16;
  uint32_t e = (h >> 10) & 0x1Fu;
  uint32_t m = h & 0x3FFu;
  uint32_t bits;
  float out;
  if (e == 0) {
    /* zero or subnormal: value = m * 2^-24, exact in fp32 */
    out = ldexpf((float)m, -24);
    return sign ? -out : out;
  }
  if (e == 31)
    bits = sign | 0x7F800000u | (m << 13);
  else
    bits = sign | ((e + 112u) << 23) | (m << 13);
  memcpy(&out, &bits, 4);
  return out;
}

uint16_t orc_f32_to_f16(float f) {
  uint32_t x, absx, sign, mant, h, rem, half;
  int e, s;
  memcpy(&x, &f, 4);
  sign = (x >> 16) & 0x8000u;
  absx = x & 0x7FFFFFFFu;
  if (absx > 0x7F800000u) /* NaN: quiet, keep top payload bits */
    return (uint16_t)(sign | 0x7E00u | ((absx >> 13) & 0x3FFu));
  if (absx == 0x7F800000u) return (uint16_t)(sign | 0x7C00u);
  e = (int)(absx >> 23) - 127;
  if (e > 15) return (uint16_t)(sign | 0x7C00u); /* >= 2^16: overflow */
  if (e >= -14) {                                  /* normal binary16 range */
    mant = absx & 0x7FFFFFu;
    h = ((uint32_t)(e + 15) << 10) | (mant >> 13);
    rem = mant & 0x1FFFu;
    if (rem > 0x1000u || (rem == 0x1000u && (h & 1u))) h += 1u; /* carry may reach inf: correct */
    return (uint16_t)(sign | h);
  }
  if (e < -25) return (uint16_t)sign; /* below half the smallest subnormal */
  /* subnormal result: units of 2^-24; value = mant * 2^(e-23) */
  mant = (absx & 0x7FFFFFu) | 0x800000u;
  s = -(e + 1); /* 14 .. 24 */
  h = mant >> s;
  rem = mant & ((1u << s) - 1u);
  half = 1u << (s - 1);
  if (rem > half || (rem == half && (h & 1u))) h += 1u;
  return (uint16_t)(sign | h);
}

float orc_bf16_to_f32(uint16_t h) {
  uint32_t bits = (uint32_t)h << 16;
  float out;
  memcpy(&out, &bits, 4);
  return out;
}

uint16_t orc_f32_to_bf16(float f) {
  uint32_t x;
  memcpy(&x, &f, 4);
  if ((x & 0x7FFFFFFFu) > 0x7F800000u) return (uint16_t)((x >> 16) | 0x40u); /* quiet NaN */
  x += 0x7FFFu + ((x >> 16) & 1u); /* round to nearest even */
  return (uint16_t)(x >> 16);
}

/* ---------------------------------------------------------------------- */
/* Operations.  Arithmetic in fp32; transcendentals in double then one
 * rounding to fp32 (R12).                                                 */

float orc_gelu_tanh(float v) {
  double d = (double)v;
  double u = sqrt(2.0 / M_PI) * (d + 0.044715 * d * d * d);
  /* 0.5 d (1 + tanh u) == d / (1 + exp(-2u)): same function, no cancellation
   * of 1 + tanh(u) for very negative d (reading R13) */
  return (float)(d / (1.0 + exp(-2.0 * u)));
}

static float op_max(float a, float b) {
  if (isnan(a)) return b;
  if (isnan(b)) return a;
  if (a == 0.0f && b == 0.0f) return (signbit(a) && signbit(b)) ? -0.0f : 0.0f;
  return a > b ? a : b;
}

static float op_min(float a, float b) {
  if (isnan(a)) return b;
  if (isnan(b)) return a;
  if (a == 0.0f && b == 0.0f) return (signbit(a) || signbit(b)) ? -0.0f : 0.0f;
  return a < b ? a : b;
}

static float round_to(float v, int elem) {
  switch (elem) {
    case ORC_F16: return orc_f16_to_f32(orc_f32_to_f16(v));
    case ORC_BF16: return orc_bf16_to_f32(orc_f32_to_bf16(v));
    default: return v;
  }
}

static float apply(const orc_node *n, const float *val, float acc, float loaded) {
  float a = n->x >= 0 ? val[n->x] : 0.0f;
  float b = n->y >= 0 ? val[n->y] : 0.0f;
  switch (n->kind) {
    case ORC_LOAD: return loaded;
    case ORC_CONST: return (float)n->c;
    case ORC_ACC: return acc;
    case ORC_ADD: return a + b;
    case ORC_SUB: return a - b;
    case ORC_MUL: return a * b;
    case ORC_DIV: return a / b;
    case ORC_MAX: return op_max(a, b);
    case ORC_MIN: return op_min(a, b);
    case ORC_NEG: return -a;
    case ORC_ABS: return fabsf(a);
    case ORC_SQRT: return sqrtf(a);
    case ORC_RELU: return a > 0.0f ? a : 0.0f;
    case ORC_EXP: return (float)exp((double)a);
    case ORC_LOG: return (float)log((double)a);
    case ORC_TANH: return (float)tanh((double)a);
    case ORC_SIGMOID: return (float)(1.0 / (1.0 + exp(-(double)a)));
    case ORC_GELU_TANH: return orc_gelu_tanh(a);
    case ORC_GELU_ERF: return (float)(0.5 * (double)a * erfc(-(double)a / sqrt(2.0))); /* 1+erf(z) = erfc(-z) */
    case ORC_CAST: return round_to(a, n->elem);
  }
  return NAN;
}

/* Integer statements (reading R30): int32 values, two's-complement wrap-around
 * after every operation (the int64 result reduced modulo 2^32).            */
static long long wrap32(long long v) {
  unsigned long long u = (unsigned long long)v & 0xFFFFFFFFull;
  return u >= 0x80000000ull ? (long long)u - 0x100000000ll : (long long)u;
}

static long long apply_int(const orc_node *n, const long long *val, long long acc, long long loaded) {
  long long a = n->x >= 0 ? val[n->x] : 0;
  long long b = n->y >= 0 ? val[n->y] : 0;
  switch (n->kind) {
    case ORC_LOAD: return loaded;
    case ORC_CONST: return wrap32((long long)n->c);
    case ORC_ACC: return acc;
    case ORC_ADD: return wrap32(a + b);
    case ORC_SUB: return wrap32(a - b);
    case ORC_MUL: return wrap32(a * b); /* |a|, |b| <= 2^31: the product fits in int64 */
    case ORC_MAX: return a > b ? a : b;
    case ORC_MIN: return a < b ? a : b;
    case ORC_NEG: return wrap32(-a);
    case ORC_ABS: return wrap32(a < 0 ? -a : a);
    case ORC_RELU: return a > 0 ? a : 0;
  }
  return 0;
}

/* ---------------------------------------------------------------------- */
/* Element addressing and typed load/store.                               */

static long long ref_offset(const orc_array *arr, const orc_ref *r, const long long *it) {
  long long o = 0;
  for (int d = 0; d < arr->rank; d++) {
    long long idx = (r->iter[d] >= 0 ? it[r->iter[d]] : 0) + r->off[d];
    o += idx * arr->stride[d];
  }
  return o;
}

static float load_elem(const orc_array *arr, long long o) {
  switch (arr->elem) {
    case ORC_F32: return ((const float *)arr->data)[o];
    case ORC_F16: return orc_f16_to_f32(((const uint16_t *)arr->data)[o]);
    case ORC_BF16: return orc_bf16_to_f32(((const uint16_t *)arr->data)[o]);
    case ORC_I32: break; /* i32 elements are read by integer statements only (load_int) */
  }
  return NAN;
}

static long long load_int(const orc_array *arr, long long o) { return ((const int32_t *)arr->data)[o]; }

static void store_elem(orc_array *arr, long long o, float v) {
  switch (arr->elem) {
    case ORC_F32: ((float *)arr->data)[o] = v; break;
    case ORC_F16: ((uint16_t *)arr->data)[o] = orc_f32_to_f16(v); break;
    case ORC_BF16: ((uint16_t *)arr->data)[o] = orc_f32_to_bf16(v); break;
    case ORC_I32: break; /* written by integer statements only (store_int) */
  }
}

static void store_int(orc_array *arr, long long o, long long v) { ((int32_t *)arr->data)[o] = (int32_t)wrap32(v); }

static long long array_span(const orc_array *a) {
  long long s = 1;
  for (int d = 0; d < a->rank; d++) {
    if (a->shape[d] <= 0) return 0;
    s += (a->shape[d] - 1) * (a->stride[d] < 0 ? -a->stride[d] : a->stride[d]);
  }
  return s;
}

/* ---------------------------------------------------------------------- */
/* Validation (the oracle's own rules; see fop.h for the product's).      */

static int fail(char *err, int errlen, const char *msg, int s) {
  if (err && errlen > 0) snprintf(err, (size_t)errlen, "statement %d: %s", s, msg);
  return 1;
}

static int check_ref(const orc_ref *r, const orc_statement *st, int narrays, const orc_array *arrays,
                     const long long *ext, int s, char *err, int errlen) {
  if (r->array < 0 || r->array >= narrays) return fail(err, errlen, "bad array index", s);
  const orc_array *a = &arrays[r->array];
  for (int k = 0; k < st->nloops; k++)
    if (ext[st->loops[k]] == 0) return 0; /* empty domain: the access never happens */
  for (int d = 0; d < a->rank; d++) {
    long long lo = r->off[d], hi = r->off[d];
    if (r->iter[d] >= 0) {
      int found = 0;
      for (int k = 0; k < st->nloops; k++) found |= st->loops[k] == r->iter[d];
      if (!found) return fail(err, errlen, "access uses a loop outside the statement", s);
      hi += ext[r->iter[d]] - 1;
    }
    if (lo < 0 || hi >= a->shape[d]) return fail(err, errlen, "access out of bounds", s);
  }
  return 0;
}

static int check_dag(const orc_node *nodes, int n, int nreads, int allow_acc, int s, char *err, int errlen) {
  if (n <= 0 || n > ORC_NODES) return fail(err, errlen, "bad node count", s);
  for (int i = 0; i < n; i++) {
    const orc_node *q = &nodes[i];
    if (q->kind == ORC_LOAD) {
      if (allow_acc || q->x < 0 || q->x >= nreads) return fail(err, errlen, "bad load", s);
      continue;
    }
    if (q->kind == ORC_ACC && !allow_acc) return fail(err, errlen, "acc outside finalize", s);
    if (q->kind == ORC_CONST || q->kind == ORC_ACC) continue;
    if (q->kind < ORC_ADD || q->kind > ORC_CAST) return fail(err, errlen, "bad node kind", s);
    if (q->x < 0 || q->x >= i) return fail(err, errlen, "operand not an earlier node", s);
    if (q->kind <= ORC_MIN && (q->y < 0 || q->y >= i)) return fail(err, errlen, "operand not an earlier node", s);
  }
  return 0;
}

/* Element types of a statement (reading R30): a pure element move copies any
 * type; a statement writing an i32 tensor is an integer statement (i32 reads,
 * integer operations, integral constants); any other statement is a float
 * statement and reads no i32 tensor. */
static int is_move(const orc_statement *st, const orc_array *arrays) {
  return !st->reduce && st->nnodes == 1 && st->nodes[0].kind == ORC_LOAD &&
         arrays[st->reads[st->nodes[0].x].array].elem == arrays[st->target.array].elem;
}

static int int_node_ok(const orc_node *q) {
  switch (q->kind) {
    case ORC_LOAD: case ORC_ACC: case ORC_ADD: case ORC_SUB: case ORC_MUL: case ORC_MAX:
    case ORC_MIN: case ORC_NEG: case ORC_ABS: case ORC_RELU: return 1;
    case ORC_CONST: return q->c == floor(q->c) && q->c >= -2147483648.0 && q->c < 2147483648.0;
  }
  return 0;
}

static int check_types(const orc_statement *st, const orc_array *arrays, int s, char *err, int errlen) {
  if (is_move(st, arrays)) return 0;
  int integer = arrays[st->target.array].elem == ORC_I32;
  for (int r = 0; r < st->nreads; r++)
    if ((arrays[st->reads[r].array].elem == ORC_I32) != integer)
      return fail(err, errlen, integer ? "integer statement reads a float tensor"
                                       : "float statement reads an i32 tensor", s);
  for (int i = 0; i < st->nnodes; i++) {
    if (integer && !int_node_ok(&st->nodes[i])) return fail(err, errlen, "operation not defined on i32", s);
    if (!integer && st->nodes[i].kind == ORC_CAST && st->nodes[i].elem == ORC_I32)
      return fail(err, errlen, "cast to i32", s);
  }
  for (int i = 0; st->reduce && i < st->nfin; i++) {
    if (integer && !int_node_ok(&st->fin[i])) return fail(err, errlen, "operation not defined on i32", s);
    if (!integer && st->fin[i].kind == ORC_CAST && st->fin[i].elem == ORC_I32)
      return fail(err, errlen, "cast to i32", s);
  }
  return 0;
}

/* ---------------------------------------------------------------------- */

static int run_statement(const orc_statement *st, const long long *ext, orc_array *arrays,
                         int narrays, int s, char *err, int errlen) {
  long long it[ORC_LOOPS] = {0};
  float val[ORC_NODES];
  long long ival[ORC_NODES];
  orc_array *tgt = &arrays[st->target.array];
  double *acc = NULL;
  unsigned char *seen = NULL;
  long long span = 0;
  long long total = 1;
  for (int k = 0; k < st->nloops; k++) total *= ext[st->loops[k]];

  /* a pure element move (transpose / copy of any type) keeps the raw bits */
  int move = is_move(st, arrays);
  int integer = !move && tgt->elem == ORC_I32;
  long long *iacc = NULL;

  if (st->reduce) {
    span = array_span(tgt);
    acc = (double *)malloc(sizeof(double) * (size_t)(span > 0 ? span : 1));
    seen = (unsigned char *)calloc((size_t)(span > 0 ? span : 1), 1);
    iacc = (long long *)malloc(sizeof(long long) * (size_t)(span > 0 ? span : 1));
    if (!acc || !seen || !iacc) {
      free(acc);
      free(iacc);
      free(seen);
      return fail(err, errlen, "out of memory", s);
    }
  }

  for (long long n = 0; n < total; n++) {
    /* it[] holds the current iteration vector (odometer, lexicographic) */
    if (move) {
      const orc_ref *r = &st->reads[st->nodes[0].x];
      const orc_array *src = &arrays[r->array];
      long long so = ref_offset(src, r, it), to = ref_offset(tgt, &st->target, it);
      size_t es = (src->elem == ORC_F32 || src->elem == ORC_I32) ? 4 : 2;
      memcpy((char *)tgt->data + to * (long long)es, (const char *)src->data + so * (long long)es, es);
    } else if (integer) {
      for (int i = 0; i < st->nnodes; i++) {
        const orc_node *q = &st->nodes[i];
        long long loaded = 0;
        if (q->kind == ORC_LOAD) {
          const orc_ref *r = &st->reads[q->x];
          loaded = load_int(&arrays[r->array], ref_offset(&arrays[r->array], r, it));
        }
        ival[i] = apply_int(q, ival, 0, loaded);
      }
      long long v = ival[st->nnodes - 1];
      long long to = ref_offset(tgt, &st->target, it);
      if (!st->reduce) {
        store_int(tgt, to, v);
      } else {
        if (!seen[to]) {
          seen[to] = 1;
          iacc[to] = st->reduce_max ? v : 0;
        }
        /* max exact; the sum wraps after every term (arithmetic modulo 2^32) */
        iacc[to] = st->reduce_max ? (v > iacc[to] ? v : iacc[to]) : wrap32(iacc[to] + v);
      }
    } else {
      for (int i = 0; i < st->nnodes; i++) {
        const orc_node *q = &st->nodes[i];
        float loaded = 0.0f;
        if (q->kind == ORC_LOAD) {
          const orc_ref *r = &st->reads[q->x];
          loaded = load_elem(&arrays[r->array], ref_offset(&arrays[r->array], r, it));
        }
        val[i] = apply(q, val, 0.0f, loaded);
      }
      float v = val[st->nnodes - 1];
      long long to = ref_offset(tgt, &st->target, it);
      if (!st->reduce) {
        store_elem(tgt, to, v);
      } else {
        if (!seen[to]) {
          seen[to] = 1;
          acc[to] = st->reduce_max ? -INFINITY : 0.0;
        }
        if (st->reduce_max) {
          acc[to] = (double)op_max((float)acc[to], v); /* max is exact: fold as the max node does */
        } else {
          acc[to] += (double)v;
        }
      }
    }
    for (int k = st->nloops - 1; k >= 0; k--) { /* advance the odometer */
      int l = st->loops[k];
      if (++it[l] < ext[l]) break;
      it[l] = 0;
    }
  }

  if (st->reduce && integer) {
    for (long long o = 0; o < span; o++) {
      if (!seen[o]) continue;
      long long r = wrap32(iacc[o]);
      if (st->nfin > 0) {
        for (int i = 0; i < st->nfin; i++) ival[i] = apply_int(&st->fin[i], ival, r, 0);
        r = ival[st->nfin - 1];
      }
      store_int(tgt, o, r);
    }
  } else if (st->reduce) {
    for (long long o = 0; o < span; o++) {
      if (!seen[o]) continue;
      float r = (float)acc[o];
      if (st->nfin > 0) {
        for (int i = 0; i < st->nfin; i++) val[i] = apply(&st->fin[i], val, r, 0.0f);
        r = val[st->nfin - 1];
      }
      store_elem(tgt, o, r);
    }
  }
  if (st->reduce) {
    free(acc);
    free(iacc);
    free(seen);
  }
  (void)narrays;
  return 0;
}

int orc_run(int nloops, const long long *extents, int narrays, orc_array *arrays,
            int nstatements, const orc_statement *statements, char *err, int errlen) {
  if (nloops < 0 || nloops > ORC_LOOPS) return fail(err, errlen, "bad loop count", -1);
  for (int l = 0; l < nloops; l++)
    if (extents[l] < 0) return fail(err, errlen, "loop extent < 0", -1);  /* 0: empty box domain */
  for (int s = 0; s < nstatements; s++) {
    const orc_statement *st = &statements[s];
    if (st->nloops < 1 || st->nloops > ORC_LOOPS) return fail(err, errlen, "bad statement loop count", s);
    for (int k = 0; k < st->nloops; k++) {
      if (st->loops[k] < 0 || st->loops[k] >= nloops) return fail(err, errlen, "bad loop id", s);
      for (int q = 0; q < k; q++)
        if (st->loops[q] == st->loops[k]) return fail(err, errlen, "loop listed twice", s);
    }
    if (st->nreads < 0 || st->nreads > ORC_READS) return fail(err, errlen, "bad read count", s);
    if (check_ref(&st->target, st, narrays, arrays, extents, s, err, errlen)) return 1;
    for (int r = 0; r < st->nreads; r++)
      if (check_ref(&st->reads[r], st, narrays, arrays, extents, s, err, errlen)) return 1;
    if (check_dag(st->nodes, st->nnodes, st->nreads, 0, s, err, errlen)) return 1;
    if (st->reduce && st->nfin > 0 && check_dag(st->fin, st->nfin, 0, 1, s, err, errlen)) return 1;
    if (check_types(st, arrays, s, err, errlen)) return 1;
    if (st->reduce)
      for (int r = 0; r < st->nreads; r++)
        if (st->reads[r].array == st->target.array)
          return fail(err, errlen, "reduce statement reads its own target", s);
    if (run_statement(st, extents, arrays, narrays, s, err, errlen)) return 1;
  }
  return 0;
}
