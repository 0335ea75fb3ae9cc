/*
 * fop_oracle.h — TEST INFRASTRUCTURE ONLY (parity oracle).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load liboracle.so.  The product path
 * (paper_conf_cgo_bastoulzrlsjfjc22_b200, include/fop.h) never includes this
 * header and never links this library; the two share no code or types.
 *
 * A plain, slow loop-nest evaluator of a fused operator (§III,
 * P:97-133): statements in textual order, each iterating its box domain in
 * lexicographic order — the original schedule theta_X = (0,i,k,0),
 * theta_Y = (1,i,j,k) of P:119-121.  The paper's scheduling and
 * vectorisation are semantics preserving (validity constraints, eq. (1),
 * P:145-157; "the scheduling algorithm will build correct scheduling
 * functions"), so the original order defines every result.
 */
#ifndef FOP_ORACLE_H
#define FOP_ORACLE_H

#include <stdint.h>

#define ORC_RANK 8
#define ORC_LOOPS 8
#define ORC_READS 8
#define ORC_NODES 64

/* element types */
enum { ORC_F32 = 0, ORC_F16 = 1, ORC_BF16 = 2, ORC_I32 = 3 };

/* node kinds (the oracle's own numbering) */
enum {
  ORC_LOAD = 1, ORC_CONST, ORC_ACC,
  ORC_ADD, ORC_SUB, ORC_MUL, ORC_DIV, ORC_MAX, ORC_MIN,
  ORC_NEG, ORC_ABS, ORC_SQRT, ORC_RELU,
  ORC_EXP, ORC_LOG, ORC_TANH, ORC_SIGMOID, ORC_GELU_TANH, ORC_GELU_ERF,
  ORC_CAST
};

typedef struct {
  void *data;                 /* host buffer, caller owned */
  int elem;                   /* ORC_F32 ... */
  int rank;
  long long shape[ORC_RANK];
  long long stride[ORC_RANK]; /* elements */
} orc_array;

typedef struct {
  int array;                  /* index into the array table */
  int iter[ORC_RANK];         /* loop id per array dim, or -1 */
  long long off[ORC_RANK];
} orc_ref;

typedef struct {
  int kind;                   /* ORC_* */
  int x, y;                   /* operand node indices, or read index for LOAD */
  int elem;                   /* CAST target */
  double c;                   /* CONST value (an fp32 value) */
} orc_node;

typedef struct {
  int reduce;                 /* 0 = assign, 1 = reduce */
  int reduce_max;             /* reduce: 0 = sum, 1 = max */
  int nloops;
  int loops[ORC_LOOPS];       /* loop ids, outermost first */
  orc_ref target;             /* write */
  int nreads;
  orc_ref reads[ORC_READS];
  int nnodes;
  orc_node nodes[ORC_NODES];
  int nfin;
  orc_node fin[ORC_NODES];
} orc_statement;

/* Run all statements in order.  Returns 0 on success, else nonzero with a
 * message in err.  extents[l] = E_l of loop l. */
int orc_run(int nloops, const long long *extents,
            int narrays, orc_array *arrays,
            int nstatements, const orc_statement *statements,
            char *err, int errlen);

/* exposed for the conversion pins */
uint16_t orc_f32_to_f16(float f);
float orc_f16_to_f32(uint16_t h);
uint16_t orc_f32_to_bf16(float f);
float orc_bf16_to_f32(uint16_t h);
float orc_gelu_tanh(float v);

#endif
