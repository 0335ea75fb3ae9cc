/*
 * fop.h — C ABI of the B200-native fused-operator library (libfop.so).
 *
 * A fused AI/DL operator is given the way the paper states its problem
 * (§II-§III): an ordered list of STATEMENTS over
 * TENSORS.  Each statement runs over a box iteration domain
 * D_S(p) = { i | 0 <= i_l < E_l } (eqs for D_X, D_Y), has one write
 * access and several read accesses, and an expression DAG (the abstract
 * f, g of Fig. 2).  Access functions are "either a constant or an
 * affine form where only one loop iterator is present with coefficient 1"
 * — that is exactly fop_access below.
 *
 * Reading (reading D1): loops are declared once for the whole fused
 * operator (fop_desc.extent[]) and each statement lists the loops it iterates,
 * outermost first.  Two statements that list the same loop id share that
 * iterator (the i/k of Fig. 2's X and Y).  This is how the dependence relation
 * delta_{X->Y} of P:149 (i_X = i_Y, k_X = k_Y) is expressed without isl.
 *
 * Semantics (what every result must equal, checked against oracle/):
 * statements execute in textual order; each iterates its loops in
 * lexicographic order (the schedule theta of P:119-121); ASSIGN stores the DAG
 * value converted (RNE) to the write tensor's dtype; REDUCE overwrites each
 * output element with op-reduce over the statement's reduction loops (loops on
 * which the write access does not depend) of the DAG value, then applies the
 * finalize DAG (e.g. /768 for a mean); a later statement reads the STORED
 * (rounded) values.  Arithmetic nodes are fp32; add/sub/mul/div/sqrt are IEEE
 * correctly rounded and never contracted (divisions too: the kernels' fast form
 * for a loop-invariant divisor returns the correctly rounded quotient).
 *
 * Integer statements (reading R30): a statement whose write tensor is
 * FOP_I32 (and that is not a pure element move) computes on int32 values — it
 * reads i32 tensors only, its DAG uses ADD SUB MUL MAX MIN NEG ABS RELU and
 * CONST with an integral immediate, every result wraps modulo 2^32 (two's
 * complement), REDUCE SUM is the sum modulo 2^32 (any association order gives
 * the same bits) and MAX the maximum.  A float statement reads no i32 tensor.
 * Anything else on i32 (DIV, SQRT, transcendentals, CAST to i32, a fractional
 * immediate, mixing i32 and float tensors) is FOP_E_INVALID.  A pure move
 * copies any dtype bit for bit.
 *
 * Ownership: the caller owns every buffer (host descriptors, device tensors,
 * workspace).  fop_plan copies the descriptor; a plan is immutable after
 * fop_plan returns and may be run concurrently on several streams (only the
 * lazy per-context module load takes an internal lock).  No function throws or
 * aborts across the ABI: every failure is a fop_status plus a thread-local
 * message (fop_last_error).
 */
#ifndef FOP_H
#define FOP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define FOP_API __attribute__((visibility("default")))
#else
#define FOP_API
#endif

#define FOP_ABI_VERSION 4

#define FOP_MAX_RANK     8   /* tensor rank */
#define FOP_MAX_LOOPS    8   /* loops of the fused operator */
#define FOP_MAX_TENSORS 16
#define FOP_MAX_STMTS    8
#define FOP_MAX_ACC      8   /* accesses per statement; acc[0] is the write */
#define FOP_MAX_NODES   48   /* DAG nodes per statement */
#define FOP_MAX_FIN      8   /* finalize nodes per REDUCE statement */
#define FOP_MAX_LAUNCH   8   /* kernel launches per plan */
#define FOP_MAX_SCEN     8   /* scenarios kept per statement ("set to 8") */
#define FOP_MAX_DEPS    16   /* dependence vectors reported per statement */
#define FOP_MAX_PEERS    8   /* GPUs of one peer group (one NVLink/NVSwitch node) */

typedef enum {
  FOP_OK = 0,
  FOP_E_INVALID = 1,     /* malformed descriptor / arguments */
  FOP_E_UNSUPPORTED = 2, /* valid, but outside what the kernels implement */
  FOP_E_ALIGN = 3,       /* pointer alignment violates the tensor dtype itself */
  FOP_E_CUDA = 4,        /* CUDA driver failure (no driver, launch error, ...) */
  FOP_E_NOMEM = 5,
  FOP_E_JIT = 6          /* NVRTC compilation of a generated kernel failed */
} fop_status;

typedef enum { FOP_F32 = 0, FOP_F16 = 1, FOP_BF16 = 2, FOP_I32 = 3 } fop_dtype;

/* IN: read only.  OUT: written.  INOUT: read and written.  TEMP: an
 * intermediate of the fused operator (graph-kernel fusion removes
 * intermediate allocations); its pointer may be NULL — the plan either
 * keeps it in registers or places it in the workspace. */
typedef enum { FOP_IN = 1, FOP_OUT = 2, FOP_INOUT = 3, FOP_TEMP = 4 } fop_role;

typedef enum { FOP_ASSIGN = 0, FOP_REDUCE = 1 } fop_kind;
typedef enum { FOP_RED_SUM = 0, FOP_RED_MAX = 1 } fop_reduce_op;

typedef enum {
  FOP_OP_LOAD = 0,      /* a = read access index (1..nacc-1) */
  FOP_OP_CONST = 1,     /* imm (fp32; an integral value in int32 range in an integer statement) */
  FOP_OP_ACC = 2,       /* finalize DAG only: the reduced value */
  FOP_OP_ADD = 3, FOP_OP_SUB = 4, FOP_OP_MUL = 5, FOP_OP_DIV = 6,
  FOP_OP_MAX = 7, FOP_OP_MIN = 8,          /* fmaxf/fminf semantics */
  FOP_OP_NEG = 9, FOP_OP_ABS = 10, FOP_OP_SQRT = 11,
  FOP_OP_RELU = 12,     /* v > 0 ? v : +0 (reading R15) */
  FOP_OP_EXP = 13, FOP_OP_LOG = 14, FOP_OP_TANH = 15, FOP_OP_SIGMOID = 16,
  FOP_OP_GELU_TANH = 17, /* 0.5 v (1 + tanh(sqrt(2/pi)(v + 0.044715 v^3))) */
  FOP_OP_GELU_ERF = 18,  /* 0.5 v (1 + erf(v / sqrt 2)) */
  FOP_OP_CAST = 19,      /* round a to dtype `cvt`, value continues as fp32 */
  FOP_OP__COUNT = 20
} fop_opcode;

typedef struct {
  int32_t rank;
  int32_t dtype;                 /* fop_dtype */
  int32_t role;                  /* fop_role */
  int32_t _pad;
  int64_t shape[FOP_MAX_RANK];
  int64_t stride[FOP_MAX_RANK];  /* in ELEMENTS; 0 allowed (expand-style broadcast) */
} fop_tensor;

/* index_r = (loop[r] >= 0 ? i_{loop[r]} : 0) + offset[r]     (P:355 access form) */
typedef struct {
  int32_t tensor;
  int32_t loop[FOP_MAX_RANK];    /* global loop id per tensor dim, -1 = constant */
  int64_t offset[FOP_MAX_RANK];
} fop_access;

typedef struct {
  int32_t op;                    /* fop_opcode */
  int32_t a, b;                  /* operand node indices (earlier nodes) or access index */
  int32_t cvt;                   /* fop_dtype for FOP_OP_CAST */
  float imm;                     /* FOP_OP_CONST */
  int32_t _pad;
} fop_node;

typedef struct {
  int32_t kind;                  /* fop_kind */
  int32_t reduce_op;             /* fop_reduce_op (REDUCE only) */
  int32_t nloops;
  int32_t loop[FOP_MAX_LOOPS];   /* loop ids, outermost first (original nest order) */
  int32_t nacc;
  fop_access acc[FOP_MAX_ACC];   /* acc[0] = write access */
  int32_t nnodes;
  fop_node node[FOP_MAX_NODES];  /* topological; the statement value is the last node */
  int32_t nfin;
  fop_node fin[FOP_MAX_FIN];     /* REDUCE finalize DAG over FOP_OP_ACC/CONST; empty = identity */
} fop_stmt;

typedef struct {
  int32_t nloops;
  int64_t extent[FOP_MAX_LOOPS]; /* E_l >= 1 (box domain) */
  int32_t ntensors;
  fop_tensor t[FOP_MAX_TENSORS];
  int32_t nstmts;
  fop_stmt s[FOP_MAX_STMTS];
} fop_desc;

/* Planner options.  fop_plan_opts_default() fills the paper's values:
 * W = (5,3,1,1,1), L = 1024 (reading R5), 8 scenarios,
 * 16-byte vectors (128-bit), readings R1 + R6 on. */
enum {
  FOP_READING_R1_THREAD_TERM = 1,  /* w5*F*N/L instead of the printed w5*F*L/N (P:338 vs P:347) */
  FOP_READING_R6_STRIDE1_C   = 2   /* |C| counts only stride-1 accesses */
};
enum { FOP_ORDER_PAPER = 0, FOP_ORDER_MEMORY = 1 };

typedef struct {
  double w[5];
  int32_t thread_limit;          /* L of Algorithm 2 */
  int32_t max_scenarios;
  int32_t max_vec_bytes;         /* 16 (LDG/STG.128) or 32 (LDG/STG.256, sm_100a) */
  int32_t readings;              /* FOP_READING_* bit set */
  int32_t force_width;           /* 0 = planner decides; k = cap vector width at k elements (1 = "novec") */
  int32_t coalesce_order;        /* FOP_ORDER_PAPER: threads follow the scenario order; MEMORY: write-memory order */
  int32_t sm_count;              /* 0 = 148 (B200); used for grid sizing */
  int32_t jit;                   /* 1 = compile kernels at fop_plan (NVRTC, sm_100a); 0 = analysis only */
  int32_t autotune;              /* 1 = compile a few geometry variants per launch; the first fop_run on a
                                    context times them on the caller's stream (synchronising once) and
                                    keeps the fastest (tile sizes are auto-tuned in the paper too).
                                    Skipped for plans that are not idempotent (in-place / read-modify-write)
                                    and while the stream is being captured into a CUDA graph. */
  /* Multi-GPU (BASELINE.json north_star (4)).  peer_world >= 1: the operator is ONE
     shard of a larger one whose loop `peer_loop` is split into peer_world contiguous blocks, one per
     GPU (every rank plans the same shard descriptor).  Each REDUCE statement whose reduction loops
     include peer_loop then combines the partial results of all ranks INSIDE its kernel: the
     COL_REDUCE epilogue pushes the rank's per-slab sums into every rank's exchange buffer over
     NVLink peer memory, waits for the others' pushes, and adds the world contributions in rank
     order (identical bits on every rank), then finalizes and stores.  Run with fop_run_peer.
     0 = no exchange (the default). */
  int32_t peer_world;
  int32_t peer_loop;             /* loop id split across the peer group (peer_world >= 1) */
  int32_t peer_timeout_ms;       /* bound on a kernel's wait for its peers; 0 = 10000.  On timeout the
                                    run's exchanged outputs are NaN and the exchange buffer's error word
                                    is set (fop_peer_group) */
  int32_t variant;               /* -1 (default): auto-tune as above.  k >= 0: no timing; every launch runs
                                    its tuning candidate k (0 = the default geometry; a launch with fewer
                                    candidates, see fop_launch_info.nvariants, runs its default).  Lets a
                                    test run each candidate the tuner could pick (they must all agree with
                                    the oracle: schedules are semantics preserving). */
} fop_plan_opts;

typedef enum {
  FOP_CLASS_EW = 0,          /* elementwise / broadcast */
  FOP_CLASS_TRANSPOSE = 1,   /* store-contiguous loop != load-contiguous loop */
  FOP_CLASS_ROW_REDUCE = 2,  /* vector loop is a reduction loop */
  FOP_CLASS_COL_REDUCE = 3   /* vector loop is parallel, reduction elsewhere */
} fop_kernel_class;

typedef struct {
  int32_t kernel_class;      /* fop_kernel_class */
  int32_t main_stmt;
  uint32_t stmt_mask;        /* statements fused into this launch (bit s) */
  int32_t vec_loop;          /* loop id carrying the explicit vector type */
  int32_t width;             /* elements per vector access on the write side */
  int32_t read_loop;         /* TRANSPOSE: loop contiguous for the transposed read, else -1 */
  int32_t read_width;        /* TRANSPOSE: elements per read vector */
  int32_t coal_loop;         /* next loop mapped to threads (scenario goal (ii)), -1 if none */
  int64_t grid;
  int32_t block;
  int32_t nseq;              /* loops each thread walks in order (read-modify-write / recurrence), 0 = none */
  int32_t seq[FOP_MAX_LOOPS];/* their ids, outermost first */
  int32_t scen_pick;         /* scenario whose innermost loop is d_v; -1 = none feasible (row N3) */
  int32_t fallback;          /* row N3 influence-tree outcome: 0 scenario as ranked, 1 looser variant (vector
                                constraint only), 2 no feasible scenario: uninfluenced schedule, no
                                explicit vector type, 3 fully sequential (every loop carries a
                                dependence) */
  int32_t peer_exchange;     /* 1: this launch combines partial results across the peer group */
  int32_t nvariants;         /* tuning candidates compiled for this launch, the default geometry included */
} fop_launch_info;

typedef struct {
  int32_t nstmts;
  int32_t nscen[FOP_MAX_STMTS];                        /* scenarios kept per statement */
  int32_t scen_len[FOP_MAX_STMTS][FOP_MAX_SCEN];
  int32_t scenario[FOP_MAX_STMTS][FOP_MAX_SCEN][3];    /* loop ids, outermost -> innermost */
  double  inner_score[FOP_MAX_STMTS][FOP_MAX_LOOPS];   /* cost at the innermost position, by stmt loop position */
  int32_t nlaunch;
  fop_launch_info launch[FOP_MAX_LAUNCH];
  size_t  workspace_bytes;
  /* validity: uniform self-dependences per statement — distance vectors by loop id,
     lexicographically positive in the statement's loop order; anti = the read precedes the write */
  int32_t ndeps[FOP_MAX_STMTS];
  int64_t dep[FOP_MAX_STMTS][FOP_MAX_DEPS][FOP_MAX_LOOPS];
  int32_t dep_anti[FOP_MAX_STMTS][FOP_MAX_DEPS];
} fop_plan_info;

typedef struct fop_plan fop_plan_t;   /* opaque, immutable after fop_plan */

FOP_API int         fop_abi_version(void);
FOP_API void        fop_plan_opts_default(fop_plan_opts* opts);

/* Validate the descriptor (row a1), analyse strides (a2), rank scenarios with
 * Algorithm 2 + cost() (a3), choose widths (a4), kernel classes and
 * launches (a5), generate and (opts->jit) compile the kernels for sm_100a.
 * Host only: needs neither a GPU nor a CUDA context.  opts may be NULL
 * (= fop_plan_opts_default).  On failure *out is NULL. */
FOP_API fop_status  fop_plan(const fop_desc* desc, const fop_plan_opts* opts, fop_plan_t** out);
FOP_API fop_status  fop_plan_info_get(const fop_plan_t* plan, fop_plan_info* out);
FOP_API size_t      fop_plan_workspace_bytes(const fop_plan_t* plan);
/* Generated CUDA source / compiled cubin of launch i (inspection, tests).
 * fop_plan_source also takes i = -1 - k: the source of launch k's narrow
 * variant (the kernel run for base pointers off the planned alignment).
 * Pointers stay owned by the plan. */
FOP_API fop_status  fop_plan_source(const fop_plan_t* plan, int32_t launch, const char** src);
FOP_API fop_status  fop_plan_cubin(const fop_plan_t* plan, int32_t launch, const void** data, size_t* size);

/* Run the fused operator.  dev_ptrs[i] = device base address of desc.t[i]
 * (NULL allowed for TEMP tensors), nptrs = desc.ntensors.  workspace: device
 * buffer of fop_plan_workspace_bytes() bytes, ZERO-FILLED before its first use
 * with this plan, NULL if 0 bytes.  It holds COL_REDUCE arrival counters (the
 * kernels return each to zero) and partial / folded sums (every value a run
 * reads was written earlier in that run), so it stays valid run after run; one
 * workspace serves one run at a time (concurrent runs need one each).
 * stream: a CUstream / cudaStream_t (NULL = legacy default stream) of the
 * CURRENT CUDA context.  Asynchronous and stream-ordered.  A base pointer that
 * is not aligned for the planned vector width silently selects a narrower
 * variant (same bits).  Returns FOP_E_CUDA if the driver or launch fails. */
FOP_API fop_status  fop_run(const fop_plan_t* plan, void* const* dev_ptrs, int32_t nptrs,
                    void* workspace, void* stream);

/* End-to-end variant: host_ptrs[i] are PINNED host buffers (dense, same
 * layout as desc.t[i]); IN/INOUT tensors are copied host->device, the
 * operator runs, OUT/INOUT tensors are copied device->host, all enqueued on
 * `stream`.  The caller synchronises the stream before reading host_ptrs. */
FOP_API fop_status  fop_run_host(const fop_plan_t* plan, void* const* host_ptrs,
                         void* const* dev_ptrs, int32_t nptrs, void* workspace, void* stream);

/* End to end for n INDEPENDENT plans (no plan reads what another writes):
 * plan k takes host_ptrs[k] / dev_ptrs[k] (nptrs[k] entries each, as in
 * fop_run_host; a NULL host pointer skips that tensor's copy) and
 * workspaces[k] (workspaces may be NULL when no plan needs one).  The copies
 * are pipelined: inputs host->device in order on an internal copy stream,
 * plan k runs on `stream` once its inputs are in, its outputs go
 * device->host on a second internal copy stream while later inputs are still
 * arriving (PCIe is full duplex).  Being independent, the plans run in the
 * order that minimises the two-direction copy makespan (Johnson's rule for
 * a two-machine flow shop; ties keep the given order).  The first copies wait for work already on
 * `stream`; `stream` waits for the last copy, so the call is ordered like one
 * fop_run_host on `stream`.  Asynchronous; the caller synchronises `stream`
 * before reading host buffers.  Host buffers should be pinned.  The internal
 * streams are created once per context and live for the process. */
FOP_API fop_status  fop_run_host_many(const fop_plan_t* const* plans, void* const* const* host_ptrs,
                                      void* const* const* dev_ptrs, const int32_t* nptrs,
                                      void* const* workspaces, int32_t n, void* stream);

/* ---------------------------------------------------------------- peer groups (multi-GPU)
 * Cross-GPU reductions fused into the reducing kernel (plans with
 * opts.peer_world >= 1, see fop_plan_opts).  Every rank owns one EXCHANGE
 * BUFFER of fop_plan_peer_bytes() bytes, zero-filled before first use, and maps
 * every other rank's buffer into its address space (fop_peer_alloc on the
 * owner, the 64-byte handle sent to the others by any means, fop_peer_open
 * there; CUDA IPC, so peers are GPUs of one node reached over NVLink /
 * NVSwitch).  Layout of a buffer, per exchanging launch: [2 parities][world
 * senders][slabs][slab columns] 64-bit words (fp32 partial sum in the low
 * half, the run's epoch in the high half: one single-copy-atomic store
 * carries both the value and its arrival flag), then [slabs] local run
 * counters; the LAST 16 bytes hold an error word (nonzero = a wait timed
 * out).  The kernels keep the buffer consistent across runs: the buffer must
 * not be touched between runs, and every rank must run the plan the same
 * number of times, in the same order relative to the plan's other runs. */
typedef struct { unsigned char bytes[64]; } fop_ipc_handle;
typedef struct {
  int32_t rank;                      /* this GPU's index in the group, 0 <= rank < world */
  int32_t world;                     /* must equal the plan's opts.peer_world */
  void* buf[FOP_MAX_PEERS];          /* every rank's exchange buffer as addressed from THIS process;
                                        buf[rank] = the local one */
} fop_peer_group;

/* Size of the exchange buffer (0 for plans without peer exchange). */
FOP_API size_t      fop_plan_peer_bytes(const fop_plan_t* plan);
/* fop_run for plans with a peer exchange: every rank of the group calls it
 * (typically on its own GPU, one process per GPU) and each launch waits, on
 * the device, for the other ranks' matching launch.  Tuning is disabled for
 * exchanging launches (all ranks must run the same geometry) and a
 * misaligned tensor pointer returns FOP_E_ALIGN before anything is launched.
 * Plans without exchange accept group = NULL (then it is fop_run). */
FOP_API fop_status  fop_run_peer(const fop_plan_t* plan, void* const* dev_ptrs, int32_t nptrs,
                                 void* workspace, const fop_peer_group* group, void* stream);
/* Exchange buffers: device memory on the current context's GPU, zero-filled,
 * owned by libfop until fop_peer_free; `handle` lets other processes map it. */
FOP_API fop_status  fop_peer_alloc(size_t bytes, void** dev_ptr, fop_ipc_handle* handle);
FOP_API fop_status  fop_peer_free(void* dev_ptr);
/* Map another process's exchange buffer (peer access over NVLink is enabled
 * lazily); unmap with fop_peer_close.  A handle of this same process's buffer
 * is rejected by CUDA: use the pointer itself. */
FOP_API fop_status  fop_peer_open(const fop_ipc_handle* handle, void** dev_ptr);
FOP_API fop_status  fop_peer_close(void* dev_ptr);

/* fop_run for n INDEPENDENT plans (no plan reads or writes what another
 * writes), back to back on `stream` in the given order: plan k's first kernel
 * is launched with programmatic stream serialization (its launch is
 * processed while plan k-1's last kernel still runs; the kernels carry no
 * explicit trigger, so plan k starts when plan k-1 completes and stream
 * order is kept; later work on `stream` sees every result).  dev_ptrs[k],
 * nptrs[k], workspaces[k] (may be NULL) as in fop_run.  Plans with a peer
 * exchange are rejected (FOP_E_INVALID): run them with fop_run_peer. */
FOP_API fop_status  fop_run_many(const fop_plan_t* const* plans, void* const* const* dev_ptrs,
                                 const int32_t* nptrs, void* const* workspaces, int32_t n, void* stream);

/* The kernel fop_run launches for `launch` on the current CUDA context (after
 * auto-tuning; the default geometry before the first run): its name, grid and
 * block.  Pointers stay owned by the plan. */
FOP_API fop_status  fop_plan_selected(const fop_plan_t* plan, int32_t launch, const char** kernel_name,
                                      int64_t* grid, int32_t* block);

FOP_API void        fop_plan_destroy(fop_plan_t* plan);
FOP_API const char* fop_status_str(fop_status s);
FOP_API const char* fop_last_error(void);      /* thread-local detail of the last failure */

#ifdef __cplusplus
}
#endif
#endif /* FOP_H */
