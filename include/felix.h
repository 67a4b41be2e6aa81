/* felix.h — C ABI of the B200-native Felix hot path (batched differentiable schedule search).
 *
 * Paper: Zhao, Sharif, Adve, Misailovic, "Felix: Optimizing Tensor Programs with Gradient Descent",
 * ASPLOS'24 (/root/reference/PAPER.md, cited "P:Lnnn").  The four primary calls follow the paper's
 * statement of the problem, Algorithm 1:
 *   felix_space_create    — one symbolic schedule s*_i: variables x_i, feature formulas Feat_k(x_i),
 *                           constraints g_ir(x_i) <= 0, divisibility splits
 *   felix_costmodel_load  — the pretrained MLP cost model C
 *   felix_search          — lines 12-19: init, then nSteps Adam steps on Eq. 4
 *   felix_round_topk      — lines 20-21: round to valid integer schedules, score, top-nMeasure
 *
 * plus test hooks (felix_eval, felix_round, felix_score, felix_init_sample) that run the same kernels.
 *
 * Conventions (all calls):
 *  - No exceptions cross the ABI.  Every call returns felix_status; on error felix_last_error()
 *    (thread-local, valid until the next felix_* call on this thread) describes it.  Argument and
 *    shape validation happens before any launch; a failed call leaves caller buffers untouched
 *    except where stated.
 *  - Handles are opaque and library-owned; *_destroy frees them (NULL is a no-op).
 *  - Host input arrays are COPIED at create/load time; the caller may free them on return.
 *  - "device" pointers are caller-owned CUDA device memory on the handle's device (e.g. torch
 *    tensors' data_ptr()); the library never frees them.  "host" pointers are ordinary host memory.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).  Calls enqueue work
 *    on it and return, except felix_round_topk, which synchronises `stream` because its outputs are
 *    host arrays.  Calls on one space must not run concurrently (the space owns its workspace).
 *  - Layouts: candidate-major SoA for per-candidate vectors: y[j * n + i] = y_j of candidate i.
 *  - The global index of local candidate i is index_base + i; it seeds the sampler and breaks top-k
 *    ties, which makes results invariant to how candidates are sharded over GPUs.
 *  - There is no CPU fallback: without a usable sm_100a device every call that needs one returns
 *    FELIX_E_CUDA.
 */
#ifndef FELIX_H_
#define FELIX_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define FELIX_ABI_VERSION 4

#if defined(__GNUC__)
#define FELIX_EXPORT __attribute__((visibility("default")))
#else
#define FELIX_EXPORT
#endif

typedef enum {
  FELIX_OK = 0,
  FELIX_E_INVALID_ARG = 1,   /* NULL / out-of-range argument                                   */
  FELIX_E_INVALID_DAG = 2,   /* node args not topological, bad opcode, type error (BOOL vs NUM) */
  FELIX_E_SHAPE = 3,         /* sizes inconsistent (e.g. n_features != cost-model dims[0])      */
  FELIX_E_UNSUPPORTED = 4,   /* valid but outside this build (e.g. hidden dim % 64 != 0)        */
  FELIX_E_CUDA = 5,          /* CUDA runtime/driver error or no sm_100 device                   */
  FELIX_E_NVRTC = 6,         /* run-time compilation of the space's expression kernels failed   */
  FELIX_E_OOM = 7            /* device allocation failed                                        */
} felix_status;

FELIX_EXPORT const char* felix_last_error(void);
FELIX_EXPORT int32_t felix_abi_version(void);

/* ---------------------------------------------------------------- feature-expression DAG
 * "each feature expression ... can only contain schedule variables, constants, and a
 * fixed set of operators ... +, -, *, /, pow, min, max, select, etc."  Nodes are given in
 * topological order; a, b, c index EARLIER nodes.  Values are NUM (real) or BOOL (comparisons and
 * logic).  Semantics used by the search ("smooth", reading O3 of DESIGN.md, with
 * S(t) = 1/2(1 + t/sqrt(1+t^2)) and R(t) = 1/2(t + sqrt(1+t^2))):
 *   MIN(a,b) = a - R(a-b)      MAX(a,b) = b + R(a-b)
 *   GT/GE(a,b) = S(a-b)        LT/LE(a,b) = S(b-a)      EQ = S(a-b+1/2) S(b-a+1/2)   NE = 1 - EQ
 *   AND = p q   OR = p + q - p q   NOT = 1 - p          SELECT(c,a,b) = b + (a-b) c
 *   FLOORDIV / CEILDIV(a,b) = a / b
 * and at integer points ("hard", used for validity and scoring): exact comparisons, SELECT picks a
 * branch, floor/ceil division.  VAR: imm = variable index j, value x_j = exp(y_j).
 * POW: a ^ imm (unary).  CONST: imm. */
typedef enum {
  FELIX_OP_CONST = 0, FELIX_OP_VAR = 1, FELIX_OP_ADD = 2, FELIX_OP_SUB = 3, FELIX_OP_MUL = 4,
  FELIX_OP_DIV = 5, FELIX_OP_NEG = 6, FELIX_OP_POW = 7, FELIX_OP_EXP = 8, FELIX_OP_LOG = 9,
  FELIX_OP_SQRT = 10, FELIX_OP_MIN = 11, FELIX_OP_MAX = 12, FELIX_OP_SELECT = 13,
  FELIX_OP_GT = 14, FELIX_OP_GE = 15, FELIX_OP_LT = 16, FELIX_OP_LE = 17, FELIX_OP_EQ = 18,
  FELIX_OP_NE = 19, FELIX_OP_AND = 20, FELIX_OP_OR = 21, FELIX_OP_NOT = 22,
  FELIX_OP_FLOORDIV = 23, FELIX_OP_CEILDIV = 24
} felix_op;

typedef struct { int32_t op, a, b, c; double imm; } felix_node;          /* 24 bytes */

/* Schedule variables (thread/block sizes, tile sizes, vector sizes, unroll factors;
 * "a size/factor of value 1 [is] a no-op").  SPLIT: a tiling factor x >= 1 whose products over each
 * split it belongs to divide the split's extent.  INT: an integer lo <= x <= hi. */
typedef enum { FELIX_VAR_SPLIT = 0, FELIX_VAR_INT = 1 } felix_var_kind;
typedef struct { int32_t kind; int32_t _pad; int64_t lo, hi; } felix_var;   /* 24 bytes */
typedef struct { int64_t extent; int32_t n; int32_t _pad; const int32_t* vars; } felix_split;

typedef struct felix_space felix_space;
typedef struct felix_costmodel felix_costmodel;

/* Creates a search space on `device`.
 * vars[n_vars], splits[n_splits] (each SPLIT var in >= 1 split; extents in [1, 2^31)),
 * nodes[n_nodes], feature_roots[n_features] (NUM nodes; n_features must equal the cost model's
 * dims[0] at search time, or S * dims[0] after felix_space_set_statements(S)),
 * constraint_roots[n_constraints] (NUM nodes, user g_r(x) <= 0).
 * The library appends the automatic log-space validity roots (reading O2), in this order
 * after the user roots:  -y_j for every SPLIT var;  sum_{j in s} y_j - ln(extent_s) per split;
 * ln(lo_j) - y_j and y_j - ln(hi_j) per INT var.  R = total number of roots (felix_space_info).
 * Builds the divisor-tuple tables of every split component with at most 65536 tuples (larger ones —
 * highly composite extents — are rounded by a branch-and-bound search over per-variable divisor lists,
 * same result; a component may hold at most 8 variables and touch at most 16 splits, else
 * FELIX_E_UNSUPPORTED), generates straight-line CUDA for the DAG (forward, reverse, hard, sampler) and
 * compiles it for sm_100a with NVRTC. */
FELIX_EXPORT felix_status felix_space_create(int device,
                                const felix_var* vars, int32_t n_vars,
                                const felix_split* splits, int32_t n_splits,
                                const felix_node* nodes, int32_t n_nodes,
                                const int32_t* feature_roots, int32_t n_features,
                                const int32_t* constraint_roots, int32_t n_constraints,
                                felix_space** out);
FELIX_EXPORT void felix_space_destroy(felix_space* s);

/* Per-statement features (TenSet-style segment sum; the paper's feature formulas are per statement,
 * P:L668-671): the feature roots are n_statements vectors of n_features /
 * n_statements features each, statement-major, and the cost is C = sum_s MLP(slog(Feat_s(x))) — every
 * statement's vector goes through the same MLP (head bias included) and the outputs are summed, for the
 * search objective (Eq. 4) and for the FP64 scores of rounded schedules alike.  Must be called before
 * any compute call (it drops the space's compiled kernels and workspaces).  FELIX_E_INVALID_ARG if
 * n_statements < 1 or does not divide n_features; FELIX_E_UNSUPPORTED if a vector is wider than 128. */
FELIX_EXPORT felix_status felix_space_set_statements(felix_space* s, int32_t n_statements);

/* Device-free check of a space description: validates it exactly like felix_space_create, generates
 * the space's CUDA source (for n_statements per-statement vectors, as felix_space_set_statements) and,
 * if compile != 0, compiles it with NVRTC for sm_100a (no GPU needed).
 * Copies up to src_cap bytes of source (NUL-terminated when it fits) into src (may be NULL) and
 * stores the full length in *src_len (may be NULL). */
FELIX_EXPORT felix_status felix_codegen(const felix_var* vars, int32_t n_vars,
                                        const felix_split* splits, int32_t n_splits,
                                        const felix_node* nodes, int32_t n_nodes,
                                        const int32_t* feature_roots, int32_t n_features,
                                        const int32_t* constraint_roots, int32_t n_constraints,
                                        int32_t n_statements, int32_t compile, char* src, int64_t src_cap,
                                        int64_t* src_len);

typedef struct {
  int32_t n_vars, n_nodes, n_features, n_constraints_user, n_roots_total, n_components;
  int64_t n_tuples_total;       /* rows of the divisor-tuple tables (branch-and-bound components: 0) */
  double nvrtc_ms;              /* time spent compiling the generated kernels                  */
  int32_t regs_fwd, regs_rev;   /* registers/thread of the generated forward / reverse kernels  */
  int64_t dag_flops_fwd;        /* arithmetic ops in one forward evaluation (per candidate)    */
  int64_t dag_flops_rev;        /* arithmetic ops of one reverse sweep over the whole DAG (per candidate,
                                   local partials + adjoint accumulations; the forward recompute excluded) */
} felix_space_info_t;
FELIX_EXPORT felix_status felix_space_info(const felix_space* s, felix_space_info_t* out);

/* Loads the cost model C: n_layers linear layers, dims[n_layers+1], dims[n_layers] == 1,
 * W[l] host row-major [dims[l+1]][dims[l]] fp32, b[l] host [dims[l+1]] fp32; ReLU between layers,
 * none after the last (TenSet MLP).  Hidden dims must be multiples of 64 and <= 1024,
 * dims[0] <= 256.  Weights are split on the host into fp16 hi/lo pairs for the tensor cores
 * and kept in fp64 for scoring. */
FELIX_EXPORT felix_status felix_costmodel_load(int device, int32_t n_layers, const int32_t* dims,
                                  const float* const* W, const float* const* b, felix_costmodel** out);
FELIX_EXPORT void felix_costmodel_destroy(felix_costmodel* m);

/* Algorithm 1 lines 12-19.  n_seeds candidates (nSeeds) x n_steps Adam steps (nSteps).
 * Per candidate the objective is Eq. 4:  L = -C(slog(Feat(e^y))) + lambda * sum_r max(g_r, 0)^2
 * (slog(F) = sign(F) log2(1+|F|), reading O4), differentiated w.r.t. y, then one torch.optim.Adam
 * step (bias-corrected, no weight decay) on y.  A candidate whose loss or gradient is
 * non-finite is not updated that step (reading R-NaN).
 * y: device fp32 SoA [n_vars][n_seeds].  If init_from_y == 0 it is OUTPUT-only and first filled by
 * the rejection sampler (felix_init_sample with rng_seed / index_base); else it is the start point.
 * final_loss: device fp32 [n_seeds] or NULL — the loss at the point of the last step's evaluation.
 * history != 0: also record varValuesHistory (Alg. 1 lines 13 and 17): every point at
 * which the objective is evaluated, sigma_x_i for i = 0 .. n_steps-1, is rounded on the device (same
 * rounding as felix_round_topk) and each schedule not seen before in this search is kept with its
 * first (step, global index); read the result with felix_history_topk.  Starting a search clears the
 * previous history.  Device memory grows with n_seeds x n_steps schedules (worst case). */
typedef struct {
  int64_t n_seeds;
  int32_t n_steps;
  float lr, beta1, beta2, eps, lambda;   /* reading O8 defaults: 0.05, 0.9, 0.999, 1e-8, 1.0 */
  uint64_t rng_seed;
  int32_t init_from_y;
  int32_t history;                       /* 0: round the final point only (felix_round_topk) */
  int64_t index_base;
} felix_search_params;
FELIX_EXPORT felix_status felix_search(felix_space* s, felix_costmodel* m, const felix_search_params* p,
                          float* y, float* final_loss, void* stream);

/* Several spaces (the tasks of one DNN, or the symbolic programs of one subgraph,
 * Eq. 3) searched together with ONE cost model: every Adam step runs each space's DAG
 * kernels on its own stream, then a single MLP pass (forward + input gradient) over the rows of all
 * spaces (the cost model is shared, Eq. 4 sums independent per-candidate terms), then each space's
 * reverse / Adam kernel.  Per space the result is what felix_search computes for it (same formulas,
 * per-candidate arithmetic; with the same MLP kernel bit for bit).
 * spaces[n_spaces], params[n_spaces], y[n_spaces] (device SoA [n_vars_i][n_seeds_i]), final_loss
 * [n_spaces] (NULL, or per-space device [n_seeds_i] / NULL).  All spaces on the cost model's device;
 * every params[i].n_steps equal; history must be 0 (FELIX_E_UNSUPPORTED otherwise).  The workspace
 * is cached on spaces[0] for the same (spaces, n_seeds, cost model). */
FELIX_EXPORT felix_status felix_search_group(felix_space* const* spaces, int32_t n_spaces, felix_costmodel* m,
                                             const felix_search_params* params, float* const* y,
                                             float* const* final_loss, void* stream);

/* Algorithm 1 lines 20-21 on the n relaxed points y (device SoA
 * [n_vars][n]): round every point (reading O10: per split component the divisor tuple nearest in
 * log space, ties to the lexicographically smallest; INT vars to the nearest integer), drop invalid
 * points (hard semantics, all user g_r <= 1e-9, finite), score C(slog(Feat_hard(x))) in FP64, drop
 * duplicate schedules (keep the smallest global index), return the best k by (score desc, global
 * index asc).  Outputs are HOST arrays: idx_out[k] global indices, score_out[k], sched_out[k][n_vars];
 * *n_out = number filled (<= k).  Synchronises `stream`. */
FELIX_EXPORT felix_status felix_round_topk(felix_space* s, felix_costmodel* m, const float* y, int64_t n,
                              int64_t index_base, int32_t k, int64_t* idx_out, double* score_out,
                              int32_t* sched_out, int32_t* n_out, void* stream);

/* Algorithm 1 lines 20-21 over the history of the last felix_search run with history != 0 (paper-
 * faithful Alg. 1: "takes all the variable values traversed in the optimization process, rounds them
 * to integers ... and removes invalid rounded schedules"): every distinct rounded schedule
 * visited at steps 0 .. n_steps-1 is validated (hard semantics) and scored in FP64 as in
 * felix_round_topk; the best k by (score desc, step asc, global index asc) are returned, each with the
 * first (step, global index) at which it was visited.  Outputs are HOST arrays: idx_out[k] global
 * indices, step_out[k], score_out[k], sched_out[k][n_vars]; *n_out = number filled (<= k);
 * *n_unique_out (may be NULL) = distinct schedules visited (valid or not).  Synchronises `stream`.
 * FELIX_E_INVALID_ARG if the last search did not record a history. */
FELIX_EXPORT felix_status felix_history_topk(felix_space* s, felix_costmodel* m, int32_t k, int64_t* idx_out,
                                int32_t* step_out, double* score_out, int32_t* sched_out, int32_t* n_out,
                                int64_t* n_unique_out, void* stream);

/* Multi-GPU exchange: candidates shard across ranks with no per-step communication
 * (Eq. 4 is a sum over seeds, Adam is elementwise); each rank's local top-k
 * records are all-gathered once and merged identically on every rank with this call.  Inputs are HOST
 * arrays of n_rows gathered records: key[n_rows] (the order key: global candidate index for
 * felix_round_topk, step * 2^40 + global index for felix_history_topk; < 0 marks an empty row),
 * score[n_rows] (FP64), sched[n_rows][n_vars] (int32).  Output: the best k distinct schedules by
 * (score desc, key asc), a schedule held by several rows kept once with its first row in that order
 * (a NaN score orders last) -- for any sharding, the single-process top-k of the union.  key_out[k],
 * score_out[k], sched_out[k][n_vars] HOST, caller-owned; *n_out = rows written (<= k).  Host only (no
 * device, no stream).  FELIX_E_INVALID_ARG on NULL pointers with n_rows > 0, n_vars < 1 or k < 0. */
FELIX_EXPORT felix_status felix_merge_topk(const int64_t* key, const double* score, const int32_t* sched,
                              int64_t n_rows, int32_t n_vars, int32_t k, int64_t* key_out, double* score_out,
                              int32_t* sched_out, int32_t* n_out);

/* ---------------------------------------------------------------- test hooks (same kernels)
 * felix_eval: one objective + gradient evaluation, no Adam.  y device [n_vars][n].  Outputs (device,
 * any may be NULL): phi [n_features][n] (slog features), g [R][n] (user roots then automatic roots),
 * cost [n] (C, higher = better), loss [n], grad [n_vars][n] (dL/dy). */
FELIX_EXPORT felix_status felix_eval(felix_space* s, felix_costmodel* m, const float* y, int64_t n, float lambda,
                        float* phi, float* g, float* cost, float* loss, float* grad, void* stream);
/* felix_eval_ex: felix_eval with two more views of the same evaluation (test hooks for the north star's
 * parity bars).  All outputs device, any may be NULL:
 *   phi, g, cost, loss, grad   as felix_eval
 *   F        double [n_features][n]: the raw smoothed features Feat_k(e^y) before slog (P:L688-766,
 *            reading O3), FP64, from the same forward code as phi — the "feature <= 1e-4" bar is on F.
 *   search_path != 0: evaluate through the kernels and launch configuration of one felix_search Adam
 *            step instead (split-cone reverse kernel: per-cone partial adjoints summed in fixed order by
 *            the kernel that applies Adam in a search), writing the loss and the dL/dy that
 *            step's Adam update would use; y is not modified.  Only loss and grad may be non-NULL
 *            (FELIX_E_INVALID_ARG otherwise). */
typedef struct {
  float* phi; float* g; float* cost; float* loss; float* grad;
  double* F;
  int32_t search_path;
  int32_t _pad;
} felix_eval_out;
FELIX_EXPORT felix_status felix_eval_ex(felix_space* s, felix_costmodel* m, const float* y, int64_t n, float lambda,
                                        const felix_eval_out* out, void* stream);
/* Rounding + validity only: sched device int32 [n][n_vars], valid device uint8 [n]. */
FELIX_EXPORT felix_status felix_round(felix_space* s, const float* y, int64_t n, int32_t* sched, uint8_t* valid,
                         void* stream);
/* FP64 score of integer schedules sched (device int32 [n][n_vars]) -> score device double [n]. */
FELIX_EXPORT felix_status felix_score(felix_space* s, felix_costmodel* m, const int32_t* sched, int64_t n,
                         double* score, void* stream);
/* Rejection sampler of Algorithm 1 line 12 (reading O9): y device fp32 [n_vars][n].
 * u(seed, cand, attempt, var) = splitmix64 finaliser chained over (seed, cand+1, attempt+1, var+1)
 * (each step h = mix(h + 0x9E3779B97F4A7C15 * k)), top 53 bits / 2^53.  For outer attempt a2 < 64:
 * each split component draws y_j = u(.., 64*a2 + a1, j) ln(ub_j) for a1 < 64 until its split roots
 * are <= 0; INT vars y_j = ln lo + u(.., 64*a2, j)(ln hi - ln lo); accept when every user root
 * (smooth) is <= 0.  Fallback y = ln(lo). */
FELIX_EXPORT felix_status felix_init_sample(felix_space* s, int64_t n, uint64_t rng_seed, int64_t index_base,
                               float* y, void* stream);

/* Process-wide execution knobs for experiments and tests; normal use needs none (the defaults are the
 * measured choices of DESIGN.md; every knob gives the same results up to fp32 summation order).  The
 * library never reads environment variables.  key / value (-1 = default):
 *   "mlp"                 0 tile kernel, 1 persistent layer chain, 2 one GEMM kernel per layer
 *   "cone_width"          cone-partition width P of the expression kernels: 1, 2, 4, 8, 16
 *   "replicas"            cone-group replicas per block: 1, 2, 4
 *   "sc_warps"            warps per split-cone reverse CTA: 1..8
 *   "chunks"              concurrent population chunks: 1..16
 *   "split_cone"          0 cone-group reverse + Adam kernel, 1 split-cone reverse kernel
 *   "tile_cta_group"      tile kernel on 1-SM tiles (1) or 2-SM cta_group::2 pairs (2)
 *   "chain_cta_group"     layer chain on 1-SM 128-row tiles (1) or 2-SM cta_group::2 256-row pairs (2)
 *   "dphi_ksplit"         layer chain: split-K parts of the dL/dphi layer, 1, 2 or 4 (partial slabs summed
 *                         in fixed order by the reverse kernel)
 *   "codegen_cone_width", "codegen_replicas"   the variant felix_codegen emits
 *   "trace"               0/1: per-block %globaltimer stamps in kernels generated afterwards
 *   "round_bnb"           0/1: 1 = every split component is rounded by the branch-and-bound kernel
 *                         (default 0: only components with more than 65536 divisor tuples are)
 *   "graph_steps"         Adam steps captured per search graph: 1..1000 (default 20)
 *   "dphi_tma"            layer chain: the dL/dphi tile written by one TMA store (1, default) or per-thread stores (0)
 *   "score_dmma"          FP64 scoring layers on the FP64 tensor cores (1, default) or the CUDA cores (0)
 *   "pdl"                 programmatic-dependent-launch edges, bit mask: 1 forward DAG kernel, 2 MLP kernels,
 *                         4 reverse and other kernels (default 0: none, measured faster)
 * FELIX_E_INVALID_ARG for an unknown key or value. */
FELIX_EXPORT felix_status felix_tune(const char* key, int32_t value);

/* Per-kernel-class device time accumulated by felix_search while profiling is enabled (CUDA events
 * on the search stream).  Classes: 0 DAG forward, 1 MLP GEMMs, 2 DAG reverse+Adam, 3 other.
 * ms[4], launches[4]; reset with felix_profile_reset. */
FELIX_EXPORT felix_status felix_profile_enable(felix_space* s, int32_t enable);
FELIX_EXPORT felix_status felix_profile_read(felix_space* s, double* ms, int64_t* launches);
FELIX_EXPORT felix_status felix_profile_reset(felix_space* s);
/* Debug: copy the per-block %globaltimer stamps of the generated kernels (only for kernels generated
 * after felix_tune("trace", 1)): uint64 [2][8192][8] = {forward, reverse} x block x stamp.  Forward
 * (felix_fwd / felix_fwd_adam): start, after griddepcontrol.wait, after the Adam prologue, after the cone
 * compute, end.  Split-cone reverse: start, after wait, after compute, end; cone-group reverse: slots
 * 4..7.  If n_words exceeds 2 * 8192 * 8, the forward kernel's per-warp cone-end stamps [8192][16] follow.
 * Only the last launch's stamps survive.  n_words bounds the copy. */
FELIX_EXPORT felix_status felix_debug_trace(felix_space* s, uint64_t* out, int64_t n_words);

#ifdef __cplusplus
}
#endif
#endif /* FELIX_H_ */
