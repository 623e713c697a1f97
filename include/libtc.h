/*
 * libtc.h — C ABI of libtc: direct (transpose-free) contraction of two dense tensors on
 * NVIDIA B200 (sm_100a).
 *
 * The operation (Section II, eq. (1) and the sum below it):
 *     C[a,b,c,d] = sum_{e,f} A[a,e,b,f] * B[d,f,c,e]
 * generalised with the Einstein convention to any expression in which every index
 * occurs in exactly two of the three tensors — or in all three: a batch (Hadamard)
 * index, not summed (reading R31) — and with the update
 *     C = alpha * sum_int A * B + beta * C          (beta == 0: C is never read)
 * (reading R3).  No transposed intermediate is ever created.
 *
 * Layout: every tensor is dense and the FIRST listed index of each
 * tensor is its fastest varying index (stride 1): offset = sum_k i_k * prod_{j<k} N_j.
 * As a row-major torch tensor the shape is the reversed index list.
 *
 * Functions are nothrow: no C++ exception crosses this boundary; every failure is a status
 * code plus a thread-local detail string (tc_last_error).  The library never aborts.
 */
#ifndef LIBTC_H
#define LIBTC_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st *tc_stream_t; /* == cudaStream_t; NULL = legacy default stream */

typedef enum { TC_F64 = 0, TC_F32 = 1, TC_TF32 = 2, TC_BF16 = 3 } tc_dtype_t;

typedef enum {
  TC_SUCCESS = 0,
  TC_ERR_INVALID_ARG = 1, /* NULL pointer/handle, C overlaps A or B, wrong device, bad opts */
  TC_ERR_PARSE = 2,       /* malformed expression or extents string                          */
  TC_ERR_INDEX = 3,       /* index in one tensor only (an index in all three is a legal batch
                             index, R31), repeated in a tensor, extent missing / duplicated /
                             naming an unknown index                                         */
  TC_ERR_EXTENT = 4,      /* extent < 1, or an element count overflows int64                 */
  TC_ERR_UNSUPPORTED = 5, /* rank > 8, > 16 distinct indices, extent > 2^31-1, dtype not built */
  TC_ERR_NO_CONFIG = 6,   /* planner found no legal configuration (a bug)                    */
  TC_ERR_CUDA = 7,        /* CUDA error at plan or launch (or no device); see tc_last_error  */
  TC_ERR_ALLOC = 8        /* allocation of plan metadata failed                              */
} tc_status_t;

typedef struct tc_plan_s *tc_plan_t; /* opaque; immutable once created */

/* Cost model used to rank configurations (Section IV-B). */
typedef enum {
  TC_COST_B200 = 0,  /* re-derived model: sectors, waves, padding, FP64 pipe, HBM */
  TC_COST_PAPER = 1  /* Alg. 3 verbatim: 128-B transactions, V100 value sets  */
} tc_cost_mode_t;

/* Options for tc_plan_ex.  Zero-initialise, then set what you need. */
typedef struct tc_plan_opts {
  int cost_mode;     /* tc_cost_mode_t                                                       */
  int host_only;     /* 1: plan without touching the GPU (no device tables; tc_execute fails) */
  int variant;       /* -1 or 0: planner's choice; k>0: force kernel variant k-1 (tests)     */
  /* forced per-index tiles (tests of Fig. 2/3-style configs): "a:16;b:4;e:1;f:16" or NULL.
     Indices not listed keep the planner's choice only if force_tiles is NULL.               */
  const char *force_tiles;
  int no_fusion;     /* 1: do not merge adjacent indices (row a2)                            */
  int tma_epilogue;  /* 1: stage C tiles in smem and store them with TMA (cp.async.bulk.tensor)
                        when C is a legal tensor map and beta == 0; 0 (default): direct stores */
  int morder;        /* 0: planner's choice; 1: m digits in C order (C's FVI first); 2: in the X
                        operand's memory order (its FVI first) — tests of both epilogues   */
  int no_tma_operands; /* 1: tcgen05 plans load operands with cp.async even where TMA boxes
                          fit (default 0: one thread issues TMA boxes when the plan allows) */
  int cta_pair;      /* tcgen05 BN = 128 plans with TMA operands: 0 planner's choice, 1 never,
                        2 always — CTA pairs (cluster of 2, M = 256 MMAs over 2 x 2 tiles)   */
  int out_f32;       /* TC_BF16 plans: 1 = C is FP32 (the accumulator without the BF16 rounding;
                        split-K partials); TC_ERR_INVALID_ARG for other dtypes */
  int stream;        /* streaming path for low-intensity tensor x matrix contractions (TC_BF16,
                        one internal and one <= 32 Y-side external index, Y in shared memory,
                        TMA boxes for X and C): 0 planner's choice (on when
                        eligible and no variant is forced), 1 never, 2 whenever eligible.  The
                        plan keeps its tcgen05 configuration for beta != 0 and unaligned
                        pointers.                                                            */
  int stream_rank;   /* 0 (default): the streaming path's model-best tiles; r > 0: its r-th
                        alternative (tc_plan_tuned times the first three)                    */
  int reserved[1];   /* must be zero (TC_ERR_INVALID_ARG otherwise)                         */
} tc_plan_opts;

/*
 * Plan a contraction.
 *   expr    : "abcd-aebf-dfce" (TCCG form C-A-B, one letter per index) or
 *             "C[a,b,c,d] = A[a,e,b,f] * B[d,f,c,e]" (bracket form).
 *   extents : "a:16;b:16;c:16;d:16;e:16;f:16", each index exactly once.
 *   dtype   : A, B and C share it.  TC_F64 is the paper's precision (R20).
 * On success *plan owns its host metadata and small device tables, allocated on the device
 * that is current at the call (unless opts->host_only).  *plan is NULL on failure.
 */
tc_status_t tc_plan(tc_plan_t *plan, const char *expr, const char *extents, tc_dtype_t dtype);
tc_status_t tc_plan_ex(tc_plan_t *plan, const char *expr, const char *extents, tc_dtype_t dtype,
                       const tc_plan_opts *opts /* nullable */);

/*
 * C = alpha * sum_int A*B + beta * C on `stream` (asynchronous; no allocation, no sync).
 * A, B, C are caller-owned DEVICE pointers on the plan's device, dense in the plan's layout
 * (for a restricted plan: the parent tensors' base pointers unless TC_SLAB_* flags said
 * otherwise).  Any cudaMalloc pointer works; 16-B aligned pointers enable the vectorised
 * loads.  beta == 0 => C is only written (NaN in the old C does not propagate, R26).
 * Errors: TC_ERR_INVALID_ARG (NULL, C overlapping A or B, wrong current device),
 * TC_ERR_CUDA (launch error; asynchronous faults surface at the caller's next sync).
 */
tc_status_t tc_execute(const tc_plan_t plan, const void *A, const void *B, void *C, double alpha,
                       double beta, tc_stream_t stream);

/*
 * Grouped contractions into one output (first step; the CCSD(T) triples
 * of P:L27, L330 accumulate the 9 sd_t_d1 and 9 sd_t_d2 contractions into one t3):
 *   C = alpha * sum_{i<n} (sum_int A_i*B_i under plans[i]) + beta * C
 * plans[i] may contract differently shaped A_i, B_i, but every plan must give C the same
 * layout (extents and element strides per position, origin, dtype, device): otherwise
 * TC_ERR_INVALID_ARG before anything is launched.  A[i], B[i] are DEVICE pointers as for
 * tc_execute; C is written by plans[0] with beta and accumulated (beta = 1) by the rest, all
 * on `stream` in order (capturable into a CUDA graph).  Errors: TC_ERR_INVALID_ARG (n < 1,
 * NULL arrays or entries, layout mismatch), then as tc_execute for each entry.
 */
tc_status_t tc_execute_group(const tc_plan_t *plans, const void *const *A, const void *const *B,
                             int n, void *C, double alpha, double beta, tc_stream_t stream);

/*
 * FUSED grouped contraction (R34): the same sum as
 * tc_execute_group,
 *   C = alpha * sum_{i<n} (sum_int A_i*B_i under plans[i]) + beta * C,
 * run as ONE persistent FP64 kernel that keeps each C tile on chip across all n members and
 * stores it once (the CCSD(T) triples of P:L27, L330, L344: 18 contractions into t3, which
 * the paper and tc_execute_group run as 18 kernels each reading and writing t3).
 * tc_group_plan: plans[i] (FP64, all giving C the same layout as in tc_execute_group, no
 * batch index, n <= 32) are read, not kept; the group owns its own tables (device memory on
 * the current device, or none when the plans are host_only — then tc_group_execute fails).
 * The common C tile is chosen so that every member's tile is at most 64 x 64 (rows = the C
 * indices of the operand holding C's FVI); TC_ERR_UNSUPPORTED when no such tile exists.
 * tc_group_execute: A[i], B[i] device pointers as for tc_execute on plans[i]; asynchronous on
 * `stream`, no allocation; beta == 0 => C is only written.  Errors: TC_ERR_INVALID_ARG (NULL,
 * C overlapping any A_i / B_i, wrong device), TC_ERR_CUDA (launch, host_only group).
 */
typedef struct tc_group_s *tc_group_t;
tc_status_t tc_group_plan(tc_group_t *group, const tc_plan_t *plans, int n);
tc_status_t tc_group_execute(const tc_group_t group, const void *const *A, const void *const *B, void *C,
                             double alpha, double beta, tc_stream_t stream);
/* JSON: the C tile (T per C position), tiles, BK, per-member Mt / Nt / Kt / k-steps and the
   simulated shared-memory wavefronts of its stage loads and box flush. */
tc_status_t tc_group_info(const tc_group_t group, char *json, size_t cap, size_t *needed);
void tc_group_destroy(tc_group_t group);                /* NULL-safe                       */

/*
 * End-to-end call with HOST buffers (used for bench.py's "e2e" figure): copies A, B (and C
 * when beta != 0) from host memory into the caller-provided device workspace, runs
 * tc_execute, copies C back, and synchronises `stream`.  workspace must hold
 * tc_plan_workspace_bytes(plan) bytes; host buffers should be pinned for full speed.
 */
size_t tc_plan_workspace_bytes(const tc_plan_t plan);
tc_status_t tc_execute_host(const tc_plan_t plan, const void *A_host, const void *B_host,
                            void *C_host, double alpha, double beta, void *workspace,
                            size_t workspace_bytes, tc_stream_t stream);

/*
 * Measured tuning (the paper's "auto-tuned across a selected set",
 * P:L346-348): the cost model ranks the kernel variants by the predicted time of their best
 * configuration; the best configurations of the top `topk` variants (and, for streaming
 * shapes, the streaming path's three best configurations: log entries 99, 98, 97) are each
 * launched 1 + `reps` times on `stream` with the caller's A, B, C (alpha = 1, beta = 0: C's
 * contents are OVERWRITTEN), each timed launch after a 256 MB scratch write that flushes L2
 * (the scratch is allocated for the call; without memory for it the launches run warm), and
 * the fastest (median over reps) becomes *tuned, a new plan with the same contraction, layout,
 * device and options as `plan` (which stays valid and unchanged).
 * Synchronises `stream`.  tc_plan_info(*tuned) lists the candidates' times ("tuned").
 * Errors: TC_ERR_INVALID_ARG (NULL, topk < 1, reps < 1), TC_ERR_CUDA (host_only plan, launch
 * failure), as tc_execute for the pointers.  *tuned is NULL on failure.
 */
tc_status_t tc_plan_tuned(tc_plan_t *tuned, const tc_plan_t plan, const void *A, const void *B,
                          void *C, int topk, int reps, tc_stream_t stream);
/* As tc_plan_tuned, but the candidates are timed as C = A*B + beta*C (C's contents change:
   it is read and accumulated into).  For plans that will run with beta != 0 — the
   accumulating members of tc_execute_group — whose best variant differs from beta = 0's
   (reading C at the tile end costs 3-8x, unevenly across variants; R33). */
tc_status_t tc_plan_tuned_beta(tc_plan_t *tuned, const tc_plan_t plan, const void *A, const void *B,
                               void *C, int topk, int reps, double beta, tc_stream_t stream);

/*
 * Plan cache (the paper's deployment model is "plan once, run many",
 * P:L77, L300): returns the cached plan of (expr, extents, dtype, opts, current device) —
 * the strings as given, byte for byte — or plans it with tc_plan_ex and caches it.  The
 * returned handle is a new reference: release it with tc_plan_destroy (plans are reference
 * counted; the cache holds one reference until tc_plan_cache_clear).  Thread-safe.  Errors:
 * as tc_plan_ex (nothing is cached on failure).
 */
tc_status_t tc_plan_cached(tc_plan_t *plan, const char *expr, const char *extents, tc_dtype_t dtype,
                           const tc_plan_opts *opts /* nullable */);
size_t tc_plan_cache_size(void);   /* plans currently cached                                   */
void tc_plan_cache_clear(void);    /* drop the cache's references (live handles stay valid)    */

/* Flags of tc_plan_restrict: the operand passed to tc_execute is the compact slab itself. */
#define TC_SLAB_A 1u
#define TC_SLAB_B 2u
#define TC_SLAB_C 4u

/*
 * Sub-plan over [begin, begin+len) of one index:
 *   external index -> slab of C (multi-GPU C-slab sharding; no reduction needed);
 *   internal index -> split-K partial sum (caller reduces the partial C's).
 * Without flags the tensors keep the parent's strides and base pointers; with TC_SLAB_X the
 * operand X is a dense tensor of its own with that index's extent = len.
 */
tc_status_t tc_plan_restrict(tc_plan_t *sub, const tc_plan_t parent, const char *index,
                             int64_t begin, int64_t len, unsigned flags);

/*
 * Plan over caller-given element strides (C, A, B are
 * "tensors of arbitrary dimensions" addressed through their layouts).  strideC / strideA /
 * strideB: one element stride per index of that tensor, in the order its letters appear in
 * expr (NULL = dense, first letter fastest).  Input strides may be any value >= 0 (0
 * broadcasts); C's must be >= 1 and non-overlapping (sorted by stride, each stride >= the
 * previous stride * its extent).  The caller's buffers must cover tc_plan_span elements.
 * Index fusion (row a2) only merges indices whose strides are contiguous in every tensor.
 * Errors: TC_ERR_INVALID_ARG (negative / overlapping strides, span overflow) + tc_plan_ex's.
 */
tc_status_t tc_plan_strided(tc_plan_t *plan, const char *expr, const char *extents, tc_dtype_t dtype,
                            const int64_t *strideC, const int64_t *strideA, const int64_t *strideB,
                            const tc_plan_opts *opts /* nullable */);
/*
 * Representative-size plans ("a representative problem
 * size is used for performance modeling ... generated code will execute correctly for any
 * problem size", "different code versions targeted at each representative problem
 * size ... the kernel is selected at runtime").
 * tc_plan_resize: bind `rep`'s configuration (kernel variant, digit orders, per-index tiles,
 *   each clamped to the new extent) to other extents of the same expression: the device
 *   tables are rebuilt, nothing is searched.  When the new extents change the normalised
 *   index structure (an extent becomes 1, so an index drops) the planner runs instead.
 *   `rep` must come from tc_plan / tc_plan_ex / tc_plan_cached (TC_ERR_INVALID_ARG else).
 * tc_plan_select: the cost model scores every version's configuration at `extents`; the
 *   best one is resized to them (*chosen = its index, nullable).  Versions must share the
 *   expression and dtype.
 * The result is an ordinary plan owned by the caller (tc_plan_destroy).
 */
tc_status_t tc_plan_resize(tc_plan_t *sized, const tc_plan_t rep, const char *extents);
tc_status_t tc_plan_select(tc_plan_t *sized, const tc_plan_t *versions, int n, const char *extents,
                           int *chosen);

/* dst[i] = src[i] rounded to BF16 (RNE), i < n, on `stream`: the single rounding of an
   FP32-reduced split-K result (plans with out_f32).  dst (BF16) and src (FP32)
   are device pointers that must not overlap.  TC_ERR_INVALID_ARG on NULL / n < 0 / overlap,
   TC_ERR_CUDA on a launch error. */
tc_status_t tc_round_bf16(void *dst, const void *src, int64_t n, tc_stream_t stream);

/* Elements the buffer of tensor t (0=C, 1=A, 2=B) must hold: largest offset touched + 1
   (= tc_plan_numel for dense plans; larger for strided ones and restricted views). */
int64_t tc_plan_span(const tc_plan_t plan, int t);

/* JSON description of the plan (classes, fused indices, tiles, variant, predicted cost,
   config-space statistics).  Writes at most cap bytes (NUL-terminated); *needed = full size. */
tc_status_t tc_plan_info(const tc_plan_t plan, char *json, size_t cap, size_t *needed);

double tc_plan_flops(const tc_plan_t plan);          /* 2 * prod(all extents) (R5)       */
int64_t tc_plan_numel(const tc_plan_t plan, int t);  /* elements of 0=C, 1=A, 2=B        */
void tc_plan_destroy(tc_plan_t plan);                /* NULL-safe; releases one reference */
const char *tc_status_string(tc_status_t status);
const char *tc_last_error(void);                     /* thread-local detail string       */
const char *tc_version(void);

/* Validation only (parse + classify), same rules and codes as tc_plan; no allocation. */
tc_status_t tc_check(const char *expr, const char *extents);

#ifdef __cplusplus
}
#endif
#endif /* LIBTC_H */
