/*
 * tc_oracle.h — CPU ORACLE for direct tensor contraction.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  It shares no code with libtc (the product): it has its
 * own parser, its own validation, its own stride arithmetic.  Nothing in it is blocked,
 * fused or reordered beyond the definition it follows.
 *
 * Definition (Section II, eq. (1) and the sum below it):
 *     C[a,b,c,d] = sum_{e,f} A[a,e,b,f] * B[d,f,c,e]
 * generalised by the Einstein convention: every index that does not appear in
 * C is summed.  Every index appears in exactly two of the three tensors, or in
 * all three: a batch (Hadamard) index (reading R31), which is
 * not summed — C[..h..] = sum A[..h..] * B[..h..] for each h.  The update reading is C = alpha * sum + beta * C (reading R3; beta == 0 => the
 * old C is never read).
 * Storage: the FIRST listed index of each tensor is the fastest
 * varying index (stride 1); offset = sum_k i_k * prod_{j<k} N_j.
 * The "direct 6D nested loop" of P:L62 is exactly what tco_run implements.
 *
 * Status codes (own numbering, equal by DESIGN.md contract to libtc's):
 *   0 ok, 1 invalid arg, 2 parse, 3 index, 4 extent, 5 unsupported.
 * Dtypes: 0 = f64, 1 = f32, 2 = tf32 (stored as f32; the oracle computes it as f32),
 *         3 = bf16 (uint16 bit patterns).  Narrow inputs are upcast exactly to double;
 *         the output is rounded RNE to the dtype (reading R21).
 * Parity status: pinned (tests/test_oracle.py: TTGT brute force, GEMM special cases,
 * rank-1 closed form, constant/delta inputs, linearity, relabelling, slab consistency).
 */
#ifndef TC_ORACLE_H
#define TC_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* Parse + validate only; returns a status code (see above). */
int tco_check(const char *expr, const char *extents);

/* Number of elements of tensor t (0 = C, 1 = A, 2 = B); -1 on error. */
int64_t tco_numel(const char *expr, const char *extents, int t);

/*
 * Compute C linear indices [lo, hi) (C's first index fastest) into C_out[0 .. hi-lo).
 *   A, B    : whole input tensors (dtype `dtype`).
 *   C_in    : whole old C (dtype `dtype`), read only when beta != 0; may be NULL if beta == 0.
 *   C_out   : hi-lo elements of dtype `dtype` (rounded result).
 *   S_out   : nullable; hi-lo doubles, S[x] = |alpha| * sum_y |A*B| + |beta| * |C_in[x]|,
 *             the scale the tolerance multiplies (SURVEY 8(c) "Tolerance").
 *   exact   : 0 = plain sequential sum (compiled with -ffp-contract=off);
 *             1 = Neumaier-compensated sum (only to bound the oracle's own error).
 *   nthreads: OpenMP threads (<= 0: library default).
 */
int tco_range(const char *expr, const char *extents, int dtype,
              const void *A, const void *B, const void *C_in, void *C_out, double *S_out,
              double alpha, double beta, int64_t lo, int64_t hi, int exact, int nthreads);

/* Same, for an explicit list of C linear indices idx[0..n). C_out / S_out have n entries. */
int tco_sample(const char *expr, const char *extents, int dtype,
               const void *A, const void *B, const void *C_in, void *C_out, double *S_out,
               double alpha, double beta, const int64_t *idx, int64_t n, int exact, int nthreads);

/* Threads the OpenMP runtime would use by default. */
int tco_max_threads(void);

#ifdef __cplusplus
}
#endif
#endif
