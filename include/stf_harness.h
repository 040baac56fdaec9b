/*
 * stf_harness.h -- test / benchmark entry points of libstf_cholesky.so.
 *
 * Not part of a factorisation: seeded input generation on the device (the
 * counter-based generator of SURVEY.md §8(d), bit-identical to synth/spd.py),
 * direct launches of the tile kernels for kernel-level parity tests, kernel
 * timing for the roofline (bench.py), and debug timelines.  Plain C, same
 * error convention as stf_cholesky.h (0 / negative code, stf_last_error()).
 * The tile kernels compute the tile tasks of PAPER.md:393 (§VII-C):
 *   GEMM(i,j,k): A_ij -= L_ik L_jk^T;  SYRK(i,k): A_ii -= L_ik L_ik^T (lower);
 *   TRSM(i,k):   A_ik <- A_ik L_kk^-T;  POTRF(k):  A_kk <- chol(A_kk).
 */
#ifndef STF_HARNESS_H
#define STF_HARNESS_H

#include <stdint.h>

#include "stf_cholesky.h"

#ifdef __cplusplus
extern "C" {
#endif

/* Fill the seeded SPD metric matrix into a TILED_2DBC descriptor (lower tiles)
 * on the devices; NULL tile pointers are skipped (multi-process mode).
 * Synchronous.  Returns 0, -4 (bad descriptor) or -101. */
int stf_fill_spd_tiles(int64_t n, int64_t nb, const stf_matrix_desc *A_desc, int ngpus, uint64_t seed);

/* Same generator into an arbitrary column-major device block: rows r0.., cols c0..
 * of the order-n matrix into dst (ld >= rows), on the current CUDA device, stream 0.
 * Synchronous. */
int stf_fill_spd_block(double *dst, int64_t ld, int64_t n, int64_t r0, int64_t c0, int64_t rows, int64_t cols,
                       uint64_t seed);

/* Direct tile-kernel launches (device pointers on the current device, stream 0,
 * synchronous; the kernel variant follows the "trsm" / "dataflow" options):
 *   stf_kernel_gemm_nt: C[M x N] -= A[M x K] B[N x K]^T; lower != 0 (SYRK, M == N,
 *                       A == B) updates only row >= col.  lda, ldb even, A, B 16-byte aligned.
 *   stf_kernel_trsm:    B[M x n] <- B L^-T, L[n x n] lower, non-unit diagonal.
 *   stf_kernel_potrf:   A[n x n] <- chol(A) in place (lower); *info = first failing column
 *                       (1-based) or 0. */
int stf_kernel_gemm_nt(int64_t M, int64_t N, int64_t K, const double *A, int64_t lda, const double *B, int64_t ldb,
                       double *C, int64_t ldc, int lower);
int stf_kernel_trsm(int64_t M, int64_t n, const double *L, int64_t ldl, double *B, int64_t ldb);
int stf_kernel_potrf(int64_t n, double *A, int64_t lda, int64_t *info);

/* Kernel timing for the roofline: `reps` launches of one tile kernel on a
 * library-owned stream of the current device, each bracketed by CUDA events
 * recorded on that same stream; *avg_ms = mean launch duration.  Inputs are
 * generated on the device (SPD generator) and restored (untimed) before each
 * TRSM / POTRF launch.  kind: 0 GEMM C[MxN] -= A[MxK] B[NxK]^T, 1 SYRK (N = M),
 * 2 TRSM B[MxN] <- B L^-T (K ignored), 3 POTRF of an M x M tile, 4 one step of the
 * critical chain POTRF(k) -> TRSM(k+1,k) -> SYRK(k+1,k) on M x M tiles (M a
 * multiple of 64, <= 1024; N, K ignored) lowered as in a factorisation: one
 * stream, captured into a graph, TRSM overlapping the POTRF when option pdl = 1;
 * the time is taken by event nodes of that graph around the three kernels.
 * Returns 0 / -4 / -101 / -103. */
int stf_bench_kernel(int kind, int64_t M, int64_t N, int64_t K, int reps, double *avg_ms);

/* Debug timeline of the last stf_potrf on one GPU slot, recorded when the
 * "debug_trace" option was 1 at plan build (timing events recorded before and
 * after every task on its stream; no SM work).  Writes up to cap_tasks records
 * of 7 int64 (kind as in stf_dag_build, i, j, k, stream index, ns since the
 * first task's start, at start and at end; -1 if unavailable) in plan order;
 * returns the number of tasks of the call (0 if not traced). */
int64_t stf_debug_last_trace(int64_t *out, int64_t cap_tasks);

/* Debug timeline of the dataflow POTRF tile kernel (one launch on the current
 * device, A: n x n column-major device matrix, ctas <= 0: default grid).
 * trace[0 .. 6T) holds %globaltimer stamps (ns) of the critical-path CTA per
 * 64-block step kb (P start, P published, S inputs ready, S published, U inputs
 * ready, U done), T = ceil(n/64); trace[6T + 3t ..] the claim / inputs-ready /
 * done stamps of bulk ticket t (0 if unused).  Returns the number of entries
 * written (<= cap) or a negative error. */
int64_t stf_debug_potrf_trace(int64_t n, double *A, int64_t lda, int ctas, int64_t *trace, int64_t cap);

/* Debug timeline of the resident-panel TRSM kernel (B[M x n] <- B L^-T, device
 * pointers, current device; requires 64 <= n <= 1024, n % 64 == 0).  With
 * T = n/64, trace[5 kb + e] holds the %globaltimer stamps (ns) of CTA 0 for
 * column block kb: e = 0 MMA step start, 1 MMA waits for the previous block's
 * solution, 2 it is available, 3 updated block handed to the solver, 4 solver
 * starts; trace[5T + kb] the solver's end.  Returns the number of entries
 * written (<= cap) or a negative error. */
int64_t stf_debug_trsm_trace(int64_t M, int64_t n, const double *L, int64_t ldl, double *B, int64_t ldb,
                             int64_t *trace, int64_t cap);

#ifdef __cplusplus
}
#endif
#endif /* STF_HARNESS_H */
