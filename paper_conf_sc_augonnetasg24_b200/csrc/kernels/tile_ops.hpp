// Host-side launchers of the sm_100a FP64 tile kernels.
//
// All matrices are column-major FP64 with an explicit leading dimension (in
// elements).  Every launcher enqueues on `stream` and returns a cudaError_t of
// the launch (asynchronous errors surface at the next synchronisation).
// `prio` is the CUDA stream-priority value recorded on the launch (and on the
// graph node when captured); lower numbers are higher priority.
#pragma once
#include <atomic>
#include <cstdint>
#include <cuda_runtime.h>

namespace stfk {

// K1/K2: C[M x N] -= A[M x K] * B[N x K]^T.  lower != 0 (SYRK, requires M == N
// and A == B) updates only the elements with row >= col of C; the strictly upper
// part of C is neither read nor written.  Requirements: A, B 16-byte aligned,
// lda, ldb even (TMA global strides are multiples of 16 bytes).
cudaError_t gemm_nt(cudaStream_t stream, int prio, int M, int N, int K, const double* A, int64_t lda,
                    const double* B, int64_t ldb, double* C, int64_t ldc, int lower);
// Same with small != 0: 64 x 64 CTA tiles (twice the CTAs of the default 128 x 64;
// latency-critical updates; same per-element k order, same bits).
cudaError_t gemm_nt_tiles(cudaStream_t stream, int prio, int M, int N, int K, const double* A, int64_t lda,
                          const double* B, int64_t ldb, double* C, int64_t ldc, int lower, int small);
// Merged update C -= A_0 B_0^T + ... + A_{p-1} B_{p-1}^T (npairs <= 4, each pair K
// deep, K a multiple of the k tile) in ONE sweep over k: the accumulators carry
// across the pairs, so the result is bit-identical to npairs gemm_nt calls in that
// order, with one C load/store and one pipeline ramp instead of npairs
// (consecutive tile updates GEMM(i,j,k), GEMM(i,j,k+1), ... of one task).
// kflag (optional, npairs == 1, K % 64 == 0): the k columns [64 c, 64 c + 64) of A and B
// are waited for until kflag[c] >= kcount (counters of the TRSM producing them), so
// the launch may overlap that TRSM (programmatic dependent launch).
cudaError_t gemm_nt_multi(cudaStream_t stream, int prio, int M, int N, int K, int npairs, const double* const* As,
                          int64_t lda, const double* const* Bs, int64_t ldb, double* C, int64_t ldc, int lower,
                          int small, const int* kflag = nullptr, int kcount = 0);

// K3: B[M x n] <- B * L^-T with L[n x n] lower triangular, non-unit diagonal
// (side = right, lower, transposed).  Recursive: base blocks of <= 64 columns
// are solved by substitution, the off-diagonal blocks by gemm_nt.
cudaError_t trsm_rlt(cudaStream_t stream, int prio, int M, int n, const double* L, int64_t ldl, double* B,
                     int64_t ldb);

// K4: in-place lower Cholesky of A[n x n] (lower triangle referenced, strictly
// upper untouched).  Recursive: POTRF(A11); TRSM(A21); SYRK(A22); POTRF(A22),
// base blocks of <= 64 solved by one CTA.  A non-positive or NaN pivot in local
// column j does atomicMin(info, col0 + j + 1); the factorisation then continues
// with NaN (results unspecified, LAPACK convention).
cudaError_t potrf_lower(cudaStream_t stream, int prio, int n, double* A, int64_t lda, int64_t col0,
                        unsigned long long* info);

// Replica destinations written by a kernel's epilogue together with the home
// tile (same offsets and leading dimension): fused push of a finished tile.
// mc != 0: p[0] is a multicast address (NVSwitch multicast object bound on every
// consumer device, cuMulticastCreate): one multimem.st per element reaches all
// replicas, the switch replicates (n == 1).
struct Mirrors {
  double* p[7];
  int n;
  int mc;
};

// K3/K4 as single-launch device-side dataflow kernels over 64 x 64 blocks
// (dataflow.cu).  `ws` is a device workspace of dataflow_ws_bytes(m, n) bytes,
// private to the launch (zeroed by the launcher with a memset on `stream`).
// dataflow_prepare() uploads the task table for the shape; it must be called
// once before the first launch of that shape inside a stream capture.  POTRF:
// every final block of L is also stored into each `mirrors` replica (fused push
// of L_kk, NEXT-3).
cudaError_t potrf_tile(cudaStream_t stream, int prio, int n, double* A, int64_t lda, int64_t col0,
                       unsigned long long* info, int* ws, const Mirrors* mirrors = nullptr,
                       unsigned long long* trace = nullptr, int ctas = 0, int pdl_trig = -1,
                       cudaGraphNode_t* chain_node = nullptr, int split = 1);
// (With split, POTRF is two launches on `stream` -- the critical chain with a few
// block-task CTAs, then the other block-task CTAs released by it through
// programmatic dependent launch; ctas > 0 overrides the CTA count; when capturing, *chain_node
// returns the chain's graph node: work that needs the finished tile must depend on
// it as well as on the stream's last node.)
cudaError_t trsm_tile(cudaStream_t stream, int prio, int M, int n, const double* L, int64_t ldl, double* B,
                      int64_t ldb, int* ws);
size_t dataflow_ws_bytes(int m, int n);

// K3 row-panel form (trsm_panel.cu): one launch, ceil(M/R) CTAs each owning R
// rows (R = 32: lower latency, 64: higher efficiency; 0 = STF_TRSM_ROWS, default
// 64), left-looking over 64-wide column blocks (DMMA update + substitution).
cudaError_t trsm_panel(cudaStream_t stream, int prio, int M, int n, const double* L, int64_t ldl, double* B,
                       int64_t ldb, int rows_per_cta = 0, const Mirrors* mirrors = nullptr);
cudaError_t dataflow_prepare(int m, int n, bool potrf);

// K3 resident-panel form (trsm_res.cu): one launch, ceil(M/16) CTAs each keeping
// its 16 x n row panel in shared memory; MMA warps (left-looking DMMA updates)
// and solver warps (substitution) overlap.  Requires trsm_res_supported(n, L, ldl):
// 64 <= n <= 1024, n % 64 == 0, ldl even, L 16-byte aligned.
bool trsm_res_supported(int n, const double* L, int64_t ldl);
cudaError_t trsm_res_parts(cudaStream_t stream, int prio, int M, int n, const double* L, int64_t ldl, double* B,
                           int64_t ldb, const Mirrors* mirrors, int parts);
// pflag (optional): progress array of the dataflow POTRF producing L (its ws + 2,
// block grid pNb = n / 64): blocks of L are waited for as the solve reaches them,
// so the launch may overlap that POTRF (programmatic dependent launch).
// kflag (optional): per-64-column-block counters; each CTA adds 1 to kflag[jb] once its
// rows of column block jb are stored (a consumer waits for ceil(M / 16)), and the CTAs
// trigger their programmatic dependents at column block `trig` (-1: at exit).
cudaError_t trsm_res(cudaStream_t stream, int prio, int M, int n, const double* L, int64_t ldl, double* B,
                     int64_t ldb, const Mirrors* mirrors = nullptr, unsigned long long* trace = nullptr,
                     const int* pflag = nullptr, int pNb = 0, int* kflag = nullptr, int trig = -1);
constexpr int kTrsmResRows = 16;  // rows per CTA of trsm_res

// K8: fill rows r0.., cols c0.. (global indices) of the seeded SPD metric matrix
// of order n into dst[rows x cols] (ld).  Same SplitMix64 spec as synth/spd.py.
cudaError_t fill_spd(cudaStream_t stream, double* dst, int64_t ld, int64_t n, int64_t r0, int64_t c0, int rows,
                     int cols, uint64_t seed);

// K7: dst[rows x cols] (ldd) = transpose(src[cols x rows] (lds)).
cudaError_t transpose_copy(cudaStream_t stream, double* dst, int64_t ldd, const double* src, int64_t lds, int rows,
                           int cols);

// Fill a device int64 sentinel used by potrf_lower's info.
cudaError_t info_reset(cudaStream_t stream, unsigned long long* info);

// Number of kernels enqueued by the launchers above, all host threads
// (monotonic; the runtime reports per-call deltas as gpu_launches).
std::atomic<int64_t>& launch_count();

// Device attributes / one-time function attribute setup (max dynamic smem).
cudaError_t kernels_init(int device);

}  // namespace stfk
