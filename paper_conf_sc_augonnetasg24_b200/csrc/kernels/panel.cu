// K3 TRSM and K4 POTRF tile kernels, plus the recursive
// drivers that split a tile into <= 64-wide base blocks and reuse the DMMA
// GEMM/SYRK kernel (gemm_dmma.cu) for every off-diagonal block.
//
// Tile task definitions (right-looking tiled Cholesky of [17],
// PAPER.md:495):
//   POTRF(k):    A_kk <- L_kk with A_kk = L_kk L_kk^T          (in place, lower)
//   TRSM(i,k):   A_ik <- A_ik L_kk^-T                          (solve X L_kk^T = A_ik)
//
// The base cases are substitution (no inverses), so every division is by the
// computed pivot and a unit-diagonal dyadic input factors bit-exactly (pin P2).
#include <cuda_runtime.h>

#include <atomic>
#include <climits>
#include <cmath>

#include "tile_ops.hpp"

namespace stfk {

constexpr int BASE = 64;  // base block order for the recursive POTRF / TRSM

// ---------------------------------------------------------------- POTRF base
// One CTA factors an n x n (n <= 64) lower block in shared memory, right-looking
// unblocked: pivot, scale the column, rank-1 update of the trailing lower part.
// Each element is updated in the order j = 0, 1, ... (the Crout order).
__global__ void __launch_bounds__(256) potrf_base_kernel(double* __restrict__ A, int64_t lda, int n, int64_t col0,
                                                         unsigned long long* info) {
  __shared__ double S[BASE][BASE + 1];
  const int tid = threadIdx.x;
  for (int idx = tid; idx < n * n; idx += blockDim.x) {
    const int i = idx % n, j = idx / n;
    if (i >= j) S[i][j] = A[(int64_t)j * lda + i];
  }
  __syncthreads();
  for (int j = 0; j < n; ++j) {
    if (tid == 0) {
      double s = S[j][j];
      if (!(s > 0.0)) {
        atomicMin(info, (unsigned long long)(col0 + j + 1));
        s = __longlong_as_double(0x7ff8000000000000LL);  // NaN: keep going, result unspecified
      } else {
        s = sqrt(s);
      }
      S[j][j] = s;
    }
    __syncthreads();
    const double d = S[j][j];
    for (int i = j + 1 + tid; i < n; i += blockDim.x) S[i][j] = S[i][j] / d;
    __syncthreads();
    const int m = n - j - 1;
    for (int idx = tid; idx < m * m; idx += blockDim.x) {
      const int i = j + 1 + idx % m, c = j + 1 + idx / m;
      if (i >= c) S[i][c] = fma(-S[i][j], S[c][j], S[i][c]);
    }
    __syncthreads();
  }
  for (int idx = tid; idx < n * n; idx += blockDim.x) {
    const int i = idx % n, j = idx / n;
    if (i >= j) A[(int64_t)j * lda + i] = S[i][j];
  }
}

// ---------------------------------------------------------------- TRSM base
// B[M x n] <- B L^-T for n <= 64: each thread owns one row of B, held in
// registers; forward substitution x_c = (b_c - sum_{p<c} x_p L_cp) / L_cc with
// the sum accumulated right-looking in p order.  L is broadcast from smem.
__global__ void __launch_bounds__(64) trsm_base_kernel(const double* __restrict__ L, int64_t ldl, int n,
                                                       double* __restrict__ B, int64_t ldb, int M) {
  __shared__ double Ls[BASE][BASE + 1];  // Ls[c][p] = L(c, p)
  for (int idx = threadIdx.x; idx < n * n; idx += blockDim.x) {
    const int c = idx % n, p = idx / n;
    Ls[c][p] = (c >= p) ? L[(int64_t)p * ldl + c] : 0.0;
  }
  __syncthreads();
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= M) return;
  double x[BASE];
#pragma unroll
  for (int c = 0; c < BASE; ++c) x[c] = (c < n) ? B[(int64_t)c * ldb + r] : 0.0;
#pragma unroll
  for (int c = 0; c < BASE; ++c) {
    if (c < n) {
      x[c] = x[c] / Ls[c][c];
#pragma unroll
      for (int c2 = c + 1; c2 < BASE; ++c2) x[c2] = fma(-x[c], Ls[c2][c], x[c2]);
    }
  }
#pragma unroll
  for (int c = 0; c < BASE; ++c)
    if (c < n) B[(int64_t)c * ldb + r] = x[c];
}

std::atomic<int64_t>& launch_count() {
  static std::atomic<int64_t> c{0};
  return c;
}

static cudaError_t launch_prio(const void* fn, dim3 grid, dim3 block, cudaStream_t s, int prio, void** args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = prio;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  ++launch_count();
  return cudaLaunchKernelExC(&cfg, fn, args);
}

// split point: half, rounded to a multiple of BASE (so sub-blocks stay aligned)
static int split(int n) {
  int h = (n / 2 + BASE - 1) / BASE * BASE;
  if (h >= n) h = n - BASE;
  return h;
}

cudaError_t trsm_rlt(cudaStream_t stream, int prio, int M, int n, const double* L, int64_t ldl, double* B,
                     int64_t ldb) {
  if (M <= 0 || n <= 0) return cudaSuccess;
  if (n <= BASE) {
    void* args[] = {(void*)&L, (void*)&ldl, (void*)&n, (void*)&B, (void*)&ldb, (void*)&M};
    return launch_prio((const void*)trsm_base_kernel, dim3((M + 63) / 64), dim3(64), stream, prio, args);
  }
  const int n1 = split(n), n2 = n - n1;
  cudaError_t e = trsm_rlt(stream, prio, M, n1, L, ldl, B, ldb);
  if (e != cudaSuccess) return e;
  // B2 -= B1 * L21^T   (L21 = L[n1:, :n1])
  e = gemm_nt(stream, prio, M, n2, n1, B, ldb, L + n1, ldl, B + (int64_t)n1 * ldb, ldb, 0);
  if (e != cudaSuccess) return e;
  return trsm_rlt(stream, prio, M, n2, L + (int64_t)n1 * ldl + n1, ldl, B + (int64_t)n1 * ldb, ldb);
}

cudaError_t potrf_lower(cudaStream_t stream, int prio, int n, double* A, int64_t lda, int64_t col0,
                        unsigned long long* info) {
  if (n <= 0) return cudaSuccess;
  if (n <= BASE) {
    void* args[] = {(void*)&A, (void*)&lda, (void*)&n, (void*)&col0, (void*)&info};
    return launch_prio((const void*)potrf_base_kernel, dim3(1), dim3(256), stream, prio, args);
  }
  const int n1 = split(n), n2 = n - n1;
  double* A21 = A + n1;
  double* A22 = A + (int64_t)n1 * lda + n1;
  cudaError_t e = potrf_lower(stream, prio, n1, A, lda, col0, info);
  if (e == cudaSuccess) e = trsm_rlt(stream, prio, n2, n1, A, lda, A21, lda);
  if (e == cudaSuccess) e = gemm_nt(stream, prio, n2, n2, n1, A21, lda, A21, lda, A22, lda, 1);
  if (e == cudaSuccess) e = potrf_lower(stream, prio, n2, A22, lda, col0 + n1, info);
  return e;
}

// ---------------------------------------------------------------- K8 generator
__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  uint64_t z = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__global__ void fill_spd_kernel(double* __restrict__ dst, int64_t ld, int64_t n, int64_t r0, int64_t c0, int rows,
                                int cols, uint64_t s) {
  const int64_t total = (int64_t)rows * cols;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    const int r = (int)(idx % rows), c = (int)(idx / rows);
    const uint64_t i = (uint64_t)(r0 + r), j = (uint64_t)(c0 + c);
    const uint64_t hi = i > j ? i : j, lo = i > j ? j : i;
    const uint64_t h = splitmix64(((hi << 32) | lo) ^ s);
    const double u = (double)(h >> 11) * 0x1.0p-53;
    double a = 2.0 * u - 1.0;
    if (i == j) a = a + (double)n;
    dst[(int64_t)c * ld + r] = a;
  }
}

cudaError_t fill_spd(cudaStream_t stream, double* dst, int64_t ld, int64_t n, int64_t r0, int64_t c0, int rows,
                     int cols, uint64_t seed) {
  if (rows <= 0 || cols <= 0) return cudaSuccess;
  // splitmix64(seed) computed on the host with the same arithmetic
  uint64_t x = seed + 0x9E3779B97F4A7C15ull;
  uint64_t z = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  const uint64_t s = z ^ (z >> 31);
  const int64_t total = (int64_t)rows * cols;
  int blocks = (int)((total + 255) / 256);
  if (blocks > 148 * 16) blocks = 148 * 16;
  ++launch_count();
  fill_spd_kernel<<<blocks, 256, 0, stream>>>(dst, ld, n, r0, c0, rows, cols, s);
  return cudaGetLastError();
}

// ---------------------------------------------------------------- K7 transpose
__global__ void transpose_kernel(double* __restrict__ dst, int64_t ldd, const double* __restrict__ src, int64_t lds,
                                 int rows, int cols) {
  __shared__ double t[32][33];
  const int bx = blockIdx.x * 32, by = blockIdx.y * 32;  // bx over dst rows, by over dst cols
  // src is cols x rows: src(c, r) at src[r*lds + c]; dst(r, c) = src(c, r)
  for (int y = threadIdx.y; y < 32; y += blockDim.y) {
    const int r = bx + y, c = by + threadIdx.x;
    if (r < rows && c < cols) t[y][threadIdx.x] = src[(int64_t)r * lds + c];
  }
  __syncthreads();
  for (int y = threadIdx.y; y < 32; y += blockDim.y) {
    const int c = by + y, r = bx + threadIdx.x;
    if (r < rows && c < cols) dst[(int64_t)c * ldd + r] = t[threadIdx.x][y];
  }
}

cudaError_t transpose_copy(cudaStream_t stream, double* dst, int64_t ldd, const double* src, int64_t lds, int rows,
                           int cols) {
  if (rows <= 0 || cols <= 0) return cudaSuccess;
  ++launch_count();
  transpose_kernel<<<dim3((rows + 31) / 32, (cols + 31) / 32), dim3(32, 8), 0, stream>>>(dst, ldd, src, lds, rows,
                                                                                          cols);
  return cudaGetLastError();
}

__global__ void info_reset_kernel(unsigned long long* info) { *info = ULLONG_MAX; }


cudaError_t info_reset(cudaStream_t stream, unsigned long long* info) {
  ++launch_count();
  info_reset_kernel<<<1, 1, 0, stream>>>(info);
  return cudaGetLastError();
}

cudaError_t gemm_init_attrs();
cudaError_t dataflow_init_attrs();
cudaError_t trsm_panel_init_attrs();
cudaError_t trsm_res_init_attrs();

cudaError_t kernels_init(int device) {
  int cur = 0;
  cudaGetDevice(&cur);
  cudaSetDevice(device);
  cudaError_t e = gemm_init_attrs();
  if (e == cudaSuccess) e = dataflow_init_attrs();
  if (e == cudaSuccess) e = trsm_panel_init_attrs();
  if (e == cudaSuccess) e = trsm_res_init_attrs();
  cudaSetDevice(cur);
  return e;
}

}  // namespace stfk
