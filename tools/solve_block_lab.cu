// Isolated timing of the resident TRSM solver's solve_block (one warp, one 16 x 64 block).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
struct Mirrors { double* p[7]; int n; };
__device__ __forceinline__ void dmma_8x8x4(double& d0, double& d1, double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};" : "+d"(d0), "+d"(d1) : "d"(a), "d"(b));
}
__device__ __forceinline__ double div_by(double a, double d, double y) {
  const double q0 = a * y; const double r = fma(-q0, d, a); return fma(r, y, q0);
}
namespace tr {
constexpr int R = 16;        // rows per CTA (one 128-byte line per column of the panel)
constexpr int W = 64;        // column block
constexpr int NMAX = 1024;   // resident panel limit (NMAX * 128 B = 128 KB)
constexpr int BK = 32;       // k of L per pipeline stage
constexpr int NST = 4;       // L ring slots
constexpr int BOXD = 16 * BK;          // doubles per TMA box [BK k-rows][16 c] (4 KB)
constexpr int STAGE = (W / 16) * BOXD; // doubles per stage (16 KB)
constexpr int DP = 2080;     // packed lower diagonal block: 64 * 65 / 2
constexpr int NT = 256;      // 8 warps; warp w runs on SM sub-partition w % 4
constexpr int NMMA = 6;      // MMA warps 0,1,2,4,5,6 (sub-partitions 0-2)
constexpr int MMA_THREADS = NMMA * 32, SOLVE_THREADS = 32;  // solver warp 3, producer warp 7 (sub-partition 3)
constexpr int BAR_MMA = 1, BAR_READY = 2, BAR_SOLVED = 3;
__host__ __device__ constexpr size_t smem_bytes(int n) {
  return 1024 + ((size_t)16 * n + (size_t)NST * STAGE + 2 * DP + 2 * W) * sizeof(double) + 2 * NST * 8;
}
// offset of diagonal-block element (r, c), r >= c, in the packed column-major lower triangle
__device__ __forceinline__ int poff(int r, int c) { return c * W - (c * (c - 1)) / 2 + (r - c); }
// panel element (r, c): column c is one 128-byte line of 16 rows, 16-byte chunks
// XOR-swizzled by c & 7 (the TMA 128B pattern), so DMMA fragment loads with the
// k-permutation k = 8 grp + 2 t + kh are conflict-free
__device__ __forceinline__ int xo(int r, int c) { return c * 16 + ((((r >> 1) ^ (c & 7)) << 1) | (r & 1)); }
// L stage element (k, c) written by TMA boxes of [BK][16 c] with the 128B swizzle
__device__ __forceinline__ int lo(int k, int c) {
  return (c >> 4) * BOXD + k * 16 + (((((c & 15) >> 1) ^ (k & 7)) << 1) | (c & 1));
}
// first stage of step jb (steps consume 2 jb stages each)
__host__ __device__ constexpr int step_q0(int jb) { return jb * (jb - 1); }
}  // namespace tr

template <int P>
__device__ __forceinline__ void solve_block(double* Xs, int c0, const double* D, const double* Y, int lane,
                                            double* X, int64_t ldx, int64_t xrow, bool wr, const Mirrors& mir) {
  using namespace tr;
  if constexpr (P < 8) {
    const int r = lane & 15;
    const int cb = c0 + 8 * P;
    // (a) serial substitution of the 8 columns of sub-block P
    double b[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) b[i] = Xs[xo(r, cb + i)];
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int c = 8 * P + i;
      const double x = div_by(b[i], D[poff(c, c)], Y[c]);
      b[i] = x;
#pragma unroll
      for (int i2 = i + 1; i2 < 8; ++i2) b[i2] = fma(-x, D[poff(8 * P + i2, c)], b[i2]);
    }
    if (lane < 16) {
#pragma unroll
      for (int i = 0; i < 8; ++i) Xs[xo(r, cb + i)] = b[i];
    }
    if (wr) {
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int64_t off = (int64_t)(cb + i) * ldx + xrow;
        X[off] = b[i];
#pragma unroll
        for (int m = 0; m < 7; ++m)
          if (m < mir.n) mir.p[m][off] = b[i];
      }
    }
    __syncwarp();
    // (b) X[:, Q] -= X[:, P] L[Q, P]^T for Q > P, all DMMAs issued before the stores
    if constexpr (P < 7) {
      const int g = lane >> 2, t = lane & 3;
      double a[2][2];
#pragma unroll
      for (int mi = 0; mi < 2; ++mi)
#pragma unroll
        for (int ks = 0; ks < 2; ++ks) a[mi][ks] = Xs[xo(8 * mi + g, cb + 4 * ks + t)];
      double acc[7 - P][2][2];
#pragma unroll
      for (int q = 0; q < 7 - P; ++q) {
        const int Q = P + 1 + q;
        double bq[2];
#pragma unroll
        for (int ks = 0; ks < 2; ++ks) {  // B[k][n] = L(8Q + n, 8P + k), negated: acc = C - A B^T
          const double v = D[poff(8 * Q + g, 8 * P + 4 * ks + t)];
          bq[ks] = __longlong_as_double(__double_as_longlong(v) ^ (long long)0x8000000000000000ULL);
        }
#pragma unroll
        for (int mi = 0; mi < 2; ++mi) {
          acc[q][mi][0] = Xs[xo(8 * mi + g, c0 + 8 * Q + 2 * t)];
          acc[q][mi][1] = Xs[xo(8 * mi + g, c0 + 8 * Q + 2 * t + 1)];
#pragma unroll
          for (int ks = 0; ks < 2; ++ks) dmma_8x8x4(acc[q][mi][0], acc[q][mi][1], a[mi][ks], bq[ks]);
        }
      }
#pragma unroll
      for (int q = 0; q < 7 - P; ++q)
#pragma unroll
        for (int mi = 0; mi < 2; ++mi) {
          Xs[xo(8 * mi + g, c0 + 8 * (P + 1 + q) + 2 * t)] = acc[q][mi][0];
          Xs[xo(8 * mi + g, c0 + 8 * (P + 1 + q) + 2 * t + 1)] = acc[q][mi][1];
        }
      __syncwarp();
    }
    solve_block<P + 1>(Xs, c0, D, Y, lane, X, ldx, xrow, wr, mir);
  }
}


__global__ void lab(double* X, long long* clk, int warps) {
  extern __shared__ double sm[];
  double* Xs = sm; double* D = Xs + 16 * 64; double* Y = D + 2080;
  for (int i = threadIdx.x; i < 16 * 64; i += blockDim.x) Xs[i] = 1.0 + (i % 7);
  for (int c = 0; c < 64; ++c) for (int r = c + threadIdx.x; r < 64; r += blockDim.x) D[tr::poff(r, c)] = (r == c) ? 1.0 + c * 1e-3 : 1e-3 * ((r + c) % 5);
  __syncthreads();
  for (int c = threadIdx.x; c < 64; c += blockDim.x) Y[c] = 1.0 / D[tr::poff(c, c)];
  __syncthreads();
  Mirrors mir{}; 
  const int lane = threadIdx.x & 31;
  if (threadIdx.x < 32) {
    long long t0 = clock64();
    for (int rep = 0; rep < 4; ++rep) solve_block<0>(Xs, 0, D, Y, lane, X, 16, lane & 15, lane < 16, mir);
    __syncwarp();
    long long t1 = clock64();
    if (lane == 0) clk[0] = (t1 - t0) / 4;
  }
}
int main() {
  double* X; long long* clk;
  cudaMalloc(&X, 16 * 64 * 8); cudaMallocManaged(&clk, 8 * 8);
  const int smem = (16 * 64 + 2080 + 64) * 8;
  lab<<<1, 32, smem>>>(X, clk, 1); lab<<<1, 32, smem>>>(X, clk, 1);
  cudaDeviceSynchronize();
  printf("solve_block (16 x 64, one warp): %lld clk per block\n", clk[0]);
  return 0;
}
