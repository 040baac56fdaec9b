// Latency of the 64-column substitution chain of the resident TRSM solver warp
// (one warp, 16 rows, b in registers), in SM clocks, with variants.
#include <cstdio>
#include <cuda_runtime.h>

constexpr int W = 64;
__device__ __forceinline__ int poff(int r, int c) { return c * W - (c * (c - 1)) / 2 + (r - c); }
__device__ __forceinline__ double div_by(double a, double d, double y) {
  const double q0 = a * y;
  const double r = fma(-q0, d, a);
  return fma(r, y, q0);
}
template <int C>
__device__ __forceinline__ void chain(double (&b)[W], const double* D, const double* Y) {
  if constexpr (C < W) {
    const double x = div_by(b[C], D[poff(C, C)], Y[C]);
    b[C] = x;
#pragma unroll
    for (int j = C + 1; j < W; ++j) b[j] = fma(-x, D[poff(j, C)], b[j]);
    chain<C + 1>(b, D, Y);
  }
}
// variant 2: D column held in registers for the next column (explicit one-column lookahead)
template <int C>
__device__ __forceinline__ void chain_rm(double (&b)[W], const double* D, const double* Y) {
  if constexpr (C < W) {
    const double x = div_by(b[C], D[poff(C, C)], Y[C]);
    b[C] = x;
    if constexpr (C + 1 < W) b[C + 1] = fma(-x, D[poff(C + 1, C)], b[C + 1]);  // critical first
    asm volatile("" ::: "memory");
#pragma unroll
    for (int j = C + 2; j < W; ++j) b[j] = fma(-x, D[poff(j, C)], b[j]);
    chain_rm<C + 1>(b, D, Y);
  }
}

__global__ void lab(double* out, long long* clk, int variant) {
  __shared__ double D[2080 + 8], Y[W];
  for (int i = threadIdx.x; i < 2080; i += blockDim.x) D[i] = 0.001 * (i % 17);
  for (int c = threadIdx.x; c < W; c += blockDim.x) { D[poff(c, c)] = 1.0 + c * 1e-3; Y[c] = 1.0 / D[poff(c, c)]; }
  __syncthreads();
  const int lane = threadIdx.x & 31;
  double b[W];
#pragma unroll
  for (int j = 0; j < W; ++j) b[j] = lane + j * 0.5;
  long long t0 = clock64();
  if (variant == 0) chain<0>(b, D, Y);
  else if (variant == 1) { if (lane < 16) chain<0>(b, D, Y); }
  else chain_rm<0>(b, D, Y);
  __syncwarp();
  long long t1 = clock64();
  double s = 0;
#pragma unroll
  for (int j = 0; j < W; ++j) s += b[j];
  out[threadIdx.x] = s;
  if (threadIdx.x == 0) clk[variant] = t1 - t0;
}

int main() {
  double* out; long long* clk;
  cudaMalloc(&out, 1024 * 8); cudaMallocManaged(&clk, 16 * 8);
  for (int v = 0; v < 3; ++v) { lab<<<1, 32>>>(out, clk, v); lab<<<1, 32>>>(out, clk, v); }
  cudaDeviceSynchronize();
  const char* names[] = {"32 lanes (rows dup)", "16 lanes (upper half idle)", "critical update first + compiler fence"};
  for (int v = 0; v < 3; ++v) printf("%-42s %lld clk  (%.1f per column)\n", names[v], clk[v], clk[v] / 64.0);
  return 0;
}
