// DMMA.8x8x4 latency and issue throughput on sm_100a, in SM clocks:
// one warp with C independent accumulator chains (C = 1: dependent latency),
// and W warps per SMSP each with C chains (pipe saturation), plus DMMA mixed
// with a dependent DFMA chain in another warp of the same SMSP (pipe sharing).
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ void dmma(double& d0, double& d1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
               : "+d"(d0), "+d"(d1) : "d"(a), "d"(b));
}

template <int C>
__global__ void chains(long long* clk, double* out, int iters, int dfma_warp) {
  double d[C][2];
  for (int c = 0; c < C; ++c) d[c][0] = d[c][1] = threadIdx.x * 1e-3 + c;
  const double a = 1.0 + threadIdx.x * 1e-9, b = 0.999999;
  __syncthreads();
  long long t0 = clock64();
  if (dfma_warp && (threadIdx.x >> 5) == (blockDim.x >> 5) - 1) {
    // last warp: dependent DFMA chain (the substitution pattern)
    double x = d[0][0];
    for (int i = 0; i < iters * 8; ++i) x = fma(x, b, 1e-9);
    d[0][0] = x;
  } else {
    for (int i = 0; i < iters; ++i)
#pragma unroll
      for (int c = 0; c < C; ++c) dmma(d[c][0], d[c][1], a, b);
  }
  long long t1 = clock64();
  if ((threadIdx.x & 31) == 0) clk[threadIdx.x >> 5] = t1 - t0;
  double s = 0;
  for (int c = 0; c < C; ++c) s += d[c][0] + d[c][1];
  out[threadIdx.x] = s;
}

template <int C>
void run(int warps, int dfma, long long* clk, double* out) {
  const int iters = 1024;
  chains<C><<<1, 32 * warps>>>(clk, out, iters, dfma);
  chains<C><<<1, 32 * warps>>>(clk, out, iters, dfma);
  cudaDeviceSynchronize();
  long long mx = 0;
  for (int w = 0; w < warps - (dfma ? 1 : 0); ++w) mx = clk[w] > mx ? clk[w] : mx;
  const double per = (double)mx / iters / C;  // clocks per DMMA per warp
  const int mma_warps = warps - (dfma ? 1 : 0);
  // SM-level DMMA rate: mma_warps * C * iters DMMAs in mx clocks -> FMA/clk/SM (256 FMA per DMMA)
  printf("chains=%2d warps=%2d%s  clk/DMMA/warp=%7.2f  SM FMA/clk=%6.2f", C, warps, dfma ? " (+1 DFMA-chain warp)" : "",
         per, 256.0 * mma_warps * C * iters / mx);
  if (dfma) printf("  DFMA chain clk/op=%.2f", (double)clk[warps - 1] / (iters * 8));
  printf("\n");
}

int main() {
  long long* clk;
  double* out;
  cudaMallocManaged(&clk, 64 * 8);
  cudaMalloc(&out, 1024 * 8);
  run<1>(1, 0, clk, out);
  run<2>(1, 0, clk, out);
  run<4>(1, 0, clk, out);
  run<8>(1, 0, clk, out);
  run<16>(1, 0, clk, out);
  run<4>(4, 0, clk, out);
  run<4>(8, 0, clk, out);
  run<8>(8, 0, clk, out);
  run<16>(8, 0, clk, out);
  run<16>(16, 0, clk, out);
  run<4>(9, 1, clk, out);
  run<16>(9, 1, clk, out);
  run<16>(17, 1, clk, out);
  return 0;
}
