// Which warps share an SM sub-partition: DMMA-saturating warps in a set, one warp
// running a dependent DFMA chain; its clk/op reveals whether it shares the FP64 pipe.
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ void dmma(double& d0, double& d1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};" : "+d"(d0), "+d"(d1) : "d"(a), "d"(b));
}
__global__ void k(long long* clk, double* out, unsigned mma_mask, int chain_warp) {
  const int w = threadIdx.x >> 5;
  double d[8][2];
  for (int c = 0; c < 8; ++c) d[c][0] = d[c][1] = threadIdx.x + c;
  double x = threadIdx.x;
  long long t0 = clock64();
  if (w == chain_warp) {
    for (int i = 0; i < 4096; ++i) x = fma(x, 0.999999, 1e-9);
  } else if (mma_mask >> w & 1) {
    for (int i = 0; i < 1024; ++i)
#pragma unroll
      for (int c = 0; c < 8; ++c) dmma(d[c][0], d[c][1], 1.0, 0.5);
  }
  long long t1 = clock64();
  if ((threadIdx.x & 31) == 0) clk[w] = t1 - t0;
  double s = x;
  for (int c = 0; c < 8; ++c) s += d[c][0] + d[c][1];
  out[threadIdx.x] = s;
}
int main() {
  long long* clk; double* out;
  cudaMallocManaged(&clk, 64 * 8); cudaMalloc(&out, 1024 * 8);
  struct { unsigned mask; int chain; const char* name; } v[] = {
    {0x77, 3, "MMA warps 0,1,2,4,5,6; chain warp 3"},
    {0x7e, 3, "MMA warps 1,2,3?->(1,2,4,5,6) chain 3, warp 0 idle"},
    {0xee, 0, "MMA warps 1,2,3,5,6,7; chain warp 0"},
    {0x00, 3, "chain warp 3 alone"},
  };
  for (auto& c : v) {
    k<<<1, 256>>>(clk, out, c.mask, c.chain); k<<<1, 256>>>(clk, out, c.mask, c.chain);
    cudaDeviceSynchronize();
    printf("%-50s chain clk/op = %.2f\n", c.name, clk[c.chain] / 4096.0);
  }
  return 0;
}
