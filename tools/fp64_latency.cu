// Latency of the operations on the POTRF critical chain (sm_100a), in SM clocks:
// dependent chains of DFMA, sqrt, reciprocal (IEEE 1/x), division, and barrier
// round trips (__syncthreads with 256 threads, named 64-thread barrier).
#include <cstdio>
#include <cuda_runtime.h>

__global__ void lat(double* out, long long* clk, double x0) {
  double x = x0 + threadIdx.x * 1e-12;
  long long t0, t1;
  const int N = 256;
  // DFMA chain
  t0 = clock64();
  for (int i = 0; i < N; ++i) x = fma(x, 0.999999, 1e-9);
  t1 = clock64();
  if (threadIdx.x == 0) clk[0] = (t1 - t0) / N;
  // sqrt chain
  t0 = clock64();
  for (int i = 0; i < N; ++i) x = sqrt(x) + 0.5;
  t1 = clock64();
  if (threadIdx.x == 0) clk[1] = (t1 - t0) / N;
  // reciprocal chain
  t0 = clock64();
  for (int i = 0; i < N; ++i) x = 1.0 / x + 0.5;
  t1 = clock64();
  if (threadIdx.x == 0) clk[2] = (t1 - t0) / N;
  // division chain
  double y = 1.37;
  t0 = clock64();
  for (int i = 0; i < N; ++i) x = x / y + 0.5;
  t1 = clock64();
  if (threadIdx.x == 0) clk[3] = (t1 - t0) / N;
  // __syncthreads round trip (all 256 threads)
  t0 = clock64();
  for (int i = 0; i < N; ++i) __syncthreads();
  t1 = clock64();
  if (threadIdx.x == 0) clk[4] = (t1 - t0) / N;
  // syncthreads + smem publish/read dependency (typical column step)
  __shared__ double s[64];
  t0 = clock64();
  for (int i = 0; i < N; ++i) {
    if (threadIdx.x == (i & 63)) s[i & 63] = x;
    __syncthreads();
    x = x + s[(i + 1) & 63] * 1e-30;
  }
  t1 = clock64();
  if (threadIdx.x == 0) clk[5] = (t1 - t0) / N;
  // named barrier, 64 threads (warps 0-1)
  if (threadIdx.x < 64) {
    t0 = clock64();
    for (int i = 0; i < N; ++i) asm volatile("bar.sync 1, 64;" ::: "memory");
    t1 = clock64();
    if (threadIdx.x == 0) clk[6] = (t1 - t0) / N;
  }
  // rsqrt chain
  t0 = clock64();
  for (int i = 0; i < N; ++i) x = rsqrt(x) + 0.5;
  t1 = clock64();
  if (threadIdx.x == 0) clk[7] = (t1 - t0) / N;
  // DMUL chain
  t0 = clock64();
  for (int i = 0; i < N; ++i) x = x * 0.999999;
  t1 = clock64();
  if (threadIdx.x == 0) clk[8] = (t1 - t0) / N;
  out[threadIdx.x] = x;
}

int main() {
  double* out;
  long long* clk;
  cudaMalloc(&out, 256 * 8);
  cudaMallocManaged(&clk, 16 * 8);
  lat<<<1, 256>>>(out, clk, 1.7);
  lat<<<1, 256>>>(out, clk, 1.7);
  cudaDeviceSynchronize();
  const char* names[] = {"DFMA", "sqrt", "1/x", "x/y", "__syncthreads(256)", "sync+smem publish", "bar.sync 64", "rsqrt", "DMUL"};
  for (int i = 0; i < 9; ++i) printf("%-22s %lld clk\n", names[i], clk[i]);
  return 0;
}
