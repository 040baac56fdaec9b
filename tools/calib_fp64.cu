// Box calibration for the FP64 roofline.
//
//  1. Fragment-layout probes for the FP64 mma.sync shapes (m8n8k4, m16n8k4,
//     m16n8k8, m16n8k16): every lane loads operands according to the layout we
//     assume and writes D back according to the layout we assume; the host
//     compares against a plain triple loop.  A mismatch means the assumed
//     layout is wrong and the GEMM kernels must not be trusted.
//  2. Peak throughput of the FP64 tensor pipe (DMMA) and of the FP64 FMA pipe
//     (DFMA), in FMA/clk/SM, from long dependency-free loops on every SM.
//
// Standalone: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o calib tools/calib_fp64.cu
// Prints one JSON object on stdout.
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); exit(1);} } while (0)

// ---------------------------------------------------------------- layout probes
// A is M x K row-major in global, B is K x N row-major, D is M x N row-major.
__global__ void probe_m8n8k4(const double* A, const double* B, double* D) {
  int l = threadIdx.x, g = l >> 2, t = l & 3;
  double a = A[g * 4 + t];
  double b = B[t * 8 + g];
  double d0 = 0, d1 = 0;
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
               : "+d"(d0), "+d"(d1) : "d"(a), "d"(b));
  D[g * 8 + 2 * t] = d0;
  D[g * 8 + 2 * t + 1] = d1;
}
__global__ void probe_m16n8k4(const double* A, const double* B, double* D) {
  int l = threadIdx.x, g = l >> 2, t = l & 3;
  double a0 = A[g * 4 + t], a1 = A[(g + 8) * 4 + t];
  double b0 = B[t * 8 + g];
  double d0 = 0, d1 = 0, d2 = 0, d3 = 0;
  asm volatile("mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};"
               : "+d"(d0), "+d"(d1), "+d"(d2), "+d"(d3) : "d"(a0), "d"(a1), "d"(b0));
  D[g * 8 + 2 * t] = d0; D[g * 8 + 2 * t + 1] = d1;
  D[(g + 8) * 8 + 2 * t] = d2; D[(g + 8) * 8 + 2 * t + 1] = d3;
}
__global__ void probe_m16n8k8(const double* A, const double* B, double* D) {
  int l = threadIdx.x, g = l >> 2, t = l & 3;
  double a0 = A[g * 8 + t], a1 = A[(g + 8) * 8 + t], a2 = A[g * 8 + t + 4], a3 = A[(g + 8) * 8 + t + 4];
  double b0 = B[t * 8 + g], b1 = B[(t + 4) * 8 + g];
  double d0 = 0, d1 = 0, d2 = 0, d3 = 0;
  asm volatile("mma.sync.aligned.m16n8k8.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
               : "+d"(d0), "+d"(d1), "+d"(d2), "+d"(d3) : "d"(a0), "d"(a1), "d"(a2), "d"(a3), "d"(b0), "d"(b1));
  D[g * 8 + 2 * t] = d0; D[g * 8 + 2 * t + 1] = d1;
  D[(g + 8) * 8 + 2 * t] = d2; D[(g + 8) * 8 + 2 * t + 1] = d3;
}
__global__ void probe_m16n8k16(const double* A, const double* B, double* D) {
  int l = threadIdx.x, g = l >> 2, t = l & 3;
  double a[8], b[4];
  for (int i = 0; i < 4; ++i) { a[2 * i] = A[g * 16 + t + 4 * i]; a[2 * i + 1] = A[(g + 8) * 16 + t + 4 * i]; }
  for (int i = 0; i < 4; ++i) b[i] = B[(t + 4 * i) * 8 + g];
  double d0 = 0, d1 = 0, d2 = 0, d3 = 0;
  asm volatile("mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7,%8,%9,%10,%11}, {%12,%13,%14,%15}, {%0,%1,%2,%3};"
               : "+d"(d0), "+d"(d1), "+d"(d2), "+d"(d3)
               : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(a[4]), "d"(a[5]), "d"(a[6]), "d"(a[7]),
                 "d"(b[0]), "d"(b[1]), "d"(b[2]), "d"(b[3]));
  D[g * 8 + 2 * t] = d0; D[g * 8 + 2 * t + 1] = d1;
  D[(g + 8) * 8 + 2 * t] = d2; D[(g + 8) * 8 + 2 * t + 1] = d3;
}

static int check_probe(const char* name, int M, int N, int K,
                       void (*kern)(const double*, const double*, double*)) {
  std::vector<double> hA(M * K), hB(K * N), hD(M * N), ref(M * N, 0.0);
  for (int i = 0; i < M * K; ++i) hA[i] = (double)((i * 7) % 13 - 6);
  for (int i = 0; i < K * N; ++i) hB[i] = (double)((i * 5) % 11 - 5);
  for (int m = 0; m < M; ++m)
    for (int n = 0; n < N; ++n)
      for (int k = 0; k < K; ++k) ref[m * N + n] += hA[m * K + k] * hB[k * N + n];
  double *dA, *dB, *dD;
  CK(cudaMalloc(&dA, M * K * 8)); CK(cudaMalloc(&dB, K * N * 8)); CK(cudaMalloc(&dD, M * N * 8));
  CK(cudaMemcpy(dA, hA.data(), M * K * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dB, hB.data(), K * N * 8, cudaMemcpyHostToDevice));
  CK(cudaMemset(dD, 0xff, M * N * 8));
  kern<<<1, 32>>>(dA, dB, dD);
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(hD.data(), dD, M * N * 8, cudaMemcpyDeviceToHost));
  int bad = 0;
  for (int i = 0; i < M * N; ++i) bad += (hD[i] != ref[i]);
  cudaFree(dA); cudaFree(dB); cudaFree(dD);
  printf("  \"probe_%s\": %s,\n", name, bad ? "false" : "true");
  return bad;
}

// ---------------------------------------------------------------- peak loops
template <int NACC>
__global__ void __launch_bounds__(256) peak_dmma(double* out, int iters) {
  double a = 1.0 + threadIdx.x * 1e-9, b = 1.0 - threadIdx.x * 1e-9;
  double c[NACC][2];
#pragma unroll
  for (int i = 0; i < NACC; ++i) { c[i][0] = 0; c[i][1] = 0; }
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < NACC; ++i)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                   : "+d"(c[i][0]), "+d"(c[i][1]) : "d"(a), "d"(b));
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < NACC; ++i) s += c[i][0] + c[i][1];
  if (s == 12345.0) out[threadIdx.x] = s;
}
template <int NACC>
__global__ void __launch_bounds__(256) peak_dmma16(double* out, int iters) {
  double a = 1.0 + threadIdx.x * 1e-9, b = 1.0 - threadIdx.x * 1e-9;
  double c[NACC][4];
#pragma unroll
  for (int i = 0; i < NACC; ++i) { c[i][0] = c[i][1] = c[i][2] = c[i][3] = 0; }
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < NACC; ++i)
      asm volatile("mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%4,%4,%4,%4,%4,%4,%4}, {%5,%5,%5,%5}, {%0,%1,%2,%3};"
                   : "+d"(c[i][0]), "+d"(c[i][1]), "+d"(c[i][2]), "+d"(c[i][3]) : "d"(a), "d"(b));
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < NACC; ++i) s += c[i][0] + c[i][1] + c[i][2] + c[i][3];
  if (s == 12345.0) out[threadIdx.x] = s;
}
template <int NACC>
__global__ void __launch_bounds__(256) peak_dfma(double* out, int iters) {
  double a = 1.0 + threadIdx.x * 1e-9, b = 1.0 - threadIdx.x * 1e-9;
  double c[NACC];
#pragma unroll
  for (int i = 0; i < NACC; ++i) c[i] = i;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < NACC; ++i) c[i] = fma(a, c[i], b);
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < NACC; ++i) s += c[i];
  if (s == 12345.0) out[threadIdx.x] = s;
}

template <typename F>
static float time_kernel(F launch, int reps) {
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  launch();
  CK(cudaDeviceSynchronize());
  CK(cudaEventRecord(e0));
  for (int r = 0; r < reps; ++r) launch();
  CK(cudaEventRecord(e1));
  CK(cudaEventSynchronize(e1));
  float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
  return ms / reps;
}

int main() {
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0));
  int clk_khz = 0; CK(cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0));
  printf("{\n  \"gpu\": \"%s\", \"sm_count\": %d, \"cc\": \"%d.%d\", \"clock_khz_attr\": %d,\n",
         p.name, p.multiProcessorCount, p.major, p.minor, clk_khz);
  printf("  \"smem_per_block_optin\": %zu, \"smem_per_sm\": %zu, \"l2_bytes\": %d, \"hbm_bytes\": %zu,\n",
         p.sharedMemPerBlockOptin, p.sharedMemPerMultiprocessor, p.l2CacheSize, p.totalGlobalMem);
  int bad = 0;
  bad += check_probe("m8n8k4", 8, 8, 4, probe_m8n8k4);
  bad += check_probe("m16n8k4", 16, 8, 4, probe_m16n8k4);
  bad += check_probe("m16n8k8", 16, 8, 8, probe_m16n8k8);
  bad += check_probe("m16n8k16", 16, 8, 16, probe_m16n8k16);

  double* out; CK(cudaMalloc(&out, 4096));
  const int sms = p.multiProcessorCount;
  const int iters = 20000;
  for (int warps : {4, 8}) {
    for (int bps : {1, 2, 4}) {
      int grid = sms * bps, threads = warps * 32;
      float ms = time_kernel([&] { peak_dmma<8><<<grid, threads>>>(out, iters); }, 5);
      double fma = (double)grid * warps * iters * 8 * 256.0;
      printf("  \"dmma_m8n8k4_w%d_b%d_tflops\": %.3f,\n", warps, bps, 2 * fma / (ms * 1e-3) / 1e12);
      ms = time_kernel([&] { peak_dmma16<4><<<grid, threads>>>(out, iters / 4); }, 5);
      fma = (double)grid * warps * (iters / 4) * 4 * 2048.0;
      printf("  \"dmma_m16n8k16_w%d_b%d_tflops\": %.3f,\n", warps, bps, 2 * fma / (ms * 1e-3) / 1e12);
      ms = time_kernel([&] { peak_dfma<16><<<grid, threads>>>(out, iters); }, 5);
      fma = (double)grid * threads * iters * 16.0;
      printf("  \"dfma_w%d_b%d_tflops\": %.3f,\n", warps, bps, 2 * fma / (ms * 1e-3) / 1e12);
    }
  }
  // Single-SM rate, independent of the chip clock governor's behaviour at full load.
  {
    float ms = time_kernel([&] { peak_dmma<8><<<1, 256>>>(out, iters); }, 3);
    double fma = 8.0 * iters * 8 * 256.0;
    printf("  \"dmma_one_sm_fma_per_ns\": %.3f,\n", fma / (ms * 1e6));
  }
  printf("  \"layout_ok\": %s\n}\n", bad ? "false" : "true");
  return bad ? 2 : 0;
}
