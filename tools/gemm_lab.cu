// Instruction-mix experiment for the DMMA GEMM mainloop (not part of the library).
// Runs the exact fragment-load + DMMA inner loop of gemm_dmma.cu over a fixed,
// resident shared-memory stage (no TMA, no barriers) to separate the cost of
// the instruction mix from the cost of the pipeline.
//   mode 0: LDS fragments + neg + DMMA (the production inner loop)
//   mode 1: LDS fragments + DMMA (no negation)
//   mode 2: DMMA only on register operands (upper bound)
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int WM, int WN, int MODE>
__global__ void __launch_bounds__((128 / WM) * (128 / WN) * 32, 1) lab(double* out, int iters) {
  extern __shared__ __align__(1024) uint8_t sm[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, gq = lane >> 2, tq = lane & 3;
  for (int i = threadIdx.x; i < 64 * 1024 / 8; i += blockDim.x) reinterpret_cast<double*>(sm)[i] = 1.0 + i * 1e-9;
  __syncthreads();
  const int wm0 = (warp % (128 / WM)) * WM, wn0 = (warp / (128 / WM)) * WN;
  auto off = [](int r, int k) -> uint32_t {
    const int box = r >> 4, mi = r & 15;
    return box * (16 * 32 * 8) + k * 128 + ((((mi >> 1) ^ (k & 7)) << 4) | ((mi & 1) << 3));
  };
  uint32_t oA[2][2], oB[2][2];
  for (int p = 0; p < 2; ++p)
    for (int kh = 0; kh < 2; ++kh) {
      oA[p][kh] = off(wm0 + 8 * p + gq, 2 * tq + kh);
      oB[p][kh] = 32768 + off(wn0 + 8 * p + gq, 2 * tq + kh);
    }
  double acc[WM / 8][WN / 8][2] = {};
  double ra = 1.0 + lane * 1e-7, rb = 1.0 - lane * 1e-7;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int grp = 0; grp < 4; ++grp) {
      double a[WM / 8][2], b[WN / 8][2];
#pragma unroll
      for (int f = 0; f < WM / 8; ++f)
#pragma unroll
        for (int kh = 0; kh < 2; ++kh)
          a[f][kh] = MODE == 2 ? ra : *reinterpret_cast<const double*>(sm + oA[f & 1][kh] + (f >> 1) * 4096 + grp * 1024);
#pragma unroll
      for (int f = 0; f < WN / 8; ++f)
#pragma unroll
        for (int kh = 0; kh < 2; ++kh) {
          double v = MODE == 2 ? rb : *reinterpret_cast<const double*>(sm + oB[f & 1][kh] + (f >> 1) * 4096 + grp * 1024);
          if (MODE == 0) v = __longlong_as_double(__double_as_longlong(v) ^ (long long)0x8000000000000000ULL);
          b[f][kh] = v;
        }
#pragma unroll
      for (int kh = 0; kh < 2; ++kh)
#pragma unroll
        for (int i = 0; i < WM / 8; ++i)
#pragma unroll
          for (int j = 0; j < WN / 8; ++j)
            asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                : "+d"(acc[i][j][0]), "+d"(acc[i][j][1]) : "d"(a[i][kh]), "d"(b[j][kh]));
    }
  }
  double s = 0;
  for (int i = 0; i < WM / 8; ++i)
    for (int j = 0; j < WN / 8; ++j) s += acc[i][j][0] + acc[i][j][1];
  if (s == 1234.5) out[threadIdx.x] = s;
}

template <int WM, int WN, int MODE>
void run(const char* name) {
  const int nt = (128 / WM) * (128 / WN) * 32;
  cudaFuncSetAttribute(lab<WM, WN, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
  double* out;
  cudaMalloc(&out, 8192);
  const int iters = 2000;
  lab<WM, WN, MODE><<<148, nt, 65536>>>(out, 10);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  lab<WM, WN, MODE><<<148, nt, 65536>>>(out, iters);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  const double fma = 148.0 * 128 * 128 * 32 * (double)iters;
  printf("%-40s %.2f TF/s (%.1f%% of 37.09)\n", name, 2 * fma / (ms * 1e-3) / 1e12, 100 * 2 * fma / (ms * 1e-3) / 1e12 / 37.09);
  cudaFree(out);
}

int main() {
  run<64, 32, 0>("8 warps 64x32: LDS+neg+DMMA");
  run<64, 32, 1>("8 warps 64x32: LDS+DMMA");
  run<64, 32, 2>("8 warps 64x32: DMMA only");
  run<32, 32, 0>("16 warps 32x32: LDS+neg+DMMA");
  run<32, 32, 1>("16 warps 32x32: LDS+DMMA");
  run<32, 32, 2>("16 warps 32x32: DMMA only");
  return 0;
}
