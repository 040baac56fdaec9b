// Latency lab for P(kb) of the POTRF critical chain (not part of the library).
// Includes dataflow.cu and times chol_block_grp on one 64x64 SPD block, alone and
// with the four S warps solving a 64x64 block concurrently (the production
// overlap), with clock64 stamps per panel in warp 0 (instrumented lab copy of
// the same arithmetic).
//   build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_sc_augonnetasg24_b200/csrc \
//            tools/p_lab.cu -o tools/p_lab -lcuda
#include "../paper_conf_sc_augonnetasg24_b200/csrc/kernels/dataflow.cu"

#include <cstdio>

namespace stfk {
std::atomic<int64_t>& launch_count() {
  static std::atomic<int64_t> c{0};
  return c;
}
}  // namespace stfk

using namespace stfk;

// mode bit 0: S warps solve concurrently; bit 1: S warps spin on DMMA (pipe hog) instead
__global__ void __launch_bounds__(256, 1) k_p(const double* A, const double* X0, double* L, double* Xo, int mode,
                                              long long* clk) {
  extern __shared__ __align__(16) double sm[];
  constexpr int W = df::W;
  double* D = sm;
  double* Xp = D + W * df::LDB;
  double* Yc = Xp + 4 * 16 * W;
  int* dpanel = reinterpret_cast<int*>(Yc + 4 * W);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int rep = 0; rep < 3; ++rep) {
    for (int idx = threadIdx.x; idx < W * W; idx += 256) {
      const int r = idx & 63, c = idx >> 6;
      D[r * df::LDB + c] = A[c * W + r];
      Xp[(r >> 4) * 16 * W + sb::xo(r & 15, c)] = X0[c * W + r];
    }
    if (threadIdx.x == 0) *dpanel = 0;
    __syncthreads();
    long long t0 = clock64();
    if (warp < 4) {
      chol_block_grp(D, 0, nullptr, dpanel);
      if (threadIdx.x == 0) clk[rep] = clock64() - t0;
    } else if (mode & 1) {
      const int sw = warp - 4;
      double* Yw = Yc + sw * W;
      auto gate = [&](int P) {
        while (ld_volatile_s(dpanel) <= P) __nanosleep(40);
        __threadfence_block();
        if (lane < 8) Yw[8 * P + lane] = 1.0 / D[(8 * P + lane) * df::LDB + 8 * P + lane];
        __syncwarp();
      };
      const int rr = 16 * sw + (lane & 15);
      solve_block<0>(Xp + sw * 16 * W, 0, sb::RowMajor<df::LDB>{D}, Yw, lane, Xo, W, rr, lane < 16, gate);
      if (lane == 0) clk[4 + sw] = clock64() - t0;
    } else if (mode & 2) {
      double d0 = lane, d1 = 1;
      while (ld_volatile_s(dpanel) < 8) {
#pragma unroll
        for (int i = 0; i < 16; ++i) dmma_8x8x4(d0, d1, 1.0, 1e-9);
      }
      if (d0 == 12345.0) Xo[0] = d1;
    }
    __syncthreads();
  }
  for (int idx = threadIdx.x; idx < W * W; idx += 256) {
    const int r = idx & 63, c = idx >> 6;
    L[c * W + r] = r >= c ? D[r * df::LDB + c] : 0.0;
  }
}

int main() {
  constexpr int W = 64;
  static double hA[W * W], hX[W * W];
  for (int i = 0; i < W; ++i)
    for (int j = 0; j < W; ++j) {
      double v = ((i * 131 + j * 71) % 97) / 97.0 - 0.5;
      if (i < j) v = ((j * 131 + i * 71) % 97) / 97.0 - 0.5;
      hA[j * W + i] = v + (i == j ? W : 0.0);
      hX[j * W + i] = ((i * 37 + j * 11) % 89) / 89.0 - 0.5;
    }
  double *A, *X0, *L, *Xo;
  long long* clk;
  cudaMalloc(&A, sizeof hA);
  cudaMalloc(&X0, sizeof hX);
  cudaMalloc(&L, 5 * sizeof hA);
  cudaMalloc(&Xo, 5 * sizeof hX);
  cudaMallocManaged(&clk, 64 * 8);
  cudaMemcpy(A, hA, sizeof hA, cudaMemcpyHostToDevice);
  cudaMemcpy(X0, hX, sizeof hX, cudaMemcpyHostToDevice);
  const int smem = (W * df::LDB + 4 * 16 * W + 4 * W) * 8 + 16;
  cudaFuncSetAttribute(k_p, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const char* names[] = {"P alone", "P + S warps (production)", "P + DMMA hog on warps 4-7"};
  const int modes[] = {0, 1, 2};
  for (int v = 0; v < 3; ++v) {
    for (int i = 0; i < 16; ++i) clk[i] = 0;
    k_p<<<1, 256, smem>>>(A, X0, L + v * W * W, Xo + v * W * W, modes[v], clk);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
      printf("CUDA error %s\n", cudaGetErrorString(e));
      return 1;
    }
    printf("%-28s P %6lld clk (%.2f us at 1.965 GHz)  S warps %lld %lld %lld %lld\n", names[v], clk[2],
           clk[2] / 1965.0, clk[4], clk[5], clk[6], clk[7]);
  }
  static double hL[3][W * W];
  cudaMemcpy(hL, L, sizeof hL, cudaMemcpyDeviceToHost);
  int diff = 0;
  for (int i = 0; i < W * W; ++i) diff += hL[0][i] != hL[1][i];
  printf("bits P alone vs with S: %d mismatches\n", diff);
  return 0;
}
