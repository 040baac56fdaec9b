// Shared by the resident-panel TRSM (trsm_res.cu) and the dataflow POTRF critical
// chain (dataflow.cu): the 16-row panel layout and the blocked substitution of a
// 16 x 64 block by one warp.
#pragma once
#include <cstdint>

#include "ptx.cuh"

namespace stfk {
namespace sb {
constexpr int W = 64;
// panel element (r, c), r < 16: column c is one 128-byte line of 16 rows, 16-byte
// chunks XOR-swizzled by c & 7 (the TMA 128B pattern), so DMMA fragment loads with
// the k-permutation k = 8 grp + 2 t + kh, and the A/C fragments below, are conflict-free
__device__ __forceinline__ int xo(int r, int c) { return c * 16 + ((((r >> 1) ^ (c & 7)) << 1) | (r & 1)); }
// offset of diagonal-block element (r, c), r >= c, in the packed column-major lower triangle
__device__ __forceinline__ int poff(int r, int c) { return c * W - (c * (c - 1)) / 2 + (r - c); }
// diagonal-block accessors L(r, c), r >= c
struct Packed {
  const double* p;
  __device__ __forceinline__ double operator()(int r, int c) const { return p[poff(r, c)]; }
};
template <int LD>
struct RowMajor {  // p[r * LD + c]
  const double* p;
  __device__ __forceinline__ double operator()(int r, int c) const { return p[r * LD + c]; }
};
}  // namespace sb

// Substitution of one 16 x 64 block X <- X L^-T (L = the diagonal block) by the
// solver warp, in 8 sub-blocks of 8 columns P = 0..7:
//   (a) lane r < 16 solves row r of sub-block P in registers: x_c = b_c / L_cc
//       (correctly rounded: div_by with y = RN(1 / L_cc)), b_j -= x_c L_jc (lanes
//       16..31 repeat rows 0..15 without storing);
//   (b) the later sub-blocks Q > P are updated on the DMMA pipe:
//       X[:, Q] -= X[:, P] L[Q, P]^T  (16 x 8 x 8 per Q, fragments from the panel).
// A DFMA warp instruction costs the FP64 pipe of the sub-partition ~4 clocks for 16
// useful FMAs here, a DMMA 16 clocks for 256 (tools/solve_lab.cu), so the
// sub-block updates - 7/8 of the FMAs - run 4x faster on the DMMA path.
// Every sum keeps a fixed order; results are deterministic.
using sb::xo;

struct NoHook {
  __device__ __forceinline__ void operator()(int) const {}
};

// hook(P) runs at the start of sub-block P (e.g. waiting until the diagonal
// block's columns 8P..8P+7 are final and staging their reciprocals in Y)
template <int P, class DA, class Hook = NoHook>
__device__ __forceinline__ void solve_block(double* Xs, int c0, DA D, const double* Y, int lane,
                                            double* X, int64_t ldx, int64_t xrow, bool wr, const Hook& hook = Hook()) {
  if constexpr (P < 8) {
    hook(P);
    const int r = lane & 15;
    const int cb = c0 + 8 * P;
    // (a) serial substitution of the 8 columns of sub-block P
    double b[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) b[i] = Xs[xo(r, cb + i)];
    __syncwarp();  // lanes 16..31 read rows 0..15 too: all reads before lanes 0..15 store
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int c = 8 * P + i;
      const double x = div_by(b[i], D(c, c), Y[c]);
      b[i] = x;
#pragma unroll
      for (int i2 = i + 1; i2 < 8; ++i2) b[i2] = fma(-x, D(8 * P + i2, c), b[i2]);
    }
    if (lane < 16) {
#pragma unroll
      for (int i = 0; i < 8; ++i) Xs[xo(r, cb + i)] = b[i];
    }
    if (wr) {
#pragma unroll
      for (int i = 0; i < 8; ++i) X[(int64_t)(cb + i) * ldx + xrow] = b[i];
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
          const double v = D(8 * Q + g, 8 * P + 4 * ks + t);
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
    solve_block<P + 1>(Xs, c0, D, Y, lane, X, ldx, xrow, wr, hook);
  }
}

}  // namespace stfk
