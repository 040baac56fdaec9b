// Latency lab for the 64x64 block Cholesky on the POTRF critical chain (not part
// of the library).  Same arithmetic in every variant (sqrt, IEEE reciprocal,
// Markstein division, fma(-L_rk, L_ck, a) updates in k order), so results must
// be bit-identical; only the work distribution and synchronisation differ.
//   V0: production chol_core (4 column quarters processed one after another)
//   V1: interleaved columns: thread (r, q) holds columns q, q+4, ...; all 256
//       threads take part in every column, two __syncthreads per column
//   V2: row owner: 64 threads hold one row each (64 registers), two 64-thread
//       named barriers per column
//   V3: V1 with one barrier per column: every row thread divides its own
//       element AND the elements of the rows it needs (redundant divisions)
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

#include "../paper_conf_sc_augonnetasg24_b200/csrc/kernels/ptx.cuh"

using stfk::div_by;
constexpr int W = 64, LDB = 65, REPS = 50;

__device__ __forceinline__ void named_bar(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }

// ---------------------------------------------------------------- V0 (copy of dataflow.cu chol_core)
__device__ __forceinline__ void chol_v0(double (&a)[16], double* S, double* Y, int nc) {
  const int r = threadIdx.x & (W - 1), q = threadIdx.x >> 6;
  for (int qq = 0; qq < 4 && 16 * qq < nc; ++qq) {
    if (q == qq) {
#pragma unroll
      for (int c = 0; c < 16; ++c) {
        const int col = 16 * qq + c;
        if (col < nc) {
          if (r == col) {
            double s = a[c];
            s = sqrt(s);
            a[c] = s;
            S[col * LDB + col] = s;
            Y[col] = 1.0 / s;
          }
          named_bar(1 + qq, 64);
          if (r > col && r < nc) {
            a[c] = div_by(a[c], S[col * LDB + col], Y[col]);
            S[r * LDB + col] = a[c];
          }
          named_bar(1 + qq, 64);
          if (r > col && r < nc) {
#pragma unroll
            for (int c2 = c + 1; c2 < 16; ++c2)
              if (16 * qq + c2 <= r) a[c2] = fma(-a[c], S[(16 * qq + c2) * LDB + col], a[c2]);
          }
        }
      }
    }
    __syncthreads();
    if (q > qq && r < nc) {
#pragma unroll
      for (int cc = 0; cc < 16; ++cc) {
        if (16 * q + cc <= r) {
#pragma unroll
          for (int c = 0; c < 16; ++c)
            a[cc] = fma(-S[r * LDB + 16 * qq + c], S[(16 * q + cc) * LDB + 16 * qq + c], a[cc]);
        }
      }
    }
  }
}

__global__ void __launch_bounds__(256, 1) k_v0(const double* A, double* L, long long* clk) {
  __shared__ double S[W * LDB], Y[W];
  const int r = threadIdx.x & 63, q = threadIdx.x >> 6;
  double a[16];
  long long tot = 0;
  for (int rep = 0; rep < REPS; ++rep) {
    for (int c = 0; c < 16; ++c) a[c] = (r >= 16 * q + c) ? A[(16 * q + c) * W + r] : 0.0;
    __syncthreads();
    long long t0 = clock64();
    chol_v0(a, S, Y, W);
    __syncthreads();
    tot += clock64() - t0;
  }
  for (int c = 0; c < 16; ++c)
    if (r >= 16 * q + c) L[(16 * q + c) * W + r] = a[c];
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

// ---------------------------------------------------------------- V1 interleaved columns
__global__ void __launch_bounds__(256, 1) k_v1(const double* A, double* L, long long* clk) {
  __shared__ double Lcol[W];
  __shared__ double sy[2];
  const int r = threadIdx.x & 63, q = threadIdx.x >> 6;
  double a[16];  // column 4m + q
  long long tot = 0;
  for (int rep = 0; rep < REPS; ++rep) {
#pragma unroll
    for (int m = 0; m < 16; ++m) a[m] = (r >= 4 * m + q) ? A[(4 * m + q) * W + r] : 0.0;
    __syncthreads();
    long long t0 = clock64();
#pragma unroll
    for (int j = 0; j < W; ++j) {
      const int mj = j >> 2, qj = j & 3;
      if (q == qj && r == j) {
        const double s = sqrt(a[mj]);
        a[mj] = s;
        sy[0] = s;
        sy[1] = 1.0 / s;
      }
      __syncthreads();
      if (q == qj && r > j) {
        a[mj] = div_by(a[mj], sy[0], sy[1]);
        Lcol[r] = a[mj];
      }
      __syncthreads();
      if (r > j) {
        const double lr = Lcol[r];
#pragma unroll
        for (int m = 0; m < 16; ++m) {
          const int c = 4 * m + q;
          if (4 * m + 3 > j && c > j && c <= r) a[m] = fma(-lr, Lcol[c], a[m]);
        }
      }
    }
    __syncthreads();
    tot += clock64() - t0;
  }
#pragma unroll
  for (int m = 0; m < 16; ++m)
    if (r >= 4 * m + q) L[(4 * m + q) * W + r] = a[m];
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

// ---------------------------------------------------------------- V2 row owner (64 threads)
__global__ void __launch_bounds__(256, 1) k_v2(const double* A, double* L, long long* clk) {
  __shared__ double Lcol[W];
  __shared__ double sy[2];
  const int r = threadIdx.x;
  double a[W];
  long long tot = 0;
  for (int rep = 0; rep < REPS; ++rep) {
    if (r < W) {
#pragma unroll
      for (int c = 0; c < W; ++c) a[c] = (r >= c) ? A[c * W + r] : 0.0;
    }
    __syncthreads();
    long long t0 = clock64();
    if (r < W) {
#pragma unroll
      for (int j = 0; j < W; ++j) {
        if (r == j) {
          const double s = sqrt(a[j]);
          a[j] = s;
          sy[0] = s;
          sy[1] = 1.0 / s;
        }
        named_bar(1, 64);
        if (r > j) {
          a[j] = div_by(a[j], sy[0], sy[1]);
          Lcol[r] = a[j];
        }
        named_bar(1, 64);
        if (r > j) {
#pragma unroll
          for (int c = j + 1; c < W; ++c)
            if (c <= r) a[c] = fma(-a[j], Lcol[c], a[c]);
        }
      }
    }
    __syncthreads();
    tot += clock64() - t0;
  }
  if (r < W) {
#pragma unroll
    for (int c = 0; c < W; ++c)
      if (r >= c) L[c * W + r] = a[c];
  }
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

// ---------------------------------------------------------------- V3: one barrier per column
// raw column j (after the update from j-1) is published by its owners together
// with the pivot's s and 1/s; every thread divides the raw values it needs.
__global__ void __launch_bounds__(256, 1) k_v3(const double* A, double* L, long long* clk) {
  __shared__ double Raw[2][W];
  __shared__ double sy[2][2];
  const int r = threadIdx.x & 63, q = threadIdx.x >> 6;
  double a[16];
  long long tot = 0;
  for (int rep = 0; rep < REPS; ++rep) {
#pragma unroll
    for (int m = 0; m < 16; ++m) a[m] = (r >= 4 * m + q) ? A[(4 * m + q) * W + r] : 0.0;
    // column 0 raw
    if (q == 0) Raw[0][r] = a[0];
    if (q == 0 && r == 0) {
      const double s = sqrt(a[0]);
      sy[0][0] = s;
      sy[0][1] = 1.0 / s;
    }
    __syncthreads();
    long long t0 = clock64();
#pragma unroll
    for (int j = 0; j < W; ++j) {
      const int b = j & 1;
      const double s = sy[b][0], y = sy[b][1];
      if (r >= j) {
        // L_rj
        const double lr = (r == j) ? s : div_by(Raw[b][r], s, y);
        if (q == (j & 3)) a[j >> 2] = lr;
        if (r > j) {
          // the next column first: element j+1 (owned by q == (j+1)&3), then publish it
          const int j1 = j + 1;
          if (j1 < W && q == (j1 & 3) && j1 <= r) {
            const double l1 = div_by(Raw[b][j1], s, y);
            a[j1 >> 2] = fma(-lr, l1, a[j1 >> 2]);
            Raw[b ^ 1][r] = a[j1 >> 2];
            if (r == j1) {
              const double s1 = sqrt(a[j1 >> 2]);
              sy[b ^ 1][0] = s1;
              sy[b ^ 1][1] = 1.0 / s1;
            }
          }
#pragma unroll
          for (int m = 0; m < 16; ++m) {
            const int c = 4 * m + q;
            if (4 * m + 3 > j + 1 && c > j + 1 && c <= r) a[m] = fma(-lr, div_by(Raw[b][c], s, y), a[m]);
          }
        }
      }
      __syncthreads();
    }
    tot += clock64() - t0;
  }
#pragma unroll
  for (int m = 0; m < 16; ++m)
    if (r >= 4 * m + q) L[(4 * m + q) * W + r] = a[m];
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

// ---------------------------------------------------------------- V4: one barrier per column, no pivot hand-off
// Every owner thread of column j+1 (q == (j+1)&3) recomputes the pivot itself:
// d = a_{j+1,j+1} - L_{j+1,j}^2 from the published diagonal Dpub[j+1] (after
// updates 0..j-1) and L_{j+1,j}; then s = sqrt(d), y = 1/s, and divides its own
// element at once.  The only barrier per column publishes the column L_{.,j+1}.
__global__ void __launch_bounds__(256, 1) k_v4(const double* A, double* L, long long* clk) {
  __shared__ double Lc[2][W];
  __shared__ double Dp[W + 2];
  const int r = threadIdx.x & 63, q = threadIdx.x >> 6;
  double a[16];  // column 4m + q
  long long tot = 0;
  for (int rep = 0; rep < REPS; ++rep) {
#pragma unroll
    for (int m = 0; m < 16; ++m) a[m] = (r >= 4 * m + q) ? A[(4 * m + q) * W + r] : 0.0;
    // column 0: owners (q == 0) compute s0 themselves from the raw a00
    if (r == 1 && q == 1) Dp[1] = a[0];  // raw a11 (column 1 = 4*0 + 1)
    if (q == 0) {
      const double s = sqrt(A[0]), y = 1.0 / s;
      if (r == 0) a[0] = s;
      else {
        a[0] = div_by(a[0], s, y);
        Lc[0][r] = a[0];
      }
    }
    __syncthreads();
    long long t0 = clock64();
#pragma unroll
    for (int j = 0; j < W - 1; ++j) {
      const int b = j & 1, j1 = j + 1, m1 = j1 >> 2;
      if (r > j) {
        const double lr = Lc[b][r];
        if (q == (j1 & 3)) {
          const double l1 = Lc[b][j1];
          const double d = fma(-l1, l1, Dp[j1]);
          const double s = sqrt(d), y = 1.0 / s;
          const double v = fma(-lr, l1, a[m1]);
          if (r == j1) a[m1] = s;
          else {
            a[m1] = div_by(v, s, y);
            Lc[b ^ 1][r] = a[m1];
          }
        }
#pragma unroll
        for (int m = 0; m < 16; ++m) {
          const int c = 4 * m + q;
          if (4 * m + 3 > j1 && c > j1 && c <= r) {
            a[m] = fma(-lr, Lc[b][c], a[m]);
            if (c == j + 2 && r == c) Dp[c] = a[m];
          }
        }
      }
      __syncthreads();
    }
    tot += clock64() - t0;
  }
#pragma unroll
  for (int m = 0; m < 16; ++m)
    if (r >= 4 * m + q) L[(4 * m + q) * W + r] = a[m];
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

// ---------------------------------------------------------------- V5: V4 without divergent branches
// Rows r <= j and elements above the diagonal are updated too (garbage that is
// never read nor stored): every condition left is warp-uniform (q) or a select.
__global__ void __launch_bounds__(256, 1) k_v5(const double* A, double* L, long long* clk) {
  __shared__ double Lc[2][W];
  __shared__ double Dp[W + 2];
  const int r = threadIdx.x & 63, q = threadIdx.x >> 6;
  double a[16];  // column 4m + q
  long long tot = 0;
  if (threadIdx.x < 2 * W) Lc[threadIdx.x >> 6][threadIdx.x & 63] = 0.0;
  for (int rep = 0; rep < REPS; ++rep) {
#pragma unroll
    for (int m = 0; m < 16; ++m) a[m] = (r >= 4 * m + q) ? A[(4 * m + q) * W + r] : 0.0;
    if (r == 1 && q == 1) Dp[1] = a[0];
    if (q == 0) {
      const double s = sqrt(A[0]), y = 1.0 / s;
      a[0] = (r == 0) ? s : div_by(a[0], s, y);
      Lc[0][r] = a[0];
    }
    __syncthreads();
    long long t0 = clock64();
#pragma unroll
    for (int j = 0; j < W - 1; ++j) {
      const int b = j & 1, j1 = j + 1, m1 = j1 >> 2;
      const double lr = Lc[b][r];
      if (q == (j1 & 3)) {  // warp-uniform: the owners of column j+1
        const double l1 = Lc[b][j1];
        const double d = fma(-l1, l1, Dp[j1]);
        const double s = sqrt(d), y = 1.0 / s;
        const double v = div_by(fma(-lr, l1, a[m1]), s, y);
        a[m1] = (r == j1) ? s : v;
        Lc[b ^ 1][r] = a[m1];
      }
#pragma unroll
      for (int m = 0; m < 16; ++m) {
        if (4 * m + 3 > j1) {                 // static
          const int c = 4 * m + q;
          if (c > j1) {                       // warp-uniform
            a[m] = fma(-lr, Lc[b][c], a[m]);
            if (c == j + 2 && r == c) Dp[c] = a[m];
          }
        }
      }
      __syncthreads();
    }
    tot += clock64() - t0;
  }
#pragma unroll
  for (int m = 0; m < 16; ++m)
    if (r >= 4 * m + q) L[(4 * m + q) * W + r] = a[m];
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

// ---------------------------------------------------------------- V6: V1 without divergent branches
__global__ void __launch_bounds__(256, 1) k_v6(const double* A, double* L, long long* clk) {
  __shared__ double Lcol[W];
  __shared__ double sy[2];
  const int r = threadIdx.x & 63, q = threadIdx.x >> 6;
  double a[16];
  long long tot = 0;
  if (threadIdx.x < W) Lcol[threadIdx.x] = 0.0;
  for (int rep = 0; rep < REPS; ++rep) {
#pragma unroll
    for (int m = 0; m < 16; ++m) a[m] = (r >= 4 * m + q) ? A[(4 * m + q) * W + r] : 0.0;
    __syncthreads();
    long long t0 = clock64();
#pragma unroll
    for (int j = 0; j < W; ++j) {
      const int mj = j >> 2, qj = j & 3;
      if (q == qj) {
        if (r == j) {
          const double s = sqrt(a[mj]);
          sy[0] = s;
          sy[1] = 1.0 / s;
        }
      }
      __syncthreads();
      if (q == qj) {
        const double s = sy[0];
        const double v = div_by(a[mj], s, sy[1]);
        a[mj] = (r == j) ? s : (r > j ? v : a[mj]);
        Lcol[r] = a[mj];
      }
      __syncthreads();
      const double lr = Lcol[r];
#pragma unroll
      for (int m = 0; m < 16; ++m) {
        if (4 * m + 3 > j) {
          const int c = 4 * m + q;
          if (c > j) a[m] = fma(-lr, Lcol[c], a[m]);
        }
      }
    }
    __syncthreads();
    tot += clock64() - t0;
  }
#pragma unroll
  for (int m = 0; m < 16; ++m)
    if (r >= 4 * m + q) L[(4 * m + q) * W + r] = a[m];
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

// ---------------------------------------------------------------- V7: V5 + deferred owner updates
// The owners of column j+1 only run the pivot chain before the barrier; their
// trailing updates from column j (columns >= j+5, not needed before iteration
// j+4) run in the next iteration, when they are not owners.  Triple-buffered
// column publication keeps column j readable through iteration j+1.
__global__ void __launch_bounds__(256, 1) k_v7(const double* A, double* L, long long* clk) {
  __shared__ double Lc[3][W];
  __shared__ double Dp[W + 2];
  const int r = threadIdx.x & 63, q = threadIdx.x >> 6;
  double a[16];  // column 4m + q
  long long tot = 0;
  if (threadIdx.x < W) Lc[0][threadIdx.x] = Lc[1][threadIdx.x] = Lc[2][threadIdx.x] = 0.0;
  for (int rep = 0; rep < REPS; ++rep) {
#pragma unroll
    for (int m = 0; m < 16; ++m) a[m] = (r >= 4 * m + q) ? A[(4 * m + q) * W + r] : 0.0;
    if (r == 1 && q == 1) Dp[1] = a[0];
    if (q == 0) {
      const double s = sqrt(A[0]), y = 1.0 / s;
      a[0] = (r == 0) ? s : div_by(a[0], s, y);
      Lc[0][r] = a[0];
    }
    __syncthreads();
    long long t0 = clock64();
#pragma unroll
    for (int j = 0; j < W - 1; ++j) {
      const int b = j % 3, bn = (j + 1) % 3, bp = (j + 2) % 3, j1 = j + 1, m1 = j1 >> 2;
      const double lr = Lc[b][r];
      if (q == (j1 & 3)) {  // owners of column j+1: the pivot chain only
        const double l1 = Lc[b][j1];
        const double d = fma(-l1, l1, Dp[j1]);
        const double s = sqrt(d), y = 1.0 / s;
        const double v = div_by(fma(-lr, l1, a[m1]), s, y);
        a[m1] = (r == j1) ? s : v;
        Lc[bn][r] = a[m1];
      } else {
        // deferred: this quarter owned column j (iteration j-1) -> its updates from column j-1
        if (j >= 1 && q == (j & 3)) {
          const double lp = Lc[bp][r];  // column j-1 lives in buffer (j-1)%3 == (j+2)%3
#pragma unroll
          for (int m = 0; m < 16; ++m) {
            if (4 * m + 3 > j) {
              const int c = 4 * m + q;
              if (c > j) a[m] = fma(-lp, Lc[bp][c], a[m]);
            }
          }
        }
#pragma unroll
        for (int m = 0; m < 16; ++m) {
          if (4 * m + 3 > j1) {
            const int c = 4 * m + q;
            if (c > j1) {
              a[m] = fma(-lr, Lc[b][c], a[m]);
              if (c == j + 2 && r == c) Dp[c] = a[m];
            }
          }
        }
      }
      __syncthreads();
    }
    tot += clock64() - t0;
  }
#pragma unroll
  for (int m = 0; m < 16; ++m)
    if (r >= 4 * m + q) L[(4 * m + q) * W + r] = a[m];
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

__global__ void __launch_bounds__(256, 1) k_v7t(const double* A, double* L, long long* clk, long long* ts) {
  __shared__ double Lc[3][W];
  __shared__ double Dp[W + 2];
  const int r = threadIdx.x & 63, q = threadIdx.x >> 6;
  double a[16];  // column 4m + q
  long long tot = 0;
  if (threadIdx.x < W) Lc[0][threadIdx.x] = Lc[1][threadIdx.x] = Lc[2][threadIdx.x] = 0.0;
  for (int rep = 0; rep < REPS; ++rep) {
#pragma unroll
    for (int m = 0; m < 16; ++m) a[m] = (r >= 4 * m + q) ? A[(4 * m + q) * W + r] : 0.0;
    if (r == 1 && q == 1) Dp[1] = a[0];
    if (q == 0) {
      const double s = sqrt(A[0]), y = 1.0 / s;
      a[0] = (r == 0) ? s : div_by(a[0], s, y);
      Lc[0][r] = a[0];
    }
    __syncthreads();
    long long t0 = clock64();
#pragma unroll
    for (int j = 0; j < W - 1; ++j) {
      const int b = j % 3, bn = (j + 1) % 3, bp = (j + 2) % 3, j1 = j + 1, m1 = j1 >> 2;
      const double lr = Lc[b][r];
      if (q == (j1 & 3)) {  // owners of column j+1: the pivot chain only
        long long c0 = clock64();
        const double l1 = Lc[b][j1];
        const double d = fma(-l1, l1, Dp[j1]);
        long long c1 = clock64();
        const double s = sqrt(d);
        long long c2 = clock64();
        const double y = 1.0 / s;
        long long c3 = clock64();
        const double v = div_by(fma(-lr, l1, a[m1]), s, y);
        a[m1] = (r == j1) ? s : v;
        Lc[bn][r] = a[m1];
        long long c4 = clock64();
        if (rep == REPS - 1 && r == 40 && j >= 8 && j < 24) {
          long long* o = ts + (j - 8) * 8;
          o[0] = c0; o[1] = c1; o[2] = c2; o[3] = c3; o[4] = c4;
        }
      } else {
        // deferred: this quarter owned column j (iteration j-1) -> its updates from column j-1
        if (j >= 1 && q == (j & 3)) {
          const double lp = Lc[bp][r];  // column j-1 lives in buffer (j-1)%3 == (j+2)%3
#pragma unroll
          for (int m = 0; m < 16; ++m) {
            if (4 * m + 3 > j) {
              const int c = 4 * m + q;
              if (c > j) a[m] = fma(-lp, Lc[bp][c], a[m]);
            }
          }
        }
#pragma unroll
        for (int m = 0; m < 16; ++m) {
          if (4 * m + 3 > j1) {
            const int c = 4 * m + q;
            if (c > j1) {
              a[m] = fma(-lr, Lc[b][c], a[m]);
              if (c == j + 2 && r == c) Dp[c] = a[m];
            }
          }
        }
      }
      __syncthreads();
      if (rep == REPS - 1 && r == 40 && q == ((j + 1) & 3) && j >= 8 && j < 24) ts[(j - 8) * 8 + 5] = clock64();
    }
    tot += clock64() - t0;
  }
#pragma unroll
  for (int m = 0; m < 16; ++m)
    if (r >= 4 * m + q) L[(4 * m + q) * W + r] = a[m];
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

// ---------------------------------------------------------------- S task: X <- X L^-T (64 x 64)
// S0: production solve_core (column quarters, one after another)
__device__ __forceinline__ void solve_v0(double (&b)[16], const double* Ls, double* Rc, double* Xpub, int ldp, int nc) {
  const int r = threadIdx.x & (W - 1), q = threadIdx.x >> 6;
  if (threadIdx.x < nc) Rc[threadIdx.x] = 1.0 / Ls[threadIdx.x * LDB + threadIdx.x];
  __syncthreads();
  for (int qq = 0; qq < 4 && 16 * qq < nc; ++qq) {
    if (q == qq) {
#pragma unroll
      for (int c = 0; c < 16; ++c) {
        const int col = 16 * qq + c;
        if (col < nc) {
          b[c] = div_by(b[c], Ls[col * LDB + col], Rc[col]);
#pragma unroll
          for (int c2 = c + 1; c2 < 16; ++c2) b[c2] = fma(-b[c], Ls[(16 * qq + c2) * LDB + col], b[c2]);
        }
      }
#pragma unroll
      for (int c = 0; c < 16; ++c) Xpub[r * ldp + 16 * qq + c] = b[c];
    }
    __syncthreads();
    if (q > qq) {
#pragma unroll
      for (int cc = 0; cc < 16; ++cc)
#pragma unroll
        for (int c = 0; c < 16; ++c)
          b[cc] = fma(-Xpub[r * ldp + 16 * qq + c], Ls[(16 * q + cc) * LDB + 16 * qq + c], b[cc]);
    }
  }
}

__global__ void __launch_bounds__(256, 1) k_s0(const double* A, const double* Lg, double* X, long long* clk) {
  extern __shared__ double dyn[];
  double *Ls = dyn, *Rc = dyn + W * LDB, *Xp = Rc + W;
  const int r = threadIdx.x & 63, q = threadIdx.x >> 6;
  for (int i = threadIdx.x; i < W * W; i += 256) Ls[(i % W) * LDB + i / W] = Lg[i];  // Ls[row][col]
  double b[16];
  long long tot = 0;
  for (int rep = 0; rep < REPS; ++rep) {
    for (int c = 0; c < 16; ++c) b[c] = A[(16 * q + c) * W + r];
    __syncthreads();
    long long t0 = clock64();
    solve_v0(b, Ls, Rc, Xp, 66, W);
    __syncthreads();
    tot += clock64() - t0;
  }
  for (int c = 0; c < 16; ++c) X[(16 * q + c) * W + r] = b[c];
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

// S1: four lanes per row in one warp (lane = 4 (r & 7) + q), columns q, q+4, ...;
// the solved x of column c is broadcast inside the row's lane quad by shuffle:
// no barrier at all.
__global__ void __launch_bounds__(256, 1) k_s1(const double* A, const double* Lg, double* X, long long* clk) {
  __shared__ double Ls[W * LDB], Rc[W];
  const int lane = threadIdx.x & 31, q = lane & 3, r = (threadIdx.x >> 5) * 8 + (lane >> 2);
  for (int i = threadIdx.x; i < W * W; i += 256) Ls[(i % W) * LDB + i / W] = Lg[i];
  double b[16];
  long long tot = 0;
  for (int rep = 0; rep < REPS; ++rep) {
#pragma unroll
    for (int m = 0; m < 16; ++m) b[m] = A[(4 * m + q) * W + r];
    if (threadIdx.x < W) Rc[threadIdx.x] = 1.0 / Ls[threadIdx.x * LDB + threadIdx.x];
    __syncthreads();
    long long t0 = clock64();
#pragma unroll
    for (int c = 0; c < W; ++c) {
      const int m = c >> 2, qc = c & 3;
      double x = div_by(b[m], Ls[c * LDB + c], Rc[c]);  // meaningful on the owner lane only
      x = __shfl_sync(0xffffffffu, x, (lane & ~3) | qc);
      b[m] = (q == qc) ? x : b[m];
#pragma unroll
      for (int m2 = 0; m2 < 16; ++m2) {
        if (4 * m2 + 3 > c) {
          const int c2 = 4 * m2 + q;
          b[m2] = (c2 > c) ? fma(-x, Ls[c2 * LDB + c], b[m2]) : b[m2];
        }
      }
    }
    __syncthreads();
    tot += clock64() - t0;
  }
#pragma unroll
  for (int m = 0; m < 16; ++m) X[(4 * m + q) * W + r] = b[m];
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

// S2: S1 software-pipelined: the next column's element is updated and divided
// (and broadcast) before the rest of this column's updates are issued.
__global__ void __launch_bounds__(256, 1) k_s2(const double* A, const double* Lg, double* X, long long* clk) {
  __shared__ double Ls[W * LDB], Rc[W];
  const int lane = threadIdx.x & 31, q = lane & 3, r = (threadIdx.x >> 5) * 8 + (lane >> 2);
  const int quad = lane & ~3;
  for (int i = threadIdx.x; i < W * W; i += 256) Ls[(i % W) * LDB + i / W] = Lg[i];
  double b[16];
  long long tot = 0;
  for (int rep = 0; rep < REPS; ++rep) {
#pragma unroll
    for (int m = 0; m < 16; ++m) b[m] = A[(4 * m + q) * W + r];
    if (threadIdx.x < W) Rc[threadIdx.x] = 1.0 / Ls[threadIdx.x * LDB + threadIdx.x];
    __syncthreads();
    long long t0 = clock64();
    // column 0
    double x = __shfl_sync(0xffffffffu, div_by(b[0], Ls[0], Rc[0]), quad);
    b[0] = (q == 0) ? x : b[0];
#pragma unroll
    for (int c = 0; c < W; ++c) {
      // x = x_c (all lanes of the quad).  Element c+1 first:
      double xn = 0.0;
      if (c + 1 < W) {
        const int e = c + 1, me = e >> 2, qe = e & 3;
        b[me] = (q == qe) ? fma(-x, Ls[e * LDB + c], b[me]) : b[me];
        xn = __shfl_sync(0xffffffffu, div_by(b[me], Ls[e * LDB + e], Rc[e]), quad | qe);
      }
      // the rest of column c's updates (elements c+2 ..)
#pragma unroll
      for (int m2 = 0; m2 < 16; ++m2) {
        if (4 * m2 + 3 > c + 1) {
          const int c2 = 4 * m2 + q;
          b[m2] = (c2 > c + 1) ? fma(-x, Ls[c2 * LDB + c], b[m2]) : b[m2];
        }
      }
      if (c + 1 < W) {
        b[(c + 1) >> 2] = (q == ((c + 1) & 3)) ? xn : b[(c + 1) >> 2];
        x = xn;
      }
    }
    __syncthreads();
    tot += clock64() - t0;
  }
#pragma unroll
  for (int m = 0; m < 16; ++m) X[(4 * m + q) * W + r] = b[m];
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

// DMMA "hog": one CTA per SM issuing dependent-free DMMA (like a co-resident GEMM CTA)
__global__ void __launch_bounds__(256, 1) k_hog(double* out, int iters) {
  double acc[8][2] = {};
  double a = 1.0 + threadIdx.x * 1e-9, b = 1.0 - threadIdx.x * 1e-9;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) stfk::dmma_8x8x4(acc[i][0], acc[i][1], a, b);
  }
  double s = 0;
  for (int i = 0; i < 8; ++i) s += acc[i][0] + acc[i][1];
  if (s == 1.2345) out[threadIdx.x] = s;
}

// ---------------------------------------------------------------- V8: V7 rolled by 4 columns
// Same arithmetic as V7, but the column loop runs over groups of 4 columns at
// run time (the 4 columns of a group unrolled) and the register window shifts
// by one element per group, so every register index is static: code ~16x
// smaller than the fully unrolled V7 (instruction-cache footprint).
// a[m] holds column 4 (g + m) + q during group g; finished columns leave a[0]
// at the shift and are published to S[r * LDB + c].
__global__ void __launch_bounds__(256, 1) k_v8(const double* A, double* L, long long* clk) {
  __shared__ double Lc[3][W];
  __shared__ double Dp[W + 2];
  __shared__ double S[W * LDB];
  const int r = threadIdx.x & 63, q = threadIdx.x >> 6;
  double a[16];
  long long tot = 0;
  for (int rep = 0; rep < REPS; ++rep) {
#pragma unroll
    for (int m = 0; m < 16; ++m) a[m] = (r >= 4 * m + q) ? A[(4 * m + q) * W + r] : 0.0;
    if (r == 1 && q == 1) Dp[1] = a[0];
    if (r == 0 && q == 0) Dp[0] = a[0];
    __syncthreads();
    if (q == 0) {
      const double s = sqrt(Dp[0]), y = 1.0 / s;
      a[0] = (r == 0) ? s : div_by(a[0], s, y);
      Lc[0][r] = a[0];
    }
    __syncthreads();
    long long t0 = clock64();
    for (int g = 0; g < 16; ++g) {
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int j = 4 * g + u;
        if (j + 1 < W) {
          const int b = j % 3, bn = (j + 1) % 3, bp = (j + 2) % 3, j1 = j + 1;
          // element of column j1 in the window: u < 3 -> a[0] of quarter u+1; u == 3 -> a[1] of quarter 0
          const int w1 = (u == 3) ? 1 : 0;
          const double lr = Lc[b][r];
          if (q == ((u + 1) & 3)) {
            const double l1 = Lc[b][j1];
            const double d = fma(-l1, l1, Dp[j1]);
            const double s = sqrt(d), y = 1.0 / s;
            const double v = div_by(fma(-lr, l1, a[w1]), s, y);
            a[w1] = (r == j1) ? s : v;
            Lc[bn][r] = a[w1];
          } else {
            if (j >= 1 && q == u) {  // deferred: updates from column j-1 to this quarter's columns > j
              const double lp = Lc[bp][r];
#pragma unroll
              for (int m = 0; m < 16; ++m)
                if (4 * m + q > u) a[m] = fma(-lp, Lc[bp][4 * (g + m) + q & 63], a[m]);
            }
#pragma unroll
            for (int m = 0; m < 16; ++m) {
              if (4 * m + q > u + 1) {  // column 4(g+m)+q > j1
                a[m] = fma(-lr, Lc[b][4 * (g + m) + q & 63], a[m]);
                if (4 * m + q == u + 2 && r == j + 2) Dp[j + 2] = a[m];
              }
            }
          }
        }
        __syncthreads();
      }
      // column 4g+q is final: publish it and shift the window
      if (r >= 4 * g + q) S[r * LDB + 4 * g + q] = a[0];
#pragma unroll
      for (int m = 0; m < 15; ++m) a[m] = a[m + 1];
      a[15] = 0.0;
    }
    __syncthreads();
    tot += clock64() - t0;
  }
  for (int i = threadIdx.x; i < W * W; i += 256) {
    const int rr = i & 63, cc = i >> 6;
    if (rr >= cc) L[cc * W + rr] = S[rr * LDB + cc];
  }
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

__global__ void __launch_bounds__(256, 1) k_v9(const double* A, double* L, long long* clk) {
  __shared__ double Lc[3][W];
  __shared__ double Dp[W + 2];
  __shared__ double S[W * LDB];
  const int r = threadIdx.x & 63, q = threadIdx.x >> 6;
  double a[16];
  long long tot = 0;
  for (int rep = 0; rep < REPS; ++rep) {
#pragma unroll
    for (int m = 0; m < 16; ++m) a[m] = (r >= 4 * m + q) ? A[(4 * m + q) * W + r] : 0.0;
    if (r == 1 && q == 1) Dp[1] = a[0];
    if (r == 0 && q == 0) Dp[0] = a[0];
    __syncthreads();
    if (q == 0) {
      const double s = sqrt(Dp[0]), y = 1.0 / s;
      a[0] = (r == 0) ? s : div_by(a[0], s, y);
      Lc[0][r] = a[0];
    }
    __syncthreads();
    long long t0 = clock64();
    for (int g = 0; g < 16; ++g) {
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int j = 4 * g + u;
        if (j + 1 < W) {
          const int b = j % 3, bn = (j + 1) % 3, bp = (j + 2) % 3, j1 = j + 1;
          // element of column j1 in the window: u < 3 -> a[0] of quarter u+1; u == 3 -> a[1] of quarter 0
          const int w1 = (u == 3) ? 1 : 0;
          const double lr = Lc[b][r];
          if (q == ((u + 1) & 3)) {
            const double l1 = Lc[b][j1];
            const double d = fma(-l1, l1, Dp[j1]);
            const double s = sqrt(d), y = 1.0 / s;
            const double v = div_by(fma(-lr, l1, a[w1]), s, y);
            a[w1] = (r == j1) ? s : v;
            Lc[bn][r] = a[w1];
          } else {
            if (j >= 1 && q == u) {  // deferred: updates from column j-1 to this quarter's columns > j
              const double lp = Lc[bp][r];
              const double* Lp = &Lc[bp][4 * g + q];
#pragma unroll
              for (int m = 0; m < 16; ++m)
                if (4 * m + q > u && m < 16 - g) a[m] = fma(-lp, Lp[4 * m], a[m]);
            }
            const double* Lb = &Lc[b][4 * g + q];
#pragma unroll
            for (int m = 0; m < 16; ++m) {
              if (4 * m + q > u + 1 && m < 16 - g) {  // column 4(g+m)+q > j1, inside the block
                a[m] = fma(-lr, Lb[4 * m], a[m]);
                if (4 * m + q == u + 2 && r == j + 2) Dp[j + 2] = a[m];
              }
            }
          }
        }
        __syncthreads();
      }
      // column 4g+q is final: publish it and shift the window
      if (r >= 4 * g + q) S[r * LDB + 4 * g + q] = a[0];
#pragma unroll
      for (int m = 0; m < 15; ++m) a[m] = a[m + 1];
      a[15] = 0.0;
    }
    __syncthreads();
    tot += clock64() - t0;
  }
  for (int i = threadIdx.x; i < W * W; i += 256) {
    const int rr = i & 63, cc = i >> 6;
    if (rr >= cc) L[cc * W + rr] = S[rr * LDB + cc];
  }
  if (threadIdx.x == 0) clk[0] = tot / REPS;
}

int main() {
  double hA[W * W];
  srand(7);
  for (int i = 0; i < W; ++i)
    for (int j = 0; j <= i; ++j) {
      const double v = (rand() / (double)RAND_MAX) * 2 - 1;
      hA[j * W + i] = hA[i * W + j] = v + (i == j ? W : 0.0);
    }
  double *A, *L;
  long long* clk;
  cudaMalloc(&A, sizeof hA);
  cudaMalloc(&L, 10 * sizeof hA);
  cudaMallocManaged(&clk, 32 * sizeof(long long));
  long long* ts;
  cudaMallocManaged(&ts, 16 * 8 * sizeof(long long));
  cudaMemcpy(A, hA, sizeof hA, cudaMemcpyHostToDevice);
  cudaMemset(L, 0, 10 * sizeof hA);
  for (int it = 0; it < 2; ++it) {
    k_v0<<<1, 256>>>(A, L, clk + 0);
    k_v1<<<1, 256>>>(A, L + W * W, clk + 1);
    k_v2<<<1, 256>>>(A, L + 2 * W * W, clk + 2);
    k_v3<<<1, 256>>>(A, L + 3 * W * W, clk + 3);
    k_v4<<<1, 256>>>(A, L + 4 * W * W, clk + 4);
    k_v5<<<1, 256>>>(A, L + 5 * W * W, clk + 5);
    k_v6<<<1, 256>>>(A, L + 6 * W * W, clk + 6);
    k_v7<<<1, 256>>>(A, L + 7 * W * W, clk + 7);
    k_v8<<<1, 256>>>(A, L + 8 * W * W, clk + 9);
    k_v9<<<1, 256>>>(A, L + 9 * W * W, clk + 13);
    k_v7t<<<1, 256>>>(A, L + 7 * W * W, clk + 8, ts);
    cudaDeviceSynchronize();
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    printf("CUDA error %s\n", cudaGetErrorString(e));
    return 1;
  }
  static double hL[10][W * W];
  cudaMemcpy(hL, L, 10 * sizeof hA, cudaMemcpyDeviceToHost);
  const char* names[] = {"V0 production quarters", "V1 interleaved, 2 syncthreads/col", "V2 row owner, 2 bar64/col",
                         "V3 interleaved, 1 syncthreads/col", "V4 redundant pivot, 1 syncthreads/col",
                         "V5 = V4 branch-free", "V6 = V1 branch-free", "V7 = V5 + deferred owner updates"};
  {
    int diff = 0;
    for (int i = 0; i < W; ++i)
      for (int j = 0; j <= i; ++j) diff += hL[8][j * W + i] != hL[0][j * W + i];
    printf("%-36s %6lld clk total  %5.0f clk/col  mismatches vs V0: %d\n", "V8 = V7 rolled by 4 (window shift)", clk[9],
           clk[9] / 64.0, diff);
    diff = 0;
    for (int i = 0; i < W; ++i)
      for (int j = 0; j <= i; ++j) diff += hL[9][j * W + i] != hL[0][j * W + i];
    printf("%-36s %6lld clk total  %5.0f clk/col  mismatches vs V0: %d\n", "V9 = V8 + bounded window", clk[13],
           clk[13] / 64.0, diff);
  }
  for (int v = 0; v < 8; ++v) {
    int diff = 0;
    for (int i = 0; i < W; ++i)
      for (int j = 0; j <= i; ++j) diff += hL[v][j * W + i] != hL[0][j * W + i];
    printf("%-36s %6lld clk total  %5.0f clk/col  mismatches vs V0: %d\n", names[v], clk[v], clk[v] / 64.0, diff);
  }
  {
    // S lab: random X, L = the V0 factor of A
    static double hX[W * W];
    for (int i = 0; i < W * W; ++i) hX[i] = (rand() / (double)RAND_MAX) * 2 - 1;
    double *Xin, *Xo, *Lf;
    cudaMalloc(&Xin, sizeof hX);
    cudaMalloc(&Xo, 3 * sizeof hX);
    cudaMalloc(&Lf, sizeof hX);
    static double hLf[W * W];
    for (int i = 0; i < W * W; ++i) hLf[i] = 0;
    for (int i = 0; i < W; ++i)
      for (int j = 0; j <= i; ++j) hLf[j * W + i] = hL[0][j * W + i];
    cudaMemcpy(Lf, hLf, sizeof hX, cudaMemcpyHostToDevice);
    cudaMemcpy(Xin, hX, sizeof hX, cudaMemcpyHostToDevice);
    for (int it = 0; it < 2; ++it) {
      cudaFuncSetAttribute(k_s0, cudaFuncAttributeMaxDynamicSharedMemorySize, 80000);
      k_s0<<<1, 256, (W * LDB + W + W * 66) * 8>>>(Xin, Lf, Xo, clk + 10);
      k_s1<<<1, 256>>>(Xin, Lf, Xo + W * W, clk + 11);
      k_s2<<<1, 256>>>(Xin, Lf, Xo + 2 * W * W, clk + 12);
      cudaDeviceSynchronize();
    }
    static double hXo[3][W * W];
    cudaMemcpy(hXo, Xo, 3 * sizeof hX, cudaMemcpyDeviceToHost);
    int diff = 0, diff2 = 0;
    for (int i = 0; i < W * W; ++i) diff += hXo[0][i] != hXo[1][i], diff2 += hXo[0][i] != hXo[2][i];
    printf("S2 pipelined shuffle      %6lld clk  %4.0f clk/col  mismatches %d\n", clk[12], clk[12] / 64.0, diff2);
    printf("S0 production solve_core  %6lld clk  %4.0f clk/col\nS1 lane-quad shuffle      %6lld clk  %4.0f clk/col  mismatches %d\n",
           clk[10], clk[10] / 64.0, clk[11], clk[11] / 64.0, diff);
  }
  {
    // the same Cholesky variants while every SM also runs a DMMA-issuing CTA
    double* hout;
    cudaMalloc(&hout, 4096);
    cudaStream_t sh, sc;
    cudaStreamCreateWithFlags(&sh, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&sc, cudaStreamNonBlocking);
    k_hog<<<148, 256, 0, sh>>>(hout, 400000);  // ~100 ms of DMMA on every SM
    for (int it = 0; it < 2; ++it) {
      k_v0<<<1, 256, 0, sc>>>(A, L, clk + 20);
      k_v1<<<1, 256, 0, sc>>>(A, L + W * W, clk + 21);
      k_v5<<<1, 256, 0, sc>>>(A, L + 5 * W * W, clk + 22);
      k_v7<<<1, 256, 0, sc>>>(A, L + 7 * W * W, clk + 23);
      cudaStreamSynchronize(sc);
    }
    cudaDeviceSynchronize();
    printf("under DMMA contention: V0 %4.0f  V1 %4.0f  V5 %4.0f  V7 %4.0f clk/col\n", clk[20] / 64.0, clk[21] / 64.0,
           clk[22] / 64.0, clk[23] / 64.0);
  }
  printf("owner thread r=40, per column: loads+fma | sqrt | rcp | div+sts | to after-barrier\n");
  for (int j = 0; j < 16; ++j) {
    long long* o = ts + j * 8;
    printf("j=%2d  %4lld %4lld %4lld %4lld %4lld  total %lld\n", j + 8, o[1] - o[0], o[2] - o[1], o[3] - o[2], o[4] - o[3],
           o[5] - o[4], (j < 15 ? ts[(j + 1) * 8] : o[5]) - o[0]);
  }
  return 0;
}
