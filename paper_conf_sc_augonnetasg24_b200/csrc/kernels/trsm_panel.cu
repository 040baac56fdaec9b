// K3 TRSM tile kernel, row-panel form (north_star "TRSM as
// a blocked triangular solve that calls those same tensor-core tiles").
//
//   TRSM(i,k):  X <- B L^-T   (X L^T = B),  B: M x n,  L: n x n lower
//
// Rows of X are independent, so each CTA owns 32 rows and sweeps the 64-wide
// column blocks left to right (left-looking):
//   for jb:  acc = B[rows, jb] - sum_{pb<jb} X[rows, pb] L[jb, pb]^T   (DMMA, operands
//            staged by cp.async into padded smem, two stages)
//            X[rows, jb] = acc L[jb, jb]^-T                              (substitution)
// No cross-CTA dependencies: no flags, no waiting, every SM-cycle is work.  The
// k-order of every sum is fixed, so results are bit-identical run to run; the
// diagonal solve returns the correctly rounded quotient by L_cc (div_by: one IEEE
// reciprocal per column, Markstein correction on the chain), so unit-diagonal
// dyadic inputs stay exact (pin P2).
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>

#include "ptx.cuh"
#include "solve_block.cuh"
#include "tile_ops.hpp"

namespace stfk {

// diagonal block staged transposed: LdT[c * LD + r] = L(r, c)
template <int LD>
struct ColT {
  const double* p;
  __device__ __forceinline__ double operator()(int r, int c) const { return p[c * LD + r]; }
};

// Rows per CTA: 32 (3 stages, latency), 64 (2 stages, higher DMMA efficiency) or
// 128 (2 half-depth stages: eight solver warps, two per SM sub-partition, so two
// substitution chains interleave on each FP64 pipe; full 64-column blocks only).
// A pipeline stage holds KD of the 64 k-columns of one update block.
template <int BM_, int KD_ = 64>
struct TP {
  static constexpr int BM = BM_, W = 64, NT = 256, STAGES = (BM_ == 32) ? 3 : 2, KD = KD_, R = 64 / KD_;
  static constexpr int SA = BM + 4;  // As[k][m] stride (= 4 mod 16 -> conflict-free fragment loads)
  static constexpr int SB = 68;      // Bs[k][n] stride
  static constexpr int SS = 65;      // solve scratch stride
  static constexpr int SL = 66;      // LdT stride (16-byte aligned columns for cp.async; warp-broadcast reads)
  static constexpr int FM = BM / 16; // m-fragments per warp (2 x 4 warp grid, warp tile BM/2 x 16)
  static constexpr int STAGE = KD * SA + KD * SB;                   // doubles per pipeline stage
  static constexpr int SOLVE = BM * SS + W * SL + W;                // S, LdT, Rc
  static constexpr int SMEM_BYTES = (STAGES * STAGE + SOLVE) * 8;  // ~210 / ~207 / ~203 KB
};

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(smem)), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ double negd_tp(double x) {
  return __longlong_as_double(__double_as_longlong(x) ^ (long long)0x8000000000000000ULL);
}

// dst[k * ld + r] = G(r, k) for r < rows (<= R), k < kc (<= KD); zero-filled otherwise.
// Fast path (full block, 16-byte aligned columns) uses cp.async; else scalar loads.
template <int R, int KD = 64>
__device__ __forceinline__ void stage_block(double* dst, int ld, const double* G, int64_t ldg, int rows, int kc,
                                            bool fast) {
  constexpr int NT = 256;
  if (fast) {
    constexpr int CH = R / 2;  // 16-byte chunks per column
    for (int idx = threadIdx.x; idx < CH * KD; idx += NT) {
      const int k = idx / CH, c = idx % CH;
      cp_async16(dst + k * ld + 2 * c, G + (int64_t)k * ldg + 2 * c);
    }
  } else {
    for (int idx = threadIdx.x; idx < R * KD; idx += NT) {
      const int k = idx / R, r = idx % R;
      dst[k * ld + r] = (r < rows && k < kc) ? __ldcg(G + (int64_t)k * ldg + r) : 0.0;
    }
  }
}

template <int BMT, int KDT = 64>
__global__ void __launch_bounds__(256, 1) trsm_panel_kernel(const double* __restrict__ L, int64_t ldl, int n,
                                                             double* __restrict__ X, int64_t ldx, int M,
                                                             const Mirrors mir) {
  using tp = TP<BMT, KDT>;
  extern __shared__ __align__(16) double smt[];
  const int r0 = blockIdx.x * tp::BM;
  const int rows = min(tp::BM, M - r0);
  const int Nb = (n + tp::W - 1) / tp::W;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int wm0 = (warp & 1) * (tp::BM / 2), wn0 = (warp >> 1) * 16;
  double* Xr = X + r0;  // this CTA's rows
  const bool rows_fast = (rows == tp::BM) && ((ldx & 1) == 0) && ((reinterpret_cast<uintptr_t>(Xr) & 15) == 0);
  const bool lal = ((ldl & 1) == 0) && ((reinterpret_cast<uintptr_t>(L) & 15) == 0);
  double* S = smt + tp::STAGES * tp::STAGE;  // solve scratch (never aliases the pipeline)
  double* LdT = S + tp::BM * tp::SS;         // LdT[p * SL + c] = L(c0 + c, c0 + p); upper part unused
  double* Rc = LdT + tp::W * tp::SL;

  // Stage (jb, s) = operands of the update of column block jb by k-columns
  // [s KD, (s + 1) KD) (block pb = s / R); it lives in ring slot s % STAGES and is
  // one cp.async group.  X block pb may be staged only after it has been solved,
  // so the first STAGES-1 stages of jb+1 are issued in two halves: those with
  // pb < jb before the solve of jb (overlapping their latency with it), those
  // with pb == jb after it.  Every prologue commits exactly STAGES-1 stage groups
  // (plus the diagonal block's) and every update iteration one group.
  auto issue = [&](int jb, int s) {
    const int c0 = jb * tp::W, nc = min(tp::W, n - c0);
    double* As = smt + (s % tp::STAGES) * tp::STAGE;
    double* Bs = As + tp::KD * tp::SA;
    stage_block<tp::BM, tp::KD>(As, tp::SA, Xr + (int64_t)s * tp::KD * ldx, ldx, rows, tp::KD, rows_fast);
    stage_block<tp::W, tp::KD>(Bs, tp::SB, L + (int64_t)s * tp::KD * ldl + c0, ldl, nc, tp::KD,
                               lal && nc == tp::W);
  };
  // diagonal block L(jb, jb) -> LdT (cp.async when full and aligned)
  auto issue_diag = [&](int jb) {
    const int c0 = jb * tp::W, nc = min(tp::W, n - c0);
    const double* G = L + (int64_t)c0 * ldl + c0;
    if (lal && nc == tp::W) {
      for (int idx = threadIdx.x; idx < 32 * tp::W; idx += tp::NT) {
        const int p = idx / 32, ch = idx % 32;
        cp_async16(LdT + p * tp::SL + 2 * ch, G + (int64_t)p * ldl + 2 * ch);
      }
    } else {
      for (int idx = threadIdx.x; idx < tp::W * tp::W; idx += tp::NT) {
        const int p = idx / tp::W, c = idx % tp::W;
        LdT[p * tp::SL + c] = (c < nc && p < nc) ? __ldg(G + (int64_t)p * ldl + c) : 0.0;
      }
    }
  };
  auto prologue_pre = [&](int jn) {
    for (int p = 0; p < tp::STAGES - 1; ++p)
      if (p < (jn - 1) * tp::R) {
        issue(jn, p);
        cp_async_commit();
      }
  };
  auto prologue_post = [&](int jn) {
    issue_diag(jn);
    cp_async_commit();
    for (int p = 0; p < tp::STAGES - 1; ++p)
      if (p >= (jn - 1) * tp::R) {
        if (p < jn * tp::R) issue(jn, p);
        cp_async_commit();
      }
  };

  issue_diag(0);
  cp_async_commit();
  for (int jb = 0; jb < Nb; ++jb) {
    const int c0 = jb * tp::W;
    const int nc = min(tp::W, n - c0);
    // acc = B[rows, jb-block]
    double acc[tp::FM][2][2];
#pragma unroll
    for (int i = 0; i < tp::FM; ++i)
#pragma unroll
      for (int j = 0; j < 2; ++j)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int r = wm0 + 8 * i + g, c = wn0 + 8 * j + 2 * t + h;
          acc[i][j][h] = (r < rows && c < nc) ? __ldcg(Xr + (int64_t)(c0 + c) * ldx + r) : 0.0;
        }
    // left-looking update over the k-columns of blocks pb < jb, one barrier per stage
    for (int st = 0; st < jb * tp::R; ++st) {
      cp_async_wait<tp::STAGES - 2>();
      __syncthreads();
      const int pf = st + tp::STAGES - 1;  // refill the slot consumed at st - 1
      if (pf < jb * tp::R) issue(jb, pf);
      cp_async_commit();
      const double* As = smt + (st % tp::STAGES) * tp::STAGE;
      const double* Bs = As + tp::KD * tp::SA;
#pragma unroll 4
      for (int k0 = 0; k0 < tp::KD; k0 += 4) {
        double a[tp::FM], b[2];
#pragma unroll
        for (int i = 0; i < tp::FM; ++i) a[i] = As[(k0 + t) * tp::SA + wm0 + 8 * i + g];
#pragma unroll
        for (int j = 0; j < 2; ++j) b[j] = negd_tp(Bs[(k0 + t) * tp::SB + wn0 + 8 * j + g]);
#pragma unroll
        for (int i = 0; i < tp::FM; ++i)
#pragma unroll
          for (int j = 0; j < 2; ++j) dmma_8x8x4(acc[i][j][0], acc[i][j][1], a[i], b[j]);
      }
    }
    cp_async_wait<0>();
    __syncthreads();  // ring free
    if (jb + 1 < Nb) prologue_pre(jb + 1);
    // ---- diagonal solve, LdT = L(jb,jb) (landed: waited above), Rc[c] = 1 / L_cc
    if (nc == tp::W) {
      // full block: BM/16 warps, one per SM sub-partition, each solve 16 rows
      // (solve_block: 8-column sub-blocks by substitution, their updates on DMMA)
      double* Xp = S;  // BM/16 swizzled [16 x 64] panels (S is free here)
#pragma unroll
      for (int i = 0; i < tp::FM; ++i)
#pragma unroll
        for (int j = 0; j < 2; ++j)
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int row = wm0 + 8 * i + g, col = wn0 + 8 * j + 2 * t + h;
            Xp[(row >> 4) * 16 * tp::W + sb::xo(row & 15, col)] = acc[i][j][h];
          }
      if (threadIdx.x < tp::W) Rc[threadIdx.x] = 1.0 / LdT[threadIdx.x * tp::SL + threadIdx.x];
      __syncthreads();
      if (warp < tp::BM / 16) {
        const int rr = 16 * warp + (lane & 15);
        solve_block<0>(Xp + warp * 16 * tp::W, 0, ColT<tp::SL>{LdT}, Rc, lane, X + (int64_t)c0 * ldx + r0, ldx, rr,
                       lane < 16 && rr < rows);
      }
      if (mir.n > 0) {  // fused push (NEXT-3): the finished block into the consumers' replicas
        __syncthreads();
        for (int idx = threadIdx.x; idx < tp::BM * tp::W; idx += tp::NT) {
          const int rr = idx % tp::BM, cc = idx / tp::BM;
          if (rr < rows) {
            const double v = Xp[(rr >> 4) * 16 * tp::W + sb::xo(rr & 15, cc)];
            const int64_t off = (int64_t)(c0 + cc) * ldx + r0 + rr;
#pragma unroll
            for (int m = 0; m < 7; ++m)
              if (m < mir.n) mirror_st(mir.p[m] + off, v, mir.mc);
          }
        }
        mirror_fence(mir.mc);
      }
    } else if constexpr (tp::BM <= 64) {
      // ragged last block: row-chunked substitution, S[r][c] = acc
  #pragma unroll
      for (int i = 0; i < tp::FM; ++i)
  #pragma unroll
        for (int j = 0; j < 2; ++j)
  #pragma unroll
          for (int h = 0; h < 2; ++h) S[(wm0 + 8 * i + g) * tp::SS + wn0 + 8 * j + 2 * t + h] = acc[i][j][h];
      if (threadIdx.x < nc) Rc[threadIdx.x] = 1.0 / LdT[threadIdx.x * tp::SL + threadIdx.x];
      __syncthreads();
      // thread (q = tid / BM, r = tid % BM), q < 4, owns row r of the 16-column chunk q.
      // Chunk q solves its columns in registers, publishes x to S, later chunks
      // subtract its contribution.
      const int q = threadIdx.x / tp::BM, r = threadIdx.x % tp::BM;
      double b[16];
      if (q < 4) {
  #pragma unroll
        for (int c = 0; c < 16; ++c) b[c] = S[r * tp::SS + 16 * q + c];
      }
      for (int qq = 0; qq < 4; ++qq) {
        if (q == qq) {
  #pragma unroll
          for (int c = 0; c < 16; ++c) {
            const int col = 16 * qq + c;
            if (col < nc) {
              b[c] = div_by(b[c], LdT[col * tp::SL + col], Rc[col]);
  #pragma unroll
              for (int c2 = c + 1; c2 < 16; ++c2) b[c2] = fma(-b[c], LdT[col * tp::SL + 16 * qq + c2], b[c2]);
            }
          }
  #pragma unroll
          for (int c = 0; c < 16; ++c) S[r * tp::SS + 16 * qq + c] = b[c];
        }
        __syncthreads();
        if (q > qq && q < 4) {
  #pragma unroll
          for (int cc = 0; cc < 16; ++cc)
  #pragma unroll
            for (int c = 0; c < 16; ++c)
              b[cc] = fma(-S[r * tp::SS + 16 * qq + c], LdT[(16 * qq + c) * tp::SL + 16 * q + cc], b[cc]);
        }
      }
      if (q < 4 && r < rows) {
  #pragma unroll
        for (int c = 0; c < 16; ++c) {
          const int col = 16 * q + c;
          if (col < nc) {
            const int64_t off = (int64_t)(c0 + col) * ldx + r0 + r;
            X[off] = b[c];
            // fused push (NEXT-3): the finished value also goes straight into the
            // consumers' replicas (peer memory over NVLink / another slot's arena)
  #pragma unroll
            for (int m = 0; m < 7; ++m)
              if (m < mir.n) mirror_st(mir.p[m] + off, b[c], mir.mc);
          }
        }
        mirror_fence(mir.n > 0 ? mir.mc : 0);
      }
    }
    __threadfence();  // X[rows, jb] is re-read (cp.async.cg, L2) by the next jb iterations
    __syncthreads();
    if (jb + 1 < Nb) prologue_post(jb + 1);
  }
}

cudaError_t trsm_panel_init_attrs() {
  cudaError_t e = cudaFuncSetAttribute(trsm_panel_kernel<32>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       TP<32>::SMEM_BYTES);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(trsm_panel_kernel<64>, cudaFuncAttributeMaxDynamicSharedMemorySize, TP<64>::SMEM_BYTES);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(trsm_panel_kernel<128, 32>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             TP<128, 32>::SMEM_BYTES);
  return e;
}

static int trsm_rows() {
  static int v = [] {
    const char* e = getenv("STF_TRSM_ROWS");
    const int r = e ? atoi(e) : 64;
    return (r == 32 || r == 128) ? r : 64;
  }();
  return v;
}

cudaError_t trsm_panel(cudaStream_t stream, int prio, int M, int n, const double* L, int64_t ldl, double* B,
                       int64_t ldb, int rows_per_cta, const Mirrors* mirrors) {
  Mirrors mir{};
  if (mirrors) mir = *mirrors;
  if (M <= 0 || n <= 0) return cudaSuccess;
  int bm = rows_per_cta == 32 || rows_per_cta == 64 || rows_per_cta == 128 ? rows_per_cta : trsm_rows();
  if (bm == 128 && n % 64 != 0) bm = 64;  // the 128-row form solves full 64-column blocks only
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((M + bm - 1) / bm);
  cfg.blockDim = dim3(256);
  cfg.dynamicSmemBytes = bm == 32 ? TP<32>::SMEM_BYTES : bm == 64 ? TP<64>::SMEM_BYTES : TP<128, 32>::SMEM_BYTES;
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = prio;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  ++launch_count();
  if (bm == 32) return cudaLaunchKernelEx(&cfg, trsm_panel_kernel<32>, L, ldl, n, B, ldb, M, mir);
  if (bm == 128) return cudaLaunchKernelEx(&cfg, trsm_panel_kernel<128, 32>, L, ldl, n, B, ldb, M, mir);
  return cudaLaunchKernelEx(&cfg, trsm_panel_kernel<64>, L, ldl, n, B, ldb, M, mir);
}

}  // namespace stfk
