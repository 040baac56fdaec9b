// K3 TRSM tile kernel, resident-panel form with warp specialisation (SURVEY.md
// §2.3 K3; north_star "TRSM as a blocked triangular solve that calls those same
// tensor-core tiles").
//
//   TRSM(i,k):  X <- B L^-T   (X L^T = B),  B: M x n,  L: n x n lower
//
// Rows of X are independent.  Each CTA owns R = 16 rows and keeps its whole
// R x n row panel resident in shared memory (n <= 1024: 128 KB), so a solved
// column block is never re-read through L2.  Left-looking over 64-wide column
// blocks jb, with two warp roles running concurrently:
//
//   MMA warps (6, SM sub-partitions 0-2):  acc = - sum_{pb<jb} X[:,pb] L[jb,pb]^T
//                     on the DMMA pipe, A operand from the resident panel, L
//                     blocks streamed by TMA (128B-swizzled boxes) through a
//                     4-slot mbarrier ring (tr::NST); k-groups split mod 3 and
//                     combined in a fixed order; the terms pb < jb-1 do not depend
//                     on the block being solved and run while it is solved.
//   producer warp (1, sub-partition 3): issues the TMA loads of the ring.
//   solver warp (1, sub-partition 3): X[:,jb] <- X[:,jb] L[jb,jb]^-T by
//                     substitution in 8-column sub-blocks (register chain with
//                     correctly rounded division, sub-block updates on DMMA),
//                     then to global memory (+ fused-push mirrors).
//
// Overlap with the producing POTRF (programmatic dependent launch, TRSM(k+1,k)
// of the panel chain): with `pflag` the kernel may start while the dataflow
// POTRF of L is still running.  pflag is that kernel's per-64-block progress
// array (prog[ib * pNb + jb] == jb + 1 once block (ib, jb) of L is final and
// stored, published with st.release.gpu): the TMA producer acquires block
// (jb, pb) before loading it (then a generic -> async proxy fence), the MMA
// warps acquire the diagonal block before staging it.  Column block jb of X
// therefore follows row block jb of L by one solve.  Without pflag the inputs
// are complete at launch (ordinary stream / graph dependency).
//
// Hand-off by named barriers: READY (MMA arrive -> solver sync) when X[:,jb]
// holds its updated right-hand side, SOLVED (solver arrive -> MMA sync) when it
// holds the solution.  Every sum has a fixed order (k-steps split mod 3
// between the MMA k-groups, combined in a fixed order), so results are
// bit-identical run to run; the quotient is the correctly rounded a / L_cc
// (div_by: one IEEE reciprocal per column + Markstein correction), so
// unit-diagonal dyadic inputs stay exact (pin P2).
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>

#include "ptx.cuh"
#include "solve_block.cuh"
#include "tile_ops.hpp"

namespace stfk {

// debug timeline (CTA 0): trace[5 jb + e] = %globaltimer at event e of column block jb
__device__ __forceinline__ void tr_stamp(unsigned long long* trace, int idx) {
  if (trace && blockIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    trace[idx] = t;
  }
}

namespace tr {
using sb::xo;
using sb::poff;
constexpr int R = kTrsmResRows;  // rows per CTA (one 128-byte line per column of the panel)
constexpr int W = 64;        // column block
constexpr int NMAX = 1024;   // resident panel limit (NMAX * 128 B = 128 KB)
constexpr int BK = 32;       // k of L per pipeline stage
constexpr int NST = 4;       // L ring slots
constexpr int BOXD = 16 * BK;          // doubles per TMA box [BK k-rows][16 c] (4 KB)
constexpr int STAGE = (W / 16) * BOXD; // doubles per stage (16 KB)
constexpr int DP = 2080;     // packed lower diagonal block: 64 * 65 / 2
constexpr int NT = 256;      // 8 warps; warp w runs on SM sub-partition w % 4
constexpr int NMMA = 6;      // MMA warps 0,1,2,4,5,6 (sub-partitions 0-2)
constexpr int MMA_THREADS = NMMA * 32, SOLVE_THREADS = 32;  // solver warp 3, producer warp 7 (sub-partition 3)
constexpr int BAR_MMA = 1, BAR_READY = 2, BAR_SOLVED = 3;
__host__ __device__ constexpr size_t smem_bytes(int n) {
  return 1024 + ((size_t)16 * n + (size_t)NST * STAGE + 2 * DP + 2 * W) * sizeof(double) + 2 * NST * 8;
}
// L stage element (k, c) written by TMA boxes of [BK][16 c] with the 128B swizzle
__device__ __forceinline__ int lo(int k, int c) {
  return (c >> 4) * BOXD + k * 16 + (((((c & 15) >> 1) ^ (k & 7)) << 1) | (c & 1));
}
// first stage of step jb (steps consume 2 jb stages each)
__host__ __device__ constexpr int step_q0(int jb) { return jb * (jb - 1); }
}  // namespace tr

__device__ __forceinline__ void bar_sync_n(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }
__device__ __forceinline__ void bar_arrive_n(int id, int n) {
  asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(n) : "memory");
}
__device__ __forceinline__ void cpa8(void* smem, const void* gmem) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(smem)), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cpa_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cpa_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void wait_final(const int* p, int v) {  // acquire: L block published by the POTRF
  int x;
  for (;;) {
    asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(x) : "l"(p) : "memory");
    if (x >= v) break;
    __nanosleep(64);
  }
}
__device__ __forceinline__ double ld_cg_early(const double* p) {  // volatile: issued where written
  double v;
  asm volatile("ld.global.cg.f64 %0, [%1];" : "=d"(v) : "l"(p));
  return v;
}

// Warp roles are pinned to SM sub-partitions (warp w runs on w % 4): the FP64 pipe
// is shared by DMMA and DFMA, and a substitution chain sharing a sub-partition
// with DMMA-saturating warps slows from 7 to 24-137 clocks per dependent op
// (tools/dmma_latency.cu), so the solver warp and the TMA producer warp get
// sub-partition 3 and the six MMA warps use the other three.
//
// MMA work split: k-group kg = q mod 3 owns pipeline stage q (32 k of one column
// block's update), n-half nh the 32 columns; the two warps of a k-group read a
// stage and release it to the producer (mbarrier), the three k-group partial sums
// are combined in a fixed order at the end of the step.
__global__ void __launch_bounds__(tr::NT, 1) trsm_res_kernel(const __grid_constant__ CUtensorMap tmL, const double* __restrict__ L,
                                                              int64_t ldl, int n, double* __restrict__ X, int64_t ldx,
                                                              int M, const Mirrors mir, unsigned long long* trace, int dbg,
                                                              const int* pflag, int pNb, int* kflag, int trig) {
  using namespace tr;
  extern __shared__ __align__(1024) uint8_t smraw[];
  double* sm = reinterpret_cast<double*>(smraw + ((1024u - (smem_u32(smraw) & 1023u)) & 1023u));
  double* Ls = sm;                      // NST x STAGE (1024-byte aligned boxes)
  double* Xs = Ls + NST * STAGE;        // panel, xo(r, c)
  double* Ld = Xs + 16 * n;             // 2 x packed diagonal blocks
  double* Rc = Ld + 2 * DP;             // 2 x 64: 1 / L_cc (IEEE) of the two diagonal blocks
  uint64_t* full = reinterpret_cast<uint64_t*>(Rc + 2 * W);  // NST: stage landed
  uint64_t* empty = full + NST;                           // NST: stage released by its 2 readers
  const int r0 = blockIdx.x * R;
  const int rows = min(R, M - r0);
  const int Nb = n / W;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int total = step_q0(Nb);  // L stages over all steps

  if (threadIdx.x == 0) {
    tma_prefetch_desc(&tmL);
    for (int s = 0; s < NST; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 2);
    }
    fence_barrier_init();
  }
  __syncthreads();

  if (warp == 7) {
    // ------------------------------------------------------------ TMA producer
    if (lane == 0 && !(dbg & 4)) {
      int jb = 1, pb = 0, h = 0;
      for (int q = 0; q < total; ++q) {
        const int s = q % NST;
        if (q >= NST) mbar_wait(&empty[s], (q / NST - 1) & 1);
        if (pflag && h == 0) {  // block (jb, pb) of L final
          wait_final(pflag + jb * pNb + pb, pb + 1);
          asm volatile("fence.proxy.async.global;" ::: "memory");
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_arrive_expect_tx(&full[s], STAGE * 8);
#pragma unroll
        for (int b = 0; b < W / 16; ++b)
          tma_load_2d(Ls + s * STAGE + b * BOXD, &tmL, jb * W + 16 * b, pb * W + h * BK, &full[s]);
        if (++h == 2) {
          h = 0;
          if (++pb == jb) {
            pb = 0;
            ++jb;
          }
        }
      }
    }
  } else if (warp != 3) {
    // ------------------------------------------------------------ MMA warps
    const int mw = warp < 4 ? warp : warp - 1;  // 0..5
    const int g = lane >> 2, t = lane & 3, nh = mw & 1, kg = mw >> 1;
    for (int jb = 0; jb < Nb; ++jb) {
      const int c0 = jb * W;
      if (threadIdx.x == 0) tr_stamp(trace, 5 * jb + 0);
      {  // packed lower triangle of L(jb, jb) for the solver (its buffer jb & 1 was freed by solve(jb-2))
        double* dst = Ld + (jb & 1) * DP;
        const double* src = L + (int64_t)c0 * ldl + c0;
        const int tm = mw * 32 + lane;  // 0..191
        if (pflag) wait_final(pflag + jb * pNb + jb, jb + 1);  // L(jb, jb) final
        for (int idx = tm; idx < W * W; idx += MMA_THREADS) {
          const int rr = idx & (W - 1), cc = idx >> 6;
          if (rr >= cc) cpa8(dst + sb::poff(rr, cc), src + (int64_t)cc * ldl + rr);
        }
        cpa_commit();
      }
      double init[2][4][2];
      if (kg == 0) {
#pragma unroll
        for (int mi = 0; mi < 2; ++mi)
#pragma unroll
          for (int nj = 0; nj < 4; ++nj)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              const int row = 8 * mi + g, col = c0 + 32 * nh + 8 * nj + 2 * t + h;
              init[mi][nj][h] = row < rows ? ld_cg_early(X + (int64_t)col * ldx + r0 + row) : 0.0;
            }
      }
      double acc[2][4][2];
#pragma unroll
      for (int mi = 0; mi < 2; ++mi)
#pragma unroll
        for (int nj = 0; nj < 4; ++nj) acc[mi][nj][0] = acc[mi][nj][1] = 0.0;
      const int q0 = step_q0(jb);
      auto mma_grp = [&](const double* Lq, int kx, int grp) {  // one 8-wide k group of a stage
        if (dbg & 2) return;
#pragma unroll
        for (int kh = 0; kh < 2; ++kh) {
          const int k = 8 * grp + 2 * t + kh;
          double a[2], b[4];
#pragma unroll
          for (int mi = 0; mi < 2; ++mi) a[mi] = Xs[xo(8 * mi + g, kx + k)];
#pragma unroll
          for (int nj = 0; nj < 4; ++nj) b[nj] = Lq[lo(k, 32 * nh + 8 * nj + g)];
#pragma unroll
          for (int mi = 0; mi < 2; ++mi)
#pragma unroll
            for (int nj = 0; nj < 4; ++nj) dmma_8x8x4(acc[mi][nj][0], acc[mi][nj][1], a[mi], b[nj]);
        }
      };
      // phase A: terms of the solved blocks pb < jb - 1, stage q to k-group q mod 3
      for (int qi = 0; qi < 2 * jb - 2; ++qi) {
        const int q = q0 + qi;
        if (q % 3 != kg) continue;
        const int s = q % NST;
        if (!(dbg & 4)) mbar_wait(&full[s], (q / NST) & 1);
#pragma unroll
        for (int grp = 0; grp < BK / 8; ++grp) mma_grp(Ls + s * STAGE, qi * BK, grp);
        __syncwarp();  // this warp's reads of stage s fed its DMMAs
        if (lane == 0) mbar_arrive(&empty[s]);
      }
      // phase B: the terms of block jb-1 need its solution; its two stages are
      // shared by all six warps (k groups split mod 3) to shorten the critical path
      if (jb > 0) {
        if (threadIdx.x == 0) tr_stamp(trace, 5 * jb + 1);
        bar_sync_n(BAR_SOLVED, MMA_THREADS + SOLVE_THREADS);
        if (threadIdx.x == 0) tr_stamp(trace, 5 * jb + 2);
#pragma unroll
        for (int hb = 0; hb < 2; ++hb) {
          const int qi = 2 * jb - 2 + hb, q = q0 + qi, s = q % NST;
          if (!(dbg & 4)) mbar_wait(&full[s], (q / NST) & 1);
#pragma unroll
          for (int grp = 0; grp < BK / 8; ++grp)
            if ((4 * hb + grp) % 3 == kg) mma_grp(Ls + s * STAGE, qi * BK, grp);
        }
      }
      // X[:, jb] = (B - acc_0) - (acc_1 + acc_2)  (fixed order)
      if (kg == 2) {
#pragma unroll
        for (int mi = 0; mi < 2; ++mi)
#pragma unroll
          for (int nj = 0; nj < 4; ++nj)
#pragma unroll
            for (int h = 0; h < 2; ++h) Xs[xo(8 * mi + g, c0 + 32 * nh + 8 * nj + 2 * t + h)] = acc[mi][nj][h];
      }
      bar_sync_n(BAR_MMA, MMA_THREADS);  // also: every warp is done with the phase-B stages
      if (jb > 0 && lane == 0)
        for (int hb = 0; hb < 2; ++hb) {
          const int q = q0 + 2 * jb - 2 + hb;
          if (q % 3 == kg) mbar_arrive(&empty[q % NST]);
        }
      if (kg == 1) {
#pragma unroll
        for (int mi = 0; mi < 2; ++mi)
#pragma unroll
          for (int nj = 0; nj < 4; ++nj)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              double* p = Xs + xo(8 * mi + g, c0 + 32 * nh + 8 * nj + 2 * t + h);
              *p = acc[mi][nj][h] + *p;
            }
      }
      bar_sync_n(BAR_MMA, MMA_THREADS);
      if (kg == 0) {
#pragma unroll
        for (int mi = 0; mi < 2; ++mi)
#pragma unroll
          for (int nj = 0; nj < 4; ++nj)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              double* p = Xs + xo(8 * mi + g, c0 + 32 * nh + 8 * nj + 2 * t + h);
              *p = (init[mi][nj][h] - acc[mi][nj][h]) - *p;
            }
      }
      cpa_wait<0>();  // this thread's part of the diagonal block landed (visible to the solver
                      // through the READY barrier below)
      if (threadIdx.x == 0) tr_stamp(trace, 5 * jb + 3);
      bar_arrive_n(BAR_READY, MMA_THREADS + SOLVE_THREADS);
    }
  } else {
    // ------------------------------------------------------------ solver warp
    // solve_block: 8-column sub-blocks by substitution, their updates on DMMA; the
    // diagonal block and its pivots' reciprocals were staged by the MMA warps
    const int r = lane & 15;
    const bool wr = lane < 16 && r < rows;
    for (int jb = 0; jb < Nb; ++jb) {
      const int c0 = jb * W;
      const double* D = Ld + (jb & 1) * DP;
      const double* Y = Rc + (jb & 1) * W;
      const bool more = jb + 1 < Nb;
      bar_sync_n(BAR_READY, MMA_THREADS + SOLVE_THREADS);  // X[:, jb] updated; L(jb,jb) staged
      {  // IEEE reciprocals of the 64 pivots (two per lane)
        double* Yw = Rc + (jb & 1) * W;
        const double d0 = D[sb::poff(lane, lane)], d1 = D[sb::poff(lane + 32, lane + 32)];
        Yw[lane] = 1.0 / d0;
        Yw[lane + 32] = 1.0 / d1;
        __syncwarp();
      }
      if (lane == 0) tr_stamp(trace, 5 * jb + 4);
      solve_block<0>(Xs, c0, sb::Packed{D}, Y, lane, X, ldx, r0 + r, wr);
      if (mir.n > 0 && wr) {  // fused push (NEXT-3): the finished block into the consumers' replicas
#pragma unroll 1
        for (int m = 0; m < mir.n && m < 7; ++m) {
          double* dst = mir.p[m];
#pragma unroll 8
          for (int j = 0; j < W; ++j) mirror_st(dst + (int64_t)(c0 + j) * ldx + r0 + r, Xs[xo(r, c0 + j)], mir.mc);
        }
        mirror_fence(mir.mc);
      }
      if (kflag) {  // this CTA's rows of column block jb are stored: count them for the SYRK
        __threadfence();
        __syncwarp();
        if (lane == 0) atomicAdd(kflag + jb, 1);
      }
      if (jb == trig) griddep_launch_dependents();  // the dependent SYRK(k+1,k) may start
      __syncwarp();
      if (lane == 0) tr_stamp(trace, 5 * Nb + jb);  // solve end
      if (more) bar_arrive_n(BAR_SOLVED, MMA_THREADS + SOLVE_THREADS);
    }
  }
}

bool make_operand_map(CUtensorMap* tm, const double* ptr, int rows, int cols, int64_t ld, int bk);

// Resident-panel TRSM in `parts` (1, 2 or 4) column parts, right-looking: for each
// part p, X_p = B_p L_pp^-T, then B_{>p} -= X_p L_{>p,p}^T (one GEMM on 64 x 64 CTA
// tiles: the whole GPU).  The substitution runs on narrower panels and the
// off-diagonal flops at GEMM rate: the critical TRSM(k+1,k) at nb = 1024 spreads
// beyond the 64 CTAs of one resident-panel launch.
cudaError_t trsm_res_parts(cudaStream_t stream, int prio, int M, int n, const double* L, int64_t ldl, double* B,
                           int64_t ldb, const Mirrors* mirrors, int parts) {
  if (parts < 2 || n % (64 * parts) || (ldb & 1) || (reinterpret_cast<uintptr_t>(B) & 15) ||
      !trsm_res_supported(n / parts, L, ldl))
    return trsm_res(stream, prio, M, n, L, ldl, B, ldb, mirrors);
  const int w = n / parts;
  for (int p = 0; p < parts; ++p) {
    const int64_t c0 = (int64_t)p * w;
    Mirrors mp{};
    if (mirrors) {
      mp = *mirrors;
      for (int m = 0; m < mp.n && m < 7; ++m) mp.p[m] = mirrors->p[m] + c0 * ldb;
    }
    cudaError_t e = trsm_res(stream, prio, M, w, L + c0 * ldl + c0, ldl, B + c0 * ldb, ldb, &mp);
    if (e == cudaSuccess && p + 1 < parts)
      e = gemm_nt_tiles(stream, prio, M, n - (int)c0 - w, w, B + c0 * ldb, ldb, L + c0 * ldl + c0 + w, ldl,
                        B + (c0 + w) * ldb, ldb, 0, 1);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

bool trsm_res_supported(int n, const double* L, int64_t ldl) {
  return n >= tr::W && n <= tr::NMAX && n % tr::W == 0 && (ldl & 1) == 0 &&
         (reinterpret_cast<uintptr_t>(L) & 15) == 0;
}

cudaError_t trsm_res_init_attrs() {
  return cudaFuncSetAttribute(trsm_res_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              (int)tr::smem_bytes(tr::NMAX));
}

cudaError_t trsm_res(cudaStream_t stream, int prio, int M, int n, const double* L, int64_t ldl, double* B,
                     int64_t ldb, const Mirrors* mirrors, unsigned long long* trace, const int* pflag, int pNb,
                     int* kflag, int trig) {
  Mirrors mir{};
  if (mirrors) mir = *mirrors;
  if (M <= 0 || n <= 0) return cudaSuccess;
  if (!trsm_res_supported(n, L, ldl)) return cudaErrorInvalidValue;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((M + tr::R - 1) / tr::R);
  cfg.blockDim = dim3(tr::NT);
  cfg.dynamicSmemBytes = tr::smem_bytes(n);
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = prio;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  ++launch_count();
  CUtensorMap tmL;  // L as an n x n column-major operand: rows = c (contiguous), cols = k
  if (!make_operand_map(&tmL, L, n, n, ldl, tr::BK)) return cudaErrorInvalidValue;
  static int dbg = [] {
    const char* e = getenv("STF_TRSM_DBG");
    return e ? atoi(e) : 0;
  }();
  return cudaLaunchKernelEx(&cfg, trsm_res_kernel, tmL, L, ldl, n, B, ldb, M, mir, trace, dbg, pflag, pNb, kflag, trig);
}

}  // namespace stfk
