// K3 TRSM and K4 POTRF of one tile as single-launch, device-side dataflow
// kernels (the STF idea of PAPER.md:144 applied inside a
// tile: block tasks run as soon as the blocks they read are final).
//
// Task definitions (right-looking tiled Cholesky of [17]):
//   POTRF on an n x n tile, 64 x 64 blocks (ib, jb), ib >= jb:
//     P(kb)        X_kk <- chol(X_kk)                         (block Cholesky, in smem)
//     S(ib,kb)     X_ik <- X_ik X_kk^-T                      (substitution, in smem)
//     U(ib,jb,kb)  X_ij <- X_ij - X_ik X_jk^T                (DMMA, lower part only if ib == jb)
//   TRSM X[m x n] <- X L^-T, L n x n lower:
//     S(ib,jb)     X_ij <- X_ij L_jj^-T
//     U(ib,jb,pb)  X_ij <- X_ij - X_ip L_jp^T   (pb < jb)
//
// Scheduling: the host writes the task list once per block-grid shape, in a
// topological order with a look-ahead of one column (the next panel's column
// is updated first).  Every CTA repeatedly takes the next ticket from an atomic
// counter, waits (acquire) until the progress counters of the blocks the task
// reads have reached the required values, runs the task, and publishes
// (release) the new progress of the block it wrote.  A CTA only ever waits for
// tasks with smaller tickets, which were claimed by CTAs that are already
// running, so the scheme cannot deadlock whatever the grid size or how many
// CTAs are co-resident.  Progress of block (ib,jb) = number of operations
// completed on it; it is final when progress == jb + 1.
//
// Operations on every block happen in a fixed order (updates by increasing k,
// then the final P/S), so results are bit-identical run to run.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <climits>
#include <cstdint>
#include <map>
#include <mutex>
#include <tuple>
#include <vector>

#include "ptx.cuh"
#include "solve_block.cuh"
#include "tile_ops.hpp"

namespace stfk {

namespace df {
constexpr int W = 64;       // block order
constexpr int LDO = 68;     // smem stride of DMMA operand blocks [k][row] (68 = 4 mod 16: conflict-free)
constexpr int LDB = 65;     // smem stride of substitution / Cholesky blocks [row][col]
constexpr int NT = 256;
// critical CTA: D [W][LDB] + XS [W][LDO] + Rc [W] + 4 swizzled 16-row panels + 4 x Y [W] + a counter
constexpr int SMEM_BYTES = (W * LDB + W * LDO + W + 4 * 16 * W + 4 * W) * 8 + 16;  // 104,720 B
// bulk_kernel: the largest block task (U operands; S panels + L block; ragged S)
constexpr int cmax(int a, int b) { return a > b ? a : b; }
constexpr int BULK_SMEM_BYTES = cmax(2 * W * LDO, cmax(4 * 16 * W + W * LDB + W, 2 * W * LDB + W)) * 8 + 16;  // 69,648 B
enum : uint32_t { T_P = 0, T_S = 1, T_U = 2 };

__host__ __device__ inline uint32_t enc(uint32_t t, uint32_t i, uint32_t j, uint32_t k) {
  return (t << 30) | (i << 20) | (j << 10) | k;
}
}  // namespace df

struct DfParams {
  double* X;
  int64_t ldx;
  const double* L;  // TRSM: the triangular factor; POTRF: unused (X itself)
  int64_t ldl;
  int m, n;    // X is m x n
  int Mb, Nb;  // block grid of X
  const uint32_t* tasks;
  int ntasks;
  int* ws;  // ws[0] ticket, ws[1] critical-chain role, ws[2 + ib * Nb + jb] progress
  int64_t col0;
  unsigned long long* info;
  int potrf;
  int crit;  // POTRF: one CTA runs the critical chain P -> S -> U -> P (blocks kept in smem)
  unsigned long long* trace;  // debug: %globaltimer stamps (null in production)
  Mirrors mir;                // POTRF: replicas of the tile, written with every final block (fused push)
  int trig;  // programmatic dependent launch: the chain CTA triggers at step `trig`, the others at their
             // start (-1: no trigger, dependents launch at completion)
};

__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define DF_STAMP(idx)                                          \
  do {                                                         \
    if (p.trace && threadIdx.x == 0) p.trace[(idx)] = gtime(); \
  } while (0)

__device__ __forceinline__ int ld_acquire(const int* p) {
  int v;
  asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(int* p, int v) {
  asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void wait_geq(const int* p, int v) {
  int ns = 32;
  while (ld_acquire(p) < v) {
    __nanosleep(ns);
    if (ns < 256) ns <<= 1;
  }
}

// Block loads: all W*W/NT = 16 loads of a thread are issued before any store, so
// the L2 latency is paid once per block, not once per element row (a loop that
// alternates load and smem store serialises them: 6.8 -> ~3 us per U task).
constexpr int kPerThread = df::W * df::W / df::NT;
// smem S[c * ld + r] = G(r0 + r, c0 + c) for r < rows, c < cols; zero elsewhere (W x W)
__device__ __forceinline__ void load_block_cm(double* S, int ld, const double* G, int64_t ldg, int rows, int cols) {
  double v[kPerThread];
#pragma unroll
  for (int u = 0; u < kPerThread; ++u) {
    const int idx = threadIdx.x + u * df::NT, r = idx & (df::W - 1), c = idx >> 6;
    v[u] = (r < rows && c < cols) ? __ldcg(G + (int64_t)c * ldg + r) : 0.0;
  }
#pragma unroll
  for (int u = 0; u < kPerThread; ++u) {
    const int idx = threadIdx.x + u * df::NT, r = idx & (df::W - 1), c = idx >> 6;
    S[c * ld + r] = v[u];
  }
}
// smem S[r * ld + c] = G(r, c)  (row-major in smem)
__device__ __forceinline__ void load_block_rm(double* S, int ld, const double* G, int64_t ldg, int rows, int cols,
                                              bool lower_only) {
  double v[kPerThread];
#pragma unroll
  for (int u = 0; u < kPerThread; ++u) {
    const int idx = threadIdx.x + u * df::NT, r = idx & (df::W - 1), c = idx >> 6;
    v[u] = (r < rows && c < cols && (!lower_only || r >= c)) ? __ldcg(G + (int64_t)c * ldg + r) : 0.0;
  }
#pragma unroll
  for (int u = 0; u < kPerThread; ++u) {
    const int idx = threadIdx.x + u * df::NT, r = idx & (df::W - 1), c = idx >> 6;
    S[r * ld + c] = v[u];
  }
}
__device__ __forceinline__ void store_block_rm(const double* S, int ld, double* G, int64_t ldg, int rows, int cols,
                                               bool lower_only) {
  for (int idx = threadIdx.x; idx < df::W * df::W; idx += df::NT) {
    const int r = idx & (df::W - 1), c = idx >> 6;
    if (r < rows && c < cols && (!lower_only || r >= c)) G[(int64_t)c * ldg + r] = S[r * ld + c];
  }
}

// mirror (fused push) forms of the stores below: plain or multimem stores
__device__ __forceinline__ void mirror_block_rm(const double* S, int ld, double* G, int64_t ldg, int rows, int cols,
                                                bool lower_only, int mc) {
  for (int idx = threadIdx.x; idx < df::W * df::W; idx += df::NT) {
    const int r = idx & (df::W - 1), c = idx >> 6;
    if (r < rows && c < cols && (!lower_only || r >= c)) mirror_st(G + (int64_t)c * ldg + r, S[r * ld + c], mc);
  }
  mirror_fence(mc);
}

__device__ __forceinline__ double negd(double x) {
  return __longlong_as_double(__double_as_longlong(x) ^ (long long)0x8000000000000000ULL);
}

// U: C[rows x cols] -= A[rows x K] * B[cols x K]^T, K <= 64; lower: keep r >= c only
__device__ void task_update(double* sm, double* C, int64_t ldc, const double* A, int64_t lda, const double* B,
                            int64_t ldb, int rows, int cols, int K, bool lower) {
  double* As = sm;
  double* Bs = sm + df::W * df::LDO;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int wm0 = (warp & 1) * 32, wn0 = (warp >> 1) * 16;
  double acc[4][2][2];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 2; ++j)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int r = wm0 + 8 * i + g, c = wn0 + 8 * j + 2 * t + h;
        acc[i][j][h] = (r < rows && c < cols && (!lower || r >= c)) ? __ldcg(C + (int64_t)c * ldc + r) : 0.0;
      }
  load_block_cm(As, df::LDO, A, lda, rows, K);   // As[k][r]
  load_block_cm(Bs, df::LDO, B, ldb, cols, K);   // Bs[k][c]
  __syncthreads();
#pragma unroll 4
  for (int k0 = 0; k0 < df::W; k0 += 4) {
    double a[4], b[2];
#pragma unroll
    for (int i = 0; i < 4; ++i) a[i] = As[(k0 + t) * df::LDO + wm0 + 8 * i + g];
#pragma unroll
    for (int j = 0; j < 2; ++j) b[j] = negd(Bs[(k0 + t) * df::LDO + wn0 + 8 * j + g]);
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 2; ++j) dmma_8x8x4(acc[i][j][0], acc[i][j][1], a[i], b[j]);
  }
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 2; ++j)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int r = wm0 + 8 * i + g, c = wn0 + 8 * j + 2 * t + h;
        if (r < rows && c < cols && (!lower || r >= c)) C[(int64_t)c * ldc + r] = acc[i][j][h];
      }
}


// Substitution core.  Thread (r = tid & 63, q = tid >> 6) holds X[r, 16q .. 16q+15]
// in b[].  Ls[c * LDB + p] = L(c, p) (lower part read only).  Chunk q solves its
// 16 columns (correctly rounded divisions via div_by), publishes them to
// Xpub[r * ldp + col], later chunks subtract x L^T; every element accumulates
// its terms in increasing column order.  On return b[] holds the solution and
// Xpub all of it.
__device__ __forceinline__ void solve_core(double (&b)[16], const double* Ls, double* Rc, double* Xpub, int ldp,
                                           int nc) {
  const int r = threadIdx.x & (df::W - 1), q = threadIdx.x >> 6;
  if (threadIdx.x < nc) Rc[threadIdx.x] = 1.0 / Ls[threadIdx.x * df::LDB + threadIdx.x];
  __syncthreads();
  for (int qq = 0; qq < 4 && 16 * qq < nc; ++qq) {
    if (q == qq) {
#pragma unroll
      for (int c = 0; c < 16; ++c) {
        const int col = 16 * qq + c;
        if (col < nc) {
          b[c] = div_by(b[c], Ls[col * df::LDB + col], Rc[col]);
#pragma unroll
          for (int c2 = c + 1; c2 < 16; ++c2) b[c2] = fma(-b[c], Ls[(16 * qq + c2) * df::LDB + col], b[c2]);
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
          b[cc] = fma(-Xpub[r * ldp + 16 * qq + c], Ls[(16 * q + cc) * df::LDB + 16 * qq + c], b[cc]);
    }
  }
}

// Cholesky core of an nc x nc block (nc <= 64), latency-optimised for the
// critical chain (tools/chol_lab.cu, bit-identical to the quarter-serial form).  Thread (r = tid & 63,
// q = tid >> 6) holds A[r, 4m + q] in a[m] (interleaved columns, so all 256
// threads share every column's update).  Column j+1 needs ONE barrier:
//   * every owner thread of column j+1 (q == (j+1) & 3, two warps) recomputes
//     the pivot itself: d = a_{j+1,j+1} - L_{j+1,j}^2 from the published
//     diagonal Dp[j+1] and L_{j+1,j}, s = sqrt(d), y = 1/s (IEEE), then divides
//     its own element, L_{r,j+1} = div_by(a_{r,j+1} - L_rj L_{j+1,j}, s, y),
//     and publishes it in Lc[(j+1) % 3];
//   * the other threads apply column j's update to their elements; the owners'
//     own updates from column j are deferred to the next iteration (their
//     columns are >= j+5, not needed before then), so the owner warps run the
//     pivot chain alone.
// Every element still receives its updates in increasing column order with the
// same fma(-L_rk, L_ck, a) as the unblocked algorithm; sqrt and division are
// correctly rounded.  Rows above the diagonal and rows >= nc carry garbage that
// is never read or stored (no divergent branches in the loop).  Non-positive
// pivot (or NaN): info = min(info, col0 + col + 1), s = NaN.
// Scratch: Lc[3 * W], Dp[W + 2].  On return S[r * LDB + c] = L(r, c) for r >= c
// (after a __syncthreads); a[] is consumed.
__device__ __forceinline__ void chol_core(double (&a)[16], double* S, double* Lc, double* Dp, int nc, int64_t col0,
                                          unsigned long long* info) {
  constexpr int W = df::W;
  const int r = threadIdx.x & (W - 1), q = threadIdx.x >> 6;
  const double kNaN = __longlong_as_double(0x7ff8000000000000LL);
  if (q == 0 && r == 0) Dp[0] = a[0];
  if (q == 1 && r == 1) Dp[1] = a[0];
  __syncthreads();
  int bad = 0;  // 1-based column of this thread's failed pivot (row r is column r's pivot row)
  if (q == 0) {
    const double d = Dp[0];
    const bool ok = d > 0.0;
    bad = (!ok && r == 0) ? 1 : bad;
    const double s = ok ? sqrt(d) : kNaN, y = 1.0 / s;
    a[0] = (r == 0) ? s : div_by(a[0], s, y);
    Lc[r] = a[0];
  }
  __syncthreads();
  // Groups of 4 columns at run time; a[m] holds column 4(g + m) + q during group g
  // (the window shifts by one element per group, so register indices stay static).
  const int ng = (nc + 3) >> 2;
  for (int g = 0; g < ng; ++g) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int j = 4 * g + u, j1 = j + 1;
      if (j1 < nc) {  // uniform
        const int b = j % 3, bn = j1 % 3, bp = (j + 2) % 3;
        const int w1 = (u == 3) ? 1 : 0;  // window slot of column j+1 in quarter (u+1)&3
        const double lr = Lc[b * W + r];
        if (q == ((u + 1) & 3)) {  // warp-uniform: the owners of column j+1 run the pivot chain
          const double l1 = Lc[b * W + j1];
          const double d = fma(-l1, l1, Dp[j1]);
          const bool ok = d > 0.0;
          bad = (!ok && r == j1) ? j1 + 1 : bad;
          const double s = ok ? sqrt(d) : kNaN, y = 1.0 / s;
          const double v = div_by(fma(-lr, l1, a[w1]), s, y);
          a[w1] = (r == j1) ? s : v;
          Lc[bn * W + r] = a[w1];
        } else {
          if (j >= 1 && q == u) {  // deferred: this quarter's updates from column j-1 (columns > j)
            const double lp = Lc[bp * W + r];
            const double* Lp = Lc + bp * W + 4 * g + q;
#pragma unroll
            for (int m = 0; m < 16; ++m)
              if (4 * m + q > u) a[m] = fma(-lp, Lp[(4 * m) & 63], a[m]);
          }
          const double* Lb = Lc + b * W + 4 * g + q;
#pragma unroll
          for (int m = 0; m < 16; ++m) {
            if (4 * m + q > u + 1) {  // column 4(g+m)+q > j+1
              a[m] = fma(-lr, Lb[(4 * m) & 63], a[m]);
              if (4 * m + q == u + 2 && r == j + 2) Dp[j + 2] = a[m];
            }
          }
        }
      }
      __syncthreads();
    }
    // column 4g+q is final: publish it, shift the window
    {
      const int c = 4 * g + q;
      if (r >= c && r < nc && c < nc) S[r * df::LDB + c] = a[0];
    }
#pragma unroll
    for (int m = 0; m < 15; ++m) a[m] = a[m + 1];
    a[15] = 0.0;
  }
  if (bad) atomicMin(info, (unsigned long long)(col0 + bad));
  __syncthreads();
}

__device__ __forceinline__ void bar_sync_id(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }
__device__ __forceinline__ void bar_arrive_id(int id, int n) {
  asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(n) : "memory");
}

// progress flags in shared memory between warp groups of one CTA: release /
// acquire at CTA scope (the writer's data stores are ordered before the flag, the
// reader's data loads after it).  compute-sanitizer racecheck models barriers,
// not flag protocols: it reports the data handed over this way as hazards
// (profiles/r02/sanitize_racecheck.txt); shared-memory atomics instead of
// ld.acquire/st.release do not change that and cost 12 us per POTRF tile.
__device__ __forceinline__ int ld_volatile_s(const int* p) {
  int v;
  asm volatile("ld.acquire.cta.shared.b32 %0, [%1];" : "=r"(v) : "r"(smem_u32(p)) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_s(int* p, int v) {
  asm volatile("st.release.cta.shared.b32 [%0], %1;" ::"r"(smem_u32(p)), "r"(v) : "memory");
}

// P(kb) of the critical chain: the full 64 x 64 diagonal block held row-major in
// D (lower part, LDB stride), in place, by warps 0-3 (group D) while warps 4-7
// solve S(kb+1, kb) against the panels as they become final (critical_chain).
// 8 panels of 8 columns:
//   (a) warp 0 factors the panel: every lane factors the 8 x 8 diagonal block
//       redundantly in registers (no shuffles on the sqrt -> reciprocal -> divide
//       chain) and the two rows it owns below it (lane, lane + 32);
//   (b) warps 1-3 (the other SM sub-partitions) apply the panel to the trailing
//       lower block on DMMA (K = 8) with a look-ahead of one panel: the next
//       panel's columns first -- then they release warp 0 (named barrier NEXT) --
//       and the remaining columns while warp 0 already factors the next panel
//       (barrier DONE hands each finished panel to them).  Each 8 x 8 output tile
//       has one owner warp for the whole block (static map), so its updates stay
//       in increasing panel order.
// After panel p, *dpanel = p + 1 tells the S warps its columns are final.
// Correctly rounded sqrt and division (div_by with y = RN(1/s)); every element
// receives its updates in increasing column order, each a single fma or a DMMA
// k-step pair: the same operations as without look-ahead, deterministic.
// The pivot's sqrt and reciprocal are the library's (IEEE); a branch-free
// rsqrt-based form with the same bits (tools/check_rcp.cu: 0 mismatches in 5 x 2^32
// operands) shortens the chain in isolation (tools/p_lab.cu: P 11.2 -> 10.1 us) but
// made the POTRF tile slower in the factorisation kernel (354 -> 370 us, same box,
// profiles/r02/potrf_chain.txt), so it is not used.
__device__ void chol_block_grp(double* D, int64_t col0, unsigned long long* info, int* dpanel, double* Ypub = nullptr) {
  constexpr int LD = df::LDB, BAR_DONE = 1, BAR_NEXT = 2, GRP = 128;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const double kNaN = __longlong_as_double(0x7ff8000000000000LL);
  if (warp == 0) {
    int bad = 0;
    // one panel; the rows below it live in v1 (rows lane) and v2 (rows lane + 32).
    // (Instantiating it per panel range without the row streams that lie wholly above
    // the panel saves FP64 issue slots but made the tile 2% slower: the larger kernel
    // code; profiles/r02/potrf_chain.txt.)
    auto panel = [&](int p) {
      const int c0 = 8 * p;
      double dg[8][8], yp[8];
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j <= i; ++j) dg[i][j] = D[(c0 + i) * LD + c0 + j];
      const int r1 = lane, r2 = lane + 32;
      const bool b1 = r1 >= c0 + 8, b2 = r2 >= c0 + 8;
      double v1[8], v2[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        v1[j] = b1 ? D[r1 * LD + c0 + j] : 0.0;
        v2[j] = b2 ? D[r2 * LD + c0 + j] : 0.0;
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const double d = dg[i][i];
        const bool ok = d > 0.0;
        if (!ok && bad == 0) bad = c0 + i + 1;
        const double sq = ok ? sqrt(d) : kNaN, y = 1.0 / sq;
        dg[i][i] = sq;
        yp[i] = y;
#pragma unroll
        for (int r = i + 1; r < 8; ++r) dg[r][i] = div_by(dg[r][i], sq, y);
#pragma unroll
        for (int r = i + 1; r < 8; ++r)
#pragma unroll
          for (int c = i + 1; c <= r; ++c) dg[r][c] = fma(-dg[r][i], dg[c][i], dg[r][c]);
        v1[i] = div_by(v1[i], sq, y);
        v2[i] = div_by(v2[i], sq, y);
#pragma unroll
        for (int c = i + 1; c < 8; ++c) {
          v1[c] = fma(-v1[i], dg[c][i], v1[c]);
          v2[c] = fma(-v2[i], dg[c][i], v2[c]);
        }
      }
      __syncwarp();  // every lane has read the diagonal block before lane 0 overwrites it
      if (lane == 0) {
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int j = 0; j <= i; ++j) D[(c0 + i) * LD + c0 + j] = dg[i][j];
        if (Ypub)  // the pivots' reciprocals RN(1/L_cc) for the S warps' divisions
#pragma unroll
          for (int i = 0; i < 8; ++i) Ypub[c0 + i] = yp[i];
      }
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        if (b1) D[r1 * LD + c0 + j] = v1[j];
        if (b2) D[r2 * LD + c0 + j] = v2[j];
      }
    };
#pragma unroll 1
    for (int p = 0; p < 8; ++p) {
      if (p > 0) bar_sync_id(BAR_NEXT, GRP);
      panel(p);
      __syncwarp();
      if (lane == 0) st_release_s(dpanel, p + 1);  // panel p is final: the S warps may use it
      bar_arrive_id(BAR_DONE, GRP);
    }
    if (bad) atomicMin(info, (unsigned long long)(col0 + bad));
  } else {
    const int mw = warp - 1;  // 0..2
    auto update = [&](int R, int Cb, int c0) {
      double* rowp = D + (8 * R + g) * LD;
      double* cp = rowp + 8 * Cb + 2 * t;
      double acc0 = cp[0], acc1 = cp[1];
#pragma unroll
      for (int ks = 0; ks < 2; ++ks) {
        const double a = rowp[c0 + 4 * ks + t];
        const double b = negd(D[(8 * Cb + g) * LD + c0 + 4 * ks + t]);
        dmma_8x8x4(acc0, acc1, a, b);
      }
      cp[0] = acc0;
      cp[1] = acc1;
    };
#pragma unroll 1
    for (int p = 0; p < 7; ++p) {
      bar_sync_id(BAR_DONE, GRP);
      const int c0 = 8 * p;
      for (int R = p + 1; R < 8; ++R)
        if ((R + 2 * (p + 1)) % 3 == mw) update(R, p + 1, c0);
      bar_arrive_id(BAR_NEXT, GRP);
      for (int Cb = p + 2; Cb < 8; ++Cb)
        for (int R = Cb; R < 8; ++R)
          if ((R + 2 * Cb) % 3 == mw) update(R, Cb, c0);
    }
    bar_sync_id(BAR_DONE, GRP);  // panel 7
  }
  bar_sync_id(4, GRP);  // every write of the group to D is done
}

// interleaved-column register blocks (chol_core layout): v[m] = G(r, 4m + q)
__device__ __forceinline__ void load_il(double (&v)[16], const double* G, int64_t ldg, int rows, int nc, bool lower) {
  const int r = threadIdx.x & (df::W - 1), q = threadIdx.x >> 6;
#pragma unroll
  for (int m = 0; m < 16; ++m) {
    const int col = 4 * m + q;
    v[m] = (r < rows && col < nc && (!lower || r >= col)) ? __ldcg(G + (int64_t)col * ldg + r) : 0.0;
  }
}

__device__ __forceinline__ void load_chunk(double (&v)[16], const double* G, int64_t ldg, int rows, int nc,
                                           bool lower) {
  const int r = threadIdx.x & (df::W - 1), q = threadIdx.x >> 6;
#pragma unroll
  for (int c = 0; c < 16; ++c) {
    const int col = 16 * q + c;
    v[c] = (r < rows && col < nc && (!lower || r >= col)) ? __ldcg(G + (int64_t)col * ldg + r) : 0.0;
  }
}
__device__ __forceinline__ void store_chunk(const double (&v)[16], double* G, int64_t ldg, int rows, int nc,
                                            bool lower) {
  const int r = threadIdx.x & (df::W - 1), q = threadIdx.x >> 6;
  if (r < rows) {
#pragma unroll
    for (int c = 0; c < 16; ++c) {
      const int col = 16 * q + c;
      if (col < nc && (!lower || r >= col)) G[(int64_t)col * ldg + r] = v[c];
    }
  }
}

__device__ __forceinline__ void store_chunk_m(const double (&v)[16], double* G, int64_t ldg, int rows, int nc, int mc) {
  const int r = threadIdx.x & (df::W - 1), q = threadIdx.x >> 6;
  if (r < rows) {
#pragma unroll
    for (int c = 0; c < 16; ++c) {
      const int col = 16 * q + c;
      if (col < nc) mirror_st(G + (int64_t)col * ldg + r, v[c], mc);
    }
  }
  mirror_fence(mc);
}

// S task: X[rows x nc] <- X L^-T with L = the nc x nc diagonal block at L (global);
// the result also goes to the mirrors at element offset `off` (fused push).
__device__ void task_solve(double* sm, double* X, int64_t ldx, const double* L, int64_t ldl, int rows, int nc,
                           const Mirrors* mir = nullptr, int64_t off = 0) {
  if (nc == df::W) {
    // full block: four warps (one per SM sub-partition) solve 16 rows each with
    // solve_block (8-column sub-blocks by substitution, their updates on DMMA) --
    // the form the critical chain uses, 8.8 -> ~6 us per task
    constexpr int W = df::W;
    double* Xp = sm;                  // 4 x [16 x 64] swizzled panels
    double* D = Xp + 4 * 16 * W;      // L row-major [W][LDB], lower part
    double* Yc = D + W * df::LDB;     // 1 / L_cc (IEEE)
    {
      double v[kPerThread];
#pragma unroll
      for (int u = 0; u < kPerThread; ++u) {
        const int idx = threadIdx.x + u * df::NT, rr = idx & (W - 1), cc = idx >> 6;
        v[u] = rr < rows ? __ldcg(X + (int64_t)cc * ldx + rr) : 0.0;
      }
#pragma unroll
      for (int u = 0; u < kPerThread; ++u) {
        const int idx = threadIdx.x + u * df::NT, rr = idx & (W - 1), cc = idx >> 6;
        Xp[(rr >> 4) * 16 * W + sb::xo(rr & 15, cc)] = v[u];
      }
    }
    load_block_rm(D, df::LDB, L, ldl, W, W, true);
    __syncthreads();
    if (threadIdx.x < W) Yc[threadIdx.x] = 1.0 / D[threadIdx.x * df::LDB + threadIdx.x];
    __syncthreads();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (warp < 4) {
      const int rr = 16 * warp + (lane & 15);
      solve_block<0>(Xp + warp * 16 * W, 0, sb::RowMajor<df::LDB>{D}, Yc, lane, X, ldx, rr, lane < 16 && rr < rows);
    }
    if (mir && mir->n) {
      __syncthreads();
      for (int m = 0; m < mir->n; ++m) {
        for (int idx = threadIdx.x; idx < W * W; idx += df::NT) {
          const int rr = idx & (W - 1), cc = idx >> 6;
          if (rr < rows) mirror_st(mir->p[m] + off + (int64_t)cc * ldx + rr, Xp[(rr >> 4) * 16 * W + sb::xo(rr & 15, cc)], mir->mc);
        }
        mirror_fence(mir->mc);
      }
    }
    return;
  }
  double* Xs = sm;                    // publication buffer [r][LDB]
  double* Ls = sm + df::W * df::LDB;  // Ls[c][p]
  double* Rc = Ls + df::W * df::LDB;
  double b[16];
  load_chunk(b, X, ldx, rows, nc, false);
  load_block_rm(Ls, df::LDB, L, ldl, nc, nc, true);
  __syncthreads();
  solve_core(b, Ls, Rc, Xs, df::LDB, nc);
  store_chunk(b, X, ldx, rows, nc, false);
  if (mir)
    for (int m = 0; m < mir->n; ++m) store_chunk_m(b, mir->p[m] + off, ldx, rows, nc, mir->mc);
}

// P task: in-place lower Cholesky of the nc x nc diagonal block at X (global)
// (+ the mirrors at element offset `off`).
__device__ void task_chol(double* sm, double* X, int64_t ldx, int nc, int64_t col0, unsigned long long* info,
                          const Mirrors* mir = nullptr, int64_t off = 0) {
  double* S = sm;
  double* Lc = sm + df::W * df::LDB;
  double* Dp = Lc + 3 * df::W;
  double a[16];
  load_il(a, X, ldx, nc, nc, true);
  chol_core(a, S, Lc, Dp, nc, col0, info);
  store_block_rm(S, df::LDB, X, ldx, nc, nc, true);
  if (mir)
    for (int m = 0; m < mir->n; ++m) mirror_block_rm(S, df::LDB, mir->p[m] + off, ldx, nc, nc, true, mir->mc);
}

// The critical path of the tile Cholesky, run by ONE CTA with its blocks kept
// in shared memory: P(kb) -> S(kb+1, kb) -> U(kb+1, kb+1, kb) -> P(kb+1) -> ...
// (bulk CTAs run every other task).  Saves the global round trip, the flag
// hand-off and the block reloads between consecutive critical tasks.
__device__ void critical_chain(const DfParams& p, double* sm) {
  constexpr int W = df::W;
  const int T = p.Nb;
  double* D = sm;                          // [r][LDB]: P publication buffer -> L_kk
  double* XS = sm + W * df::LDB;           // [r][LDO]: X(kb+1, kb), A and B of U
  double* Rc = XS + W * df::LDO;           // W
  double* Lc = XS;                         // 3 W: chol_core scratch (XS is dead during P)
  double* Dp = XS + 3 * W;                 // W + 2
  double* Xp = Rc + W;                     // 4 x [16 x 64] swizzled panels of S(kb+1, kb)
  double* Yc = Xp + 4 * 16 * W;            // W: 1 / L_cc of L_kk, published by the P warp with each panel (4 W reserved)
  int* dpanel = reinterpret_cast<int*>(Yc + 4 * W);  // panels of P(kb) final so far
  int* prog = p.ws + 2;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int wm0 = (warp & 1) * 32, wn0 = (warp >> 1) * 16;
  const int r = threadIdx.x & (W - 1), q = threadIdx.x >> 6;
  double a[16];
  load_il(a, p.X, p.ldx, min(W, p.n), min(W, p.n), true);  // P(0) input: nothing precedes it
  for (int kb = 0; kb < T; ++kb) {
    if (kb == p.trig) griddep_launch_dependents();  // the dependent TRSM(k+1,k) may start (it polls prog[])
    const int nk = min(W, p.n - kb * W);
    double* Xkk = p.X + (int64_t)kb * W * p.ldx + kb * W;
    // ---- P(kb), and S(kb+1, kb) concurrently on the other four warps
    DF_STAMP(6 * kb + 0);
    const int ib = kb + 1, rows = ib < T ? min(W, p.n - ib * W) : 0;
    double* Xik = p.X + (int64_t)kb * W * p.ldx + ib * W;
    // fast U(ib, ib, kb) (full blocks): warps 0-3 own the 36 lower 8 x 8 tiles, warp w
    // the rows Ia = 7 - w (Ia + 1 tiles) and Ib = w (Ib + 1 tiles), 9 tiles each (one
    // SM sub-partition each: the DMMA pipe is split evenly); C is prefetched into the
    // accumulators right after P, the operands come straight from the S panels
    const bool fastU = nk == W && rows == W;
    const int Ia = 7 - (warp & 3), Ib = warp & 3;
    double uA[8][2], uB[4][2];
    if (nk == W) {
      if (kb == 0) load_block_rm(D, df::LDB, Xkk, p.ldx, W, W, true);  // P(0) input: nothing precedes it
      if (threadIdx.x == 0) *dpanel = 0;
      __syncthreads();
      if (warp < 4) {  // ---- group D: P(kb), then L_kk to global and published
        chol_block_grp(D, p.col0 + (int64_t)kb * W, p.info, dpanel, Yc);
        for (int idx = threadIdx.x; idx < W * W; idx += 128) {
          const int rr = idx & (W - 1), cc = idx >> 6;
          if (rr >= cc) Xkk[(int64_t)cc * p.ldx + rr] = D[rr * df::LDB + cc];
        }
        for (int m = 0; m < p.mir.n; ++m) {
          for (int idx = threadIdx.x; idx < W * W; idx += 128) {
            const int rr = idx & (W - 1), cc = idx >> 6;
            if (rr >= cc) mirror_st(p.mir.p[m] + (Xkk - p.X) + (int64_t)cc * p.ldx + rr, D[rr * df::LDB + cc], p.mir.mc);
          }
          mirror_fence(p.mir.mc);
        }
        bar_sync_id(4, 128);
        if (threadIdx.x == 0) {
          __threadfence();
          st_release(&prog[kb * p.Nb + kb], kb + 1);
        }
        DF_STAMP(6 * kb + 1);
        if (fastU) {  // C = block (ib, ib) after its earlier updates, into the U accumulators
          if (threadIdx.x == 0) wait_geq(&prog[ib * p.Nb + ib], kb);
          bar_sync_id(4, 128);
          const double* Cii = p.X + (int64_t)ib * W * p.ldx + ib * W;
#pragma unroll
          for (int J = 0; J < 8; ++J)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              const int rA = 8 * Ia + g, rB = 8 * Ib + g, c = 8 * J + 2 * t + h;
              uA[J][h] = (J <= Ia && rA >= c) ? __ldcg(Cii + (int64_t)c * p.ldx + rA) : 0.0;
              if (J < 4) uB[J][h] = (J <= Ib && rB >= c) ? __ldcg(Cii + (int64_t)c * p.ldx + rB) : 0.0;
            }
        }
      } else if (rows > 0) {  // ---- group S: X(kb+1, kb) <- X L_kk^-T, panel by panel as P finishes them
        const int tid = threadIdx.x - 128, sw = warp - 4;
        if (tid == 0) {
          wait_geq(&prog[ib * p.Nb + kb], kb);  // all updates U(kb+1, kb, k'), k' < kb, done
          if (p.trace) p.trace[6 * kb + 2] = gtime();
        }
        bar_sync_id(3, 128);
#pragma unroll 1
        for (int h = 0; h < 2; ++h) {  // 2 x 16 loads in flight per thread
          double v[16];
#pragma unroll
          for (int u = 0; u < 16; ++u) {
            const int idx = tid + (16 * h + u) * 128, rr = idx & (W - 1), cc = idx >> 6;
            v[u] = rr < rows ? __ldcg(Xik + (int64_t)cc * p.ldx + rr) : 0.0;
          }
#pragma unroll
          for (int u = 0; u < 16; ++u) {
            const int idx = tid + (16 * h + u) * 128, rr = idx & (W - 1), cc = idx >> 6;
            Xp[(rr >> 4) * 16 * W + sb::xo(rr & 15, cc)] = v[u];
          }
        }
        bar_sync_id(3, 128);
        // 1 / L_cc: published by the P warp with each panel (RN(1/L_cc), the value the
        // division by L_cc needs); sub-block P needs panel P of L_kk final
        auto gate = [&](int P) {
          while (ld_volatile_s(dpanel) <= P) __nanosleep(40);  // keep the issue slots for the P warps
          __threadfence_block();
        };
        const int rr = 16 * sw + (lane & 15);
        solve_block<0>(Xp + sw * 16 * W, 0, sb::RowMajor<df::LDB>{D}, Yc, lane, Xik, p.ldx, rr, lane < 16 && rr < rows,
                       gate);
        __syncwarp();
        for (int m = 0; m < p.mir.n; ++m) {  // fused push of the finished block
          if (lane < 16 && rr < rows)
            for (int c = 0; c < W; ++c)
              mirror_st(p.mir.p[m] + (Xik - p.X) + (int64_t)c * p.ldx + rr, Xp[sw * 16 * W + sb::xo(lane & 15, c)],
                        p.mir.mc);
          mirror_fence(p.mir.mc);
        }
        bar_sync_id(3, 128);
        if (tid == 0) {
          __threadfence();
          st_release(&prog[ib * p.Nb + kb], kb + 1);
          if (p.trace) p.trace[6 * kb + 3] = gtime();
        }
      }
      __syncthreads();
      if (kb + 1 == T) return;
      if (fastU) {
        // ---- U(ib, ib, kb): D <- lower(C - X X^T) on warps 0-3, X(m, k) from the S panels
        if (warp < 4) {
          DF_STAMP(6 * kb + 4);
          // X(m, k) = Xp[(m >> 4) 16 W + xo(m & 15, k)]: for the fragment rows m = 8 R + g and
          // k = k0 + t the offset is off[R][(k0 >> 2) & 1] + 16 k0 (the swizzle depends on k & 7)
          int off[8][2];
#pragma unroll
          for (int R = 0; R < 8; ++R)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              const int m = 8 * R + g;
              off[R][h] = (m >> 4) * 16 * W + sb::xo(m & 15, 4 * h + t) - 16 * 4 * h;
            }
          const int oA0 = Ia == 7 ? off[7][0] : Ia == 6 ? off[6][0] : Ia == 5 ? off[5][0] : off[4][0];
          const int oA1 = Ia == 7 ? off[7][1] : Ia == 6 ? off[6][1] : Ia == 5 ? off[5][1] : off[4][1];
          const int oB0 = Ib == 0 ? off[0][0] : Ib == 1 ? off[1][0] : Ib == 2 ? off[2][0] : off[3][0];
          const int oB1 = Ib == 0 ? off[0][1] : Ib == 1 ? off[1][1] : Ib == 2 ? off[2][1] : off[3][1];
#pragma unroll 2
          for (int k0 = 0; k0 < W; k0 += 4) {
            const int h = (k0 >> 2) & 1, kk = 16 * k0;
            const double aA = Xp[(h ? oA1 : oA0) + kk], aB = Xp[(h ? oB1 : oB0) + kk];
#pragma unroll
            for (int J = 0; J < 8; ++J) {
              if (J <= Ia) {  // warp-uniform
                const double b = negd(Xp[off[J][h] + kk]);
                dmma_8x8x4(uA[J][0], uA[J][1], aA, b);
                if (J < 4 && J <= Ib) dmma_8x8x4(uB[J][0], uB[J][1], aB, b);
              }
            }
          }
#pragma unroll
          for (int J = 0; J < 8; ++J)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              const int c = 8 * J + 2 * t + h;
              if (J <= Ia) D[(8 * Ia + g) * df::LDB + c] = uA[J][h];
              if (J < 4 && J <= Ib) D[(8 * Ib + g) * df::LDB + c] = uB[J][h];
            }
          DF_STAMP(6 * kb + 5);
        }
        continue;  // the next step's first __syncthreads orders D and Xp
      }
      for (int idx = threadIdx.x; idx < W * W; idx += df::NT) {  // X for U's operands
        const int m = idx >> 6, k = idx & (W - 1);
        XS[m * df::LDO + k] = Xp[(m >> 4) * 16 * W + sb::xo(m & 15, k)];
      }
      __syncthreads();
    } else {
      // ragged last block (n % 64 != 0): the register-resident Cholesky core
      chol_core(a, D, Lc, Dp, nk, p.col0 + (int64_t)kb * W, p.info);
      store_block_rm(D, df::LDB, Xkk, p.ldx, nk, nk, true);
      for (int m = 0; m < p.mir.n; ++m)
        mirror_block_rm(D, df::LDB, p.mir.p[m] + (Xkk - p.X), p.ldx, nk, nk, true, p.mir.mc);
      __syncthreads();
      if (threadIdx.x == 0) {
        __threadfence();
        st_release(&prog[kb * p.Nb + kb], kb + 1);
      }
      DF_STAMP(6 * kb + 1);
      return;  // a ragged block is the last one
    }
    // ---- U(ib, ib, kb): D <- lower(C - X X^T), C = block (ib, ib) after all earlier updates
    if (threadIdx.x == 0) wait_geq(&prog[ib * p.Nb + ib], kb);
    __syncthreads();
    DF_STAMP(6 * kb + 4);
    double* Cii = p.X + (int64_t)ib * W * p.ldx + ib * W;
    double acc[4][2][2];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 2; ++j)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int rr = wm0 + 8 * i + g, cc = wn0 + 8 * j + 2 * t + h;
          acc[i][j][h] = (rr < rows && cc < rows && rr >= cc) ? __ldcg(Cii + (int64_t)cc * p.ldx + rr) : 0.0;
        }
    // operands: A(m, k) = B(m, k) = X(m, k) = XS[m * LDO + k]; columns k >= nk are zero-padded below
    if (nk < W)
      for (int idx = threadIdx.x; idx < W * W; idx += df::NT) {
        const int m = idx >> 6, k = idx & (W - 1);
        if (k >= nk) XS[m * df::LDO + k] = 0.0;
      }
    __syncthreads();
#pragma unroll 4
    for (int k0 = 0; k0 < W; k0 += 4) {
      double av[4], bv[2];
#pragma unroll
      for (int i = 0; i < 4; ++i) av[i] = XS[(wm0 + 8 * i + g) * df::LDO + k0 + t];
#pragma unroll
      for (int j = 0; j < 2; ++j) bv[j] = negd(XS[(wn0 + 8 * j + g) * df::LDO + k0 + t]);
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 2; ++j) dmma_8x8x4(acc[i][j][0], acc[i][j][1], av[i], bv[j]);
    }
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 2; ++j)
#pragma unroll
        for (int h = 0; h < 2; ++h) D[(wm0 + 8 * i + g) * df::LDB + wn0 + 8 * j + 2 * t + h] = acc[i][j][h];
    __syncthreads();
#pragma unroll
    for (int m = 0; m < 16; ++m) {
      const int col = 4 * m + q;
      a[m] = (r < rows && col < rows && r >= col) ? D[r * df::LDB + col] : 0.0;
    }
    __syncthreads();  // D is rewritten by the next chol_core
    DF_STAMP(6 * kb + 5);
  }
}

// The ticket loop of the block tasks (see the header comment).  kBulk: the POTRF
// block tasks other than the critical chain's (S and U only; the launch that runs
// them next to the chain launch), compiled for 2 CTAs per SM.
template <bool kBulk>
__device__ __forceinline__ void ticket_loop(const DfParams& p, double* sm, int* s_task) {
  const int W = df::W;
  int* prog = p.ws + 2;
  bool triggered = false;
  for (;;) {
    if (threadIdx.x == 0) *s_task = atomicAdd(&p.ws[0], 1);
    __syncthreads();
    const int ticket = *s_task;
    if (ticket >= p.ntasks) return;
    if (kBulk && !triggered && p.trig >= 0 && ticket >= p.trig) {  // the dependent TRSM(k+1,k) may start
      griddep_launch_dependents();
      triggered = true;
    }
    DF_STAMP(6 * p.Nb + 3 * ticket + 0);
    const uint32_t code = p.tasks[ticket];
    const uint32_t type = code >> 30;
    const int ib = (code >> 20) & 1023, jb = (code >> 10) & 1023, kb = code & 1023;
    const int rows = min(W, p.m - ib * W);
    if (threadIdx.x == 0) {
      if (p.potrf) {
        if (!kBulk && type == df::T_P) {
          wait_geq(&prog[kb * p.Nb + kb], kb);
        } else if (type == df::T_S) {
          wait_geq(&prog[kb * p.Nb + kb], kb + 1);
          wait_geq(&prog[ib * p.Nb + kb], kb);
        } else {
          wait_geq(&prog[ib * p.Nb + kb], kb + 1);
          wait_geq(&prog[jb * p.Nb + kb], kb + 1);
          wait_geq(&prog[ib * p.Nb + jb], kb);
        }
      } else {
        if (type == df::T_S) {
          wait_geq(&prog[ib * p.Nb + jb], jb);
        } else {
          wait_geq(&prog[ib * p.Nb + kb], kb + 1);
          wait_geq(&prog[ib * p.Nb + jb], kb);
        }
      }
    }
    __syncthreads();
    DF_STAMP(6 * p.Nb + 3 * ticket + 1);
    if (kBulk || p.potrf) {
      double* Xkk = p.X + (int64_t)kb * W * p.ldx + kb * W;
      const int nk = min(W, p.n - kb * W);
      if (!kBulk && type == df::T_P) {
        task_chol(sm, Xkk, p.ldx, nk, p.col0 + (int64_t)kb * W, p.info, &p.mir, Xkk - p.X);
      } else if (type == df::T_S) {
        double* Xik = p.X + (int64_t)kb * W * p.ldx + ib * W;
        task_solve(sm, Xik, p.ldx, Xkk, p.ldx, rows, nk, &p.mir, Xik - p.X);
      } else {
        const int cols = min(W, p.n - jb * W);
        task_update(sm, p.X + (int64_t)jb * W * p.ldx + ib * W, p.ldx, p.X + (int64_t)kb * W * p.ldx + ib * W, p.ldx,
                    p.X + (int64_t)kb * W * p.ldx + jb * W, p.ldx, rows, cols, nk, ib == jb);
      }
    } else {
      if (type == df::T_S) {
        const int nc = min(W, p.n - jb * W);
        task_solve(sm, p.X + (int64_t)jb * W * p.ldx + ib * W, p.ldx, p.L + (int64_t)jb * W * p.ldl + jb * W, p.ldl,
                   rows, nc);
      } else {
        const int cols = min(W, p.n - jb * W), K = min(W, p.n - kb * W);
        task_update(sm, p.X + (int64_t)jb * W * p.ldx + ib * W, p.ldx, p.X + (int64_t)kb * W * p.ldx + ib * W, p.ldx,
                    p.L + (int64_t)kb * W * p.ldl + jb * W, p.ldl, rows, cols, K, false);
      }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      __threadfence();
      const int tgt = p.potrf ? (type == df::T_U ? ib * p.Nb + jb : ib * p.Nb + kb) : (ib * p.Nb + jb);
      st_release(&prog[tgt], kb + 1);
    }
    DF_STAMP(6 * p.Nb + 3 * ticket + 2);
  }
}

__global__ void __launch_bounds__(df::NT) dataflow_kernel(const DfParams p) {
  extern __shared__ __align__(16) double sm[];
  __shared__ int s_task;
  if (p.crit) {
    // the first CTA to start takes the critical chain (it is resident by construction)
    if (threadIdx.x == 0) s_task = (atomicCAS(&p.ws[1], 0, 1) == 0);
    __syncthreads();
    if (s_task) {
      critical_chain(p, sm);
      return;
    }
    __syncthreads();
  }
  if (p.trig >= 0) griddep_launch_dependents();
  ticket_loop<false>(p, sm, &s_task);
}

// POTRF as two launches: the critical chain plus a few block-task CTAs
// (dataflow_kernel: the register-heavy panel code, one CTA per SM) and most block
// tasks (bulk_kernel, 2 CTAs per SM with 70 KB of shared memory: they fit next to
// a GEMM CTA).  The first launch releases the second at its start (programmatic
// dependent launch) and both take tickets from one counter; the first can finish
// every task alone, so the tile completes even when the launches are serialised
// (profilers, sanitizers).  The bulk CTAs release the next dependent (TRSM(k+1,k))
// once the tickets reach p.trig.
__global__ void __launch_bounds__(df::NT, 2) bulk_kernel(const DfParams p) {
  extern __shared__ __align__(16) double sm[];
  __shared__ int s_task;
  ticket_loop<true>(p, sm, &s_task);
}

// ------------------------------------------------------------------ host side
namespace {

bool on_chain(uint32_t code) {  // P(kb), S(kb+1, kb), U(kb+1, kb+1, kb)
  const uint32_t type = code >> 30;
  const int ib = (code >> 20) & 1023, jb = (code >> 10) & 1023, kb = code & 1023;
  if (type == df::T_P) return true;
  if (type == df::T_S) return ib == kb + 1;
  return ib == kb + 1 && jb == kb + 1;
}

std::vector<uint32_t> build_tasks(bool potrf, int Mb, int Nb, bool crit) {
  std::vector<uint32_t> t;
  using df::enc;
  if (potrf && crit) {
    std::vector<uint32_t> all = build_tasks(true, Mb, Nb, false);
    for (uint32_t c : all)
      if (!on_chain(c)) t.push_back(c);
    return t;
  }
  if (potrf) {
    const int T = Nb;
    // look-ahead-1 topological order (see header comment)
    t.push_back(enc(df::T_P, 0, 0, 0));
    for (int i = 1; i < T; ++i) t.push_back(enc(df::T_S, i, 0, 0));
    for (int i = 1; i < T; ++i) t.push_back(enc(df::T_U, i, 1, 0));
    // per step: P(kb+1) and its solves; then the column kb+2 -- the next panel's
    // inputs -- first receives the update from column kb and then from column kb+1
    // (the look-ahead), ahead of the bulk updates of the columns behind it; every
    // block still sees its updates in increasing k, so a task only waits on
    // smaller tickets (deadlock-free)
    for (int kb = 0; kb + 1 < T; ++kb) {
      t.push_back(enc(df::T_P, kb + 1, kb + 1, kb + 1));
      for (int i = kb + 2; i < T; ++i) t.push_back(enc(df::T_S, i, kb + 1, kb + 1));
      if (kb + 2 < T) {
        for (int i = kb + 2; i < T; ++i) t.push_back(enc(df::T_U, i, kb + 2, kb));
        for (int i = kb + 2; i < T; ++i) t.push_back(enc(df::T_U, i, kb + 2, kb + 1));
      }
      for (int j = kb + 3; j < T; ++j)
        for (int i = j; i < T; ++i) t.push_back(enc(df::T_U, i, j, kb));
    }
  } else {
    for (int i = 0; i < Mb; ++i) t.push_back(enc(df::T_S, i, 0, 0));
    if (Nb > 1)
      for (int i = 0; i < Mb; ++i) t.push_back(enc(df::T_U, i, 1, 0));
    for (int pb = 0; pb + 1 < Nb; ++pb) {
      for (int i = 0; i < Mb; ++i) t.push_back(enc(df::T_S, i, pb + 1, pb + 1));
      for (int j = pb + 2; j < Nb; ++j)
        for (int i = 0; i < Mb; ++i) t.push_back(enc(df::T_U, i, j, pb));
      if (pb + 2 < Nb)
        for (int i = 0; i < Mb; ++i) t.push_back(enc(df::T_U, i, pb + 2, pb + 1));
    }
  }
  return t;
}

std::mutex g_mu;
std::map<std::tuple<int, int, int, int>, std::pair<uint32_t*, int>> g_tables;  // (dev, mode, Mb, Nb)
// mode 2 (POTRF without the chain): ticket at which the tasks of panel step s start
// (the position P(s) has in the full order), s = 0..Nb
std::map<std::pair<int, int>, std::vector<int>> g_step_ticket;  // (Mb, Nb)
int g_num_sms[64];

// mode: 0 TRSM, 1 POTRF (all tasks), 2 POTRF without the critical chain
cudaError_t get_table(int mode, int Mb, int Nb, const uint32_t** out, int* count) {
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> g(g_mu);
  auto key = std::make_tuple(dev, mode, Mb, Nb);
  auto it = g_tables.find(key);
  if (it != g_tables.end()) {
    *out = it->second.first;
    *count = it->second.second;
    return cudaSuccess;
  }
  // Must not be called while a stream is being captured (cudaMemcpy); the runtime
  // calls dataflow_prepare() before capture.
  std::vector<uint32_t> t = build_tasks(mode >= 1, Mb, Nb, mode == 2);
  if (mode == 2) {
    std::vector<int> st((size_t)Nb + 1, (int)t.size());
    int cnt = 0;
    for (uint32_t c : build_tasks(true, Mb, Nb, false)) {
      if ((c >> 30) == df::T_P) st[(size_t)(c & 1023)] = cnt;
      if (!on_chain(c)) ++cnt;
    }
    g_step_ticket[{Mb, Nb}] = st;
  }
  uint32_t* d = nullptr;
  cudaError_t e = cudaMalloc(&d, t.size() * sizeof(uint32_t));
  if (e != cudaSuccess) return e;
  e = cudaMemcpy(d, t.data(), t.size() * sizeof(uint32_t), cudaMemcpyHostToDevice);
  if (e != cudaSuccess) return e;
  g_tables[key] = {d, (int)t.size()};
  *out = d;
  *count = (int)t.size();
  return cudaSuccess;
}

// CTAs of a dataflow POTRF launch (option potrf_ctas = 0): 3 per 64-block column
// (16 .. 96) for one launch: the critical chain needs the bulk updates of the next
// columns done in time (profiles: nb = 1024 0.69 -> 0.59 ms, nb = 2048 3.4 -> 1.3 ms
// at 2 per column; with the look-ahead P of round 2 the chain waited for its S input
// at 2 per column: 396 -> 375 us at 3, tools/potrf_trace.py).  With the two-launch
// form, 2 per column measured n = 8192 -0.7%, n = 16384 -0.2%, n = 32768 -0.1% time
// against 3 but the tile alone 348 -> 369 us (profiles/r02/split_potrf.txt): 3 kept.
int df_max_ctas(int T = 16) { return std::min(96, std::max(16, 3 * T)); }

int num_sms() {
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 64 && g_num_sms[dev]) return g_num_sms[dev];
  int n = 148;
  cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
  if (dev < 64) g_num_sms[dev] = n;
  return n;
}

cudaError_t launch_df(cudaStream_t s, int prio, DfParams& p, int max_ctas) {
  cudaError_t e = cudaMemsetAsync(p.ws, 0, dataflow_ws_bytes(p.m, p.n), s);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  int grid = max_ctas;
  if (grid < 1) grid = 1;
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(df::NT);
  cfg.dynamicSmemBytes = df::SMEM_BYTES;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = prio;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  ++launch_count();
  return cudaLaunchKernelEx(&cfg, dataflow_kernel, p);
}

}  // namespace

size_t dataflow_ws_bytes(int m, int n) {
  const int Mb = (m + df::W - 1) / df::W, Nb = (n + df::W - 1) / df::W;
  // ticket, chain role, per-block progress, then Nb counters of the chain TRSM(k+1,k)
  // that follows a POTRF with programmatic launch (zeroed with the rest)
  return ((size_t)(2 + Mb * Nb + Nb) * sizeof(int) + 255) / 256 * 256;
}

cudaError_t dataflow_prepare(int m, int n, bool potrf) {
  const int Mb = (m + df::W - 1) / df::W, Nb = (n + df::W - 1) / df::W;
  const uint32_t* t;
  int c;
  if (!potrf) return get_table(0, Mb, Nb, &t, &c);
  cudaError_t e = get_table(1, Mb, Nb, &t, &c);
  if (e == cudaSuccess) e = get_table(2, Mb, Nb, &t, &c);
  return e;
}

static int df_crit() {
  static int v = [] {
    const char* e = getenv("STF_DF_CRIT");
    return e ? atoi(e) : 1;
  }();
  return v;
}

cudaError_t dataflow_init_attrs() {
  cudaError_t e = cudaFuncSetAttribute(dataflow_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, df::SMEM_BYTES);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(bulk_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, df::BULK_SMEM_BYTES);
  return e;
}



cudaError_t potrf_tile(cudaStream_t stream, int prio, int n, double* A, int64_t lda, int64_t col0,
                       unsigned long long* info, int* ws, const Mirrors* mirrors, unsigned long long* trace,
                       int ctas_override, int pdl_trig, cudaGraphNode_t* chain_node, int split) {
  if (chain_node) *chain_node = nullptr;
  if (n <= 0) return cudaSuccess;
  DfParams p{};
  p.X = A;
  p.ldx = lda;
  p.L = nullptr;
  p.ldl = 0;
  p.m = p.n = n;
  p.Mb = p.Nb = (n + df::W - 1) / df::W;
  p.crit = df_crit();
  cudaError_t e = get_table(p.crit ? 2 : 1, p.Mb, p.Nb, &p.tasks, &p.ntasks);
  if (e != cudaSuccess) return e;
  p.ws = ws;
  p.col0 = col0;
  p.info = info;
  p.potrf = 1;
  if (mirrors) p.mir = *mirrors;
  const int T = p.Nb;
  const int par = T * (T - 1) / 2 > 0 ? T * (T - 1) / 2 : 1;  // widest update wave
  int ctas = std::min(par, std::min(ctas_override > 0 ? ctas_override : df_max_ctas(T), num_sms()));
  // + the critical-chain CTA; at least one bulk CTA when there are bulk tasks (the
  // chain waits on updates only bulk CTAs claim)
  if (p.crit) ctas = std::min(p.ntasks, std::max(ctas, 2) - 1) + 1;
  p.trace = trace;
  p.trig = pdl_trig;
  if (!p.crit || !split || p.ntasks == 0 || ctas < 3) return launch_df(stream, prio, p, ctas);
  // two launches: the chain + `heavy` block-task CTAs (dataflow_kernel), then bulk_kernel with
  // the rest of the CTAs, released by the first at its start
  e = cudaMemsetAsync(p.ws, 0, dataflow_ws_bytes(p.m, p.n), stream);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = prio;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cfg.blockDim = dim3(df::NT);
  cfg.stream = stream;
  const int heavy = std::max(1, std::min(4, (ctas - 1) / 8));
  cfg.gridDim = dim3(1 + heavy);
  cfg.dynamicSmemBytes = df::SMEM_BYTES;
  DfParams pc = p;
  pc.trig = 0;  // releases its dependent (the bulk launch) at its start
  ++launch_count();
  e = cudaLaunchKernelEx(&cfg, dataflow_kernel, pc);
  if (e != cudaSuccess) return e;
  if (chain_node) {
    cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
    const cudaGraphNode_t* deps = nullptr;
    size_t nd = 0;
    if (cudaStreamGetCaptureInfo_v3(stream, &st, nullptr, nullptr, &deps, nullptr, &nd) == cudaSuccess &&
        st == cudaStreamCaptureStatusActive && nd == 1)
      *chain_node = deps[0];
    cudaGetLastError();
  }
  // bulk CTAs release TRSM(k+1,k) at the first ticket of panel step pdl_trig
  DfParams pb = p;
  pb.trig = -1;
  if (pdl_trig >= 0) {
    std::lock_guard<std::mutex> g(g_mu);
    const std::vector<int>& stt = g_step_ticket[{p.Mb, p.Nb}];
    pb.trig = stt.empty() ? 0 : stt[(size_t)std::min(pdl_trig, p.Nb)];
  }
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.numAttrs = 2;
  cfg.gridDim = dim3(ctas - 1 - heavy);
  cfg.dynamicSmemBytes = df::BULK_SMEM_BYTES;
  ++launch_count();
  return cudaLaunchKernelEx(&cfg, bulk_kernel, pb);
}

cudaError_t trsm_tile(cudaStream_t stream, int prio, int M, int n, const double* L, int64_t ldl, double* B,
                      int64_t ldb, int* ws) {
  if (M <= 0 || n <= 0) return cudaSuccess;
  DfParams p{};
  p.X = B;
  p.ldx = ldb;
  p.L = L;
  p.ldl = ldl;
  p.m = M;
  p.n = n;
  p.Mb = (M + df::W - 1) / df::W;
  p.Nb = (n + df::W - 1) / df::W;
  cudaError_t e = get_table(0, p.Mb, p.Nb, &p.tasks, &p.ntasks);
  if (e != cudaSuccess) return e;
  p.ws = ws;
  p.col0 = 0;
  p.info = nullptr;
  p.potrf = 0;
  p.crit = 0;
  p.trace = nullptr;
  p.trig = -1;
  const int par = p.Mb * (p.Nb > 1 ? p.Nb - 1 : 1);
  return launch_df(stream, prio, p, std::min(par, std::min(4 * df_max_ctas(16), num_sms())));
}

}  // namespace stfk
