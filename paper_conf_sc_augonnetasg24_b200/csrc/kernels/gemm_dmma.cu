// K1 / K2: FP64 tile update C -= A * B^T on the sm_100a FP64 tensor pipe (DMMA),
// operands staged by TMA into 128B-swizzled shared memory through an mbarrier
// pipeline (north_star "SYRK/GEMM trailing updates as FP64
// tensor-core (DMMA) contractions fed by TMA into shared memory").
//
// Tile task definitions ("calling cuBLAS ... kernels within tasks",
// right-looking tiled Cholesky of ref. [17] PAPER.md:495):
//   GEMM(i,j,k):  A_ij <- A_ij - L_ik * L_jk^T
//   SYRK(i,k):    A_ii <- A_ii - L_ik * L_ik^T   (lower triangle only)
//
// B200 facts shaping the design (profiles/calib_fp64_r01.json):
//   * tcgen05 has no f64 kind; FP64 tensor math is warp-level mma.sync -> DMMA.8x8x4,
//     peak 64 FMA/clk/SM = 37.1 TFLOP/s measured (148 SMs, 1965 MHz held under load).
//   * DMMA accumulates in registers, so the design is the classic register-tiled
//     warp GEMM fed by a TMA/mbarrier producer warp.
//
// CTA tile 128 x 128 x 16, 4 stages (128 KB smem), 8 warps (warp tile 64 x 32 ->
// 64 FP64 accumulators / thread); thread 0 doubles as the TMA producer.
// Shared-memory layout of one operand stage: 8 boxes of [16 k-rows][16 m] doubles,
// each k-row 128 B with the 128B swizzle (16-byte chunk c stored at c ^ (row & 7)).
// Fragment k-permutation: within a k8 group the DMMA with kh in {0,1} takes
// k = 2*t + kh from lane t = lane&3, so the 4 rows a half-warp touches have
// row&7 in {kh, kh+2, kh+4, kh+6}: conflict-free 64-bit LDS under the swizzle.
// The k order is fixed, so results are deterministic run to run.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>

#include "ptx.cuh"
#include "tile_ops.hpp"

namespace stfk {

template <int BK_, int STAGES_, int BN_ = 128, int MINB_ = 1, int BM_ = 128>
struct Cfg {
  static constexpr int BM = BM_, BN = BN_, BK = BK_, STAGES = STAGES_, MINB = MINB_;
  static constexpr int BOX = 16;                  // doubles per 128-byte swizzle row
  static constexpr int BOX_BYTES = BOX * BK * 8;  // 2 KB at BK = 16
  static constexpr int A_BYTES = BM * BK * 8;     // 16 KB at BK = 16
  static constexpr int B_BYTES = BN * BK * 8;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 1024 /*align*/ + STAGES * 8 + STAGES * 4;
};
using CfgK16 = Cfg<16, 4>;  // 4 x 32 KB stages
using CfgK32 = Cfg<32, 3>;  // 3 x 64 KB stages
using CfgN64 = Cfg<32, 2, 64, 2>;  // 128 x 64 CTA tile, 2 x 48 KB stages, 2 CTAs / SM (full GEMMs only)
// 64 x 64 CTA tile, 4 warps of 32 x 32, 3 x 32 KB stages, 2 CTAs / SM: SYRK tiles of order <= 1024
// (136 CTAs at nb = 1024, one wave on 148 SMs: the critical SYRK(k+1,k) spreads over the whole GPU
// instead of 72 CTAs of 128 x 64).  Same per-element k order as the other tiles: same bits.
using CfgS64 = Cfg<32, 3, 64, 2, 64>;

// Exact negation as a sign-bit flip on the integer pipe (keeps the FP64/DMMA pipe free).
__device__ __forceinline__ double neg(double x) {
  return __longlong_as_double(__double_as_longlong(x) ^ (long long)0x8000000000000000ULL);
}

// Byte offset of element (row r in [0,128), k in [0,BK)) inside one operand stage.
template <class g>
__device__ __forceinline__ uint32_t swz_off(int r, int k) {
  const int box = r >> 4, mi = r & 15;
  return box * g::BOX_BYTES + k * 128 + ((((mi >> 1) ^ (k & 7)) << 4) | ((mi & 1) << 3));
}

// Further operand pairs of a merged update C -= A B^T + A2 B2^T + ... (up to 4
// pairs, each K deep): consecutive tile updates in one k sweep.
struct ExtraPairs {
  CUtensorMap a[3], b[3];
  int npairs;  // total pairs including (tmA, tmB): 1..4
  // Overlap with the producing TRSM (programmatic dependent launch, SYRK(k+1,k) of
  // the panel chain): k columns [64 c, 64 c + 64) of the operands are final once
  // kflag[c] >= kcount (the TRSM's CTAs count their finished column blocks);
  // null: operands complete at launch.
  const int* kflag;
  int kcount;
};

// k-tile kt: pair p = kt / KT1 (p = 0: tmA, tmB), tile kt - p KT1 of that pair
template <class g>
__device__ __forceinline__ void load_stage(uint8_t* smem, int s, const CUtensorMap* tmA, const CUtensorMap* tmB,
                                           const ExtraPairs* ex, int KT1, int m0, int n0, int kt, uint64_t* full) {
  if (ex->kflag) {  // k columns of this tile published by the TRSM (acquire), then visible to TMA
    const int* f = ex->kflag + (kt * g::BK) / 64;
    for (;;) {
      int v;
      asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(f) : "memory");
      if (v >= ex->kcount) break;
      __nanosleep(64);
    }
    asm volatile("fence.proxy.async.global;" ::: "memory");
  }
  mbar_arrive_expect_tx(&full[s], g::STAGE_BYTES);
  uint8_t* sa = smem + s * g::STAGE_BYTES;
  uint8_t* sb = sa + g::A_BYTES;
  const int pr = kt / KT1;
  const CUtensorMap* ma = pr == 0 ? tmA : &ex->a[pr - 1];
  const CUtensorMap* mb = pr == 0 ? tmB : &ex->b[pr - 1];
  const int kk = kt - pr * KT1;
#pragma unroll
  for (int b = 0; b < g::BM / g::BOX; ++b) tma_load_2d(sa + b * g::BOX_BYTES, ma, m0 + b * g::BOX, kk * g::BK, &full[s]);
#pragma unroll
  for (int b = 0; b < g::BN / g::BOX; ++b) tma_load_2d(sb + b * g::BOX_BYTES, mb, n0 + b * g::BOX, kk * g::BK, &full[s]);
}

// All warps are consumers (a dedicated producer warp would lower the register cap:
// the register file is split per SM sub-partition, 9 warps round up to 12).  The
// refill of a stage is issued by the LAST warp to finish reading it (shared-memory
// arrival counter), i.e. at the earliest possible moment, with the next k-tile
// STAGES ahead; consumers wait only on the TMA "full" mbarriers.
template <int WM, int WN, class g>
__global__ void __launch_bounds__((g::BM / WM) * (g::BN / WN) * 32, g::MINB)
    gemm_nt_dmma_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                        const __grid_constant__ ExtraPairs ex, double* __restrict__ C, int64_t ldc, int M, int N,
                        int K, int lower) {
  constexpr int NCW = (g::BM / WM) * (g::BN / WN);
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // keep the pointer derived from the __shared__ array (integer offset only) so
  // the compiler emits LDS, not generic LD, for the fragment loads
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + g::STAGES * g::STAGE_BYTES);
  int* released = reinterpret_cast<int*>(full + g::STAGES);  // per-stage arrival counters

  int tm, tn;
  if (lower) {
    // linear block -> CTA tiles touching the lower triangle.  BN == BM: tn <= tm
    // (row tm holds tm + 1 tiles); BN == BM / 2: tn <= 2 tm + 1 (row tm holds 2 tm + 2).
    const int b = blockIdx.x;
    if (g::BN == g::BM) {
      int t = (int)((sqrtf(8.0f * b + 1.0f) - 1.0f) * 0.5f);
      while ((t + 1) * (t + 2) / 2 <= b) ++t;
      while (t * (t + 1) / 2 > b) --t;
      tm = t;
      tn = b - t * (t + 1) / 2;
    } else {
      int t = (int)((sqrtf(4.0f * b + 1.0f) - 1.0f) * 0.5f);
      while ((t + 1) * (t + 2) <= b) ++t;
      while (t * (t + 1) > b) --t;
      tm = t;
      tn = b - t * (t + 1);
    }
  } else {
    // L2-aware order: CTAs are dispatched in linear block order; walk the M tiles in
    // groups of 16 rows before moving along N, so the CTAs resident at once (2 per
    // SM) share ~16 A row panels and ~18 B column panels instead of sweeping all of A
    // per B panel (a 1024-tile update, 8 x 16 CTAs, is one group: unchanged)
    constexpr int G = 16;
    const int tMg = gridDim.x, tNg = gridDim.y;
    const int bid = blockIdx.x + blockIdx.y * tMg, per = G * tNg;
    const int grp = bid / per, first = grp * G, gs = min(tMg - first, G), rr = bid - grp * per;
    tm = first + rr % gs;
    tn = rr / gs;
  }
  const int m0 = tm * g::BM, n0 = tn * g::BN;
  const int KT1 = (K + g::BK - 1) / g::BK;
  const int KT = KT1 * ex.npairs;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    tma_prefetch_desc(&tmA);
    tma_prefetch_desc(&tmB);
    for (int pr = 1; pr < ex.npairs; ++pr) {
      tma_prefetch_desc(&ex.a[pr - 1]);
      tma_prefetch_desc(&ex.b[pr - 1]);
    }
    for (int s = 0; s < g::STAGES; ++s) {
      mbar_init(&full[s], 1);
      released[s] = 0;
    }
    fence_barrier_init();
    for (int kt = 0; kt < g::STAGES && kt < KT; ++kt) load_stage<g>(smem, kt, &tmA, &tmB, &ex, KT1, m0, n0, kt, full);
  }
  __syncthreads();

  const int wm0 = (warp % (g::BM / WM)) * WM;
  const int wn0 = (warp / (g::BM / WM)) * WN;
  const int gq = lane >> 2, tq = lane & 3;

  // In lower mode, warps of a diagonal CTA whose warp tile is strictly upper idle.
  const bool warp_dead = lower && (m0 + wm0 + WM <= n0 + wn0);  // warp tile strictly above the diagonal

  // acc = C, loaded straight into the accumulators (64 independent loads in
  // flight, latency hidden behind the first TMA wait); the mainloop adds
  // A * (-B)^T with the B fragments sign-flipped (exact), so acc = C - A B^T.
  double acc[WM / 8][WN / 8][2];
#pragma unroll
  for (int i = 0; i < WM / 8; ++i) {
    const int m = m0 + wm0 + 8 * i + gq;
#pragma unroll
    for (int j = 0; j < WN / 8; ++j)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int n = n0 + wn0 + 8 * j + 2 * tq + h;
        const bool in = !warp_dead && m < M && n < N && (!lower || m >= n);
        acc[i][j][h] = in ? __ldg(C + (int64_t)n * ldc + m) : 0.0;
      }
  }

  // Per-lane fragment offsets: swz_off(w0 + 8f + gq, 2tq + kh) depends on f only
  // through the box (f >> 1, an immediate) and the chunk bit 2 (f & 1).
  uint32_t offA[2][2], offB[2][2];
#pragma unroll
  for (int p = 0; p < 2; ++p)
#pragma unroll
    for (int kh = 0; kh < 2; ++kh) {
      offA[p][kh] = swz_off<g>(wm0 + 8 * p + gq, 2 * tq + kh);
      offB[p][kh] = g::A_BYTES + swz_off<g>(wn0 + 8 * p + gq, 2 * tq + kh);
    }

  for (int kt = 0; kt < KT; ++kt) {
    const int s = kt % g::STAGES;
    mbar_wait(&full[s], (kt / g::STAGES) & 1);
    const uint8_t* st = smem + s * g::STAGE_BYTES;
    if (!warp_dead) {
#pragma unroll
      for (int grp = 0; grp < g::BK / 8; ++grp) {
        double a[WM / 8][2], b[WN / 8][2];
#pragma unroll
        for (int f = 0; f < WM / 8; ++f)
#pragma unroll
          for (int kh = 0; kh < 2; ++kh)
            a[f][kh] = *reinterpret_cast<const double*>(st + offA[f & 1][kh] + (f >> 1) * g::BOX_BYTES + grp * 8 * 128);
#pragma unroll
        for (int f = 0; f < WN / 8; ++f)
#pragma unroll
          for (int kh = 0; kh < 2; ++kh)
            b[f][kh] = neg(*reinterpret_cast<const double*>(st + offB[f & 1][kh] + (f >> 1) * g::BOX_BYTES + grp * 8 * 128));
#pragma unroll
        for (int kh = 0; kh < 2; ++kh)
#pragma unroll
          for (int i = 0; i < WM / 8; ++i)
#pragma unroll
            for (int j = 0; j < WN / 8; ++j) dmma_8x8x4(acc[i][j][0], acc[i][j][1], a[i][kh], b[j][kh]);
      }
    }
    __syncwarp();  // this warp's reads of stage s are complete (their values fed its DMMAs)
    if (lane == 0 && kt + g::STAGES < KT) {
      __threadfence_block();
      if (atomicAdd(&released[s], 1) == NCW - 1) {  // last reader of stage s refills it
        released[s] = 0;
        __threadfence_block();
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        load_stage<g>(smem, s, &tmA, &tmB, &ex, KT1, m0, n0, kt + g::STAGES, full);
      }
    }
  }

  if (warp_dead) return;
  // ---------------- epilogue: C -= acc
#pragma unroll
  for (int i = 0; i < WM / 8; ++i) {
    const int m = m0 + wm0 + 8 * i + gq;
#pragma unroll
    for (int j = 0; j < WN / 8; ++j) {
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int n = n0 + wn0 + 8 * j + 2 * tq + h;
        if (m < M && n < N && (!lower || m >= n)) C[(int64_t)n * ldc + m] = acc[i][j][h];
      }
    }
  }
}

// ------------------------------------------------------------------ host side
static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  });
  return fn;
}

// rows x cols column-major FP64 operand, box {16 rows, bk cols}, 128B swizzle, OOB -> 0.
bool make_operand_map(CUtensorMap* tm, const double* ptr, int rows, int cols, int64_t ld, int bk) {
  auto fn = encode_fn();
  if (!fn) return false;
  cuuint64_t dims[2] = {(cuuint64_t)rows, (cuuint64_t)cols};
  cuuint64_t strides[1] = {(cuuint64_t)ld * sizeof(double)};
  cuuint32_t box[2] = {16u, (cuuint32_t)bk};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = fn(tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, const_cast<double*>(ptr), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

// Variants: warps 8 (64x32 warp tiles, 224 regs, 2 warps / SM sub-partition) or
// 16 (32x32, <= 128 regs, 4 warps / sub-partition); BK 16 (4 stages) or 32 (3
// stages).  STF_GEMM_WARPS / STF_GEMM_BK select; defaults 8 warps, BK 32 (best
// in the concurrent factorisation, profiles/r01/ablations_*.txt).
static int env_or(const char* name, int dflt) {
  const char* e = getenv(name);
  return e ? atoi(e) : dflt;
}
static int gemm_warps() {
  static int v = env_or("STF_GEMM_WARPS", 8) == 16 ? 16 : 8;
  return v;
}
static int gemm_bk() {
  static int v = env_or("STF_GEMM_BK", 32) == 16 ? 16 : 32;
  return v;
}
// CTA tile: STF_GEMM_NARROW = 2 (default): 128 x 64, 8 warps of 32 x 32, 2 CTAs per SM
// (one CTA's start-up and epilogue hide behind the other's mainloop: 95.6% of peak
// on 8192^2 x 1024); 1: 128 x 64, 4 warps of 64 x 32; 0: 128 x 128, 1 CTA per SM.
static int gemm_narrow() {
  static int v = env_or("STF_GEMM_NARROW", 2);
  return v;
}

// warps of the 64 x 64 CTA tile: 4 (32 x 32 each) or 8 (32 x 16; STF_S64_WARPS)
static int s64_warps() {
  static int v = env_or("STF_S64_WARPS", 8) == 4 ? 4 : 8;
  return v;
}
// SYRK (lower) tiles up to this order use the 64 x 64 CTA tile (STF_SYRK64_MAX, default 1024)
static int syrk64_max() {
  static int v = env_or("STF_SYRK64_MAX", 1024);
  return v;
}

template <class G>
static cudaError_t launch_variant(cudaLaunchConfig_t& cfg, const CUtensorMap& tmA, const CUtensorMap& tmB,
                                  const ExtraPairs& ex, double* C, int64_t ldc, int M, int N, int K, int lower) {
  cfg.dynamicSmemBytes = G::SMEM_BYTES;
  if (gemm_warps() == 16) {
    cfg.blockDim = dim3(512, 1, 1);
    return cudaLaunchKernelEx(&cfg, gemm_nt_dmma_kernel<32, 32, G>, tmA, tmB, ex, C, ldc, M, N, K, lower);
  }
  cfg.blockDim = dim3(256, 1, 1);
  return cudaLaunchKernelEx(&cfg, gemm_nt_dmma_kernel<64, 32, G>, tmA, tmB, ex, C, ldc, M, N, K, lower);
}

cudaError_t gemm_nt(cudaStream_t stream, int prio, int M, int N, int K, const double* A, int64_t lda,
                    const double* B, int64_t ldb, double* C, int64_t ldc, int lower) {
  return gemm_nt_tiles(stream, prio, M, N, K, A, lda, B, ldb, C, ldc, lower, 0);
}

cudaError_t gemm_nt_tiles(cudaStream_t stream, int prio, int M, int N, int K, const double* A, int64_t lda,
                          const double* B, int64_t ldb, double* C, int64_t ldc, int lower, int small) {
  const double* As[1] = {A};
  const double* Bs[1] = {B};
  return gemm_nt_multi(stream, prio, M, N, K, 1, As, lda, Bs, ldb, C, ldc, lower, small);
}

cudaError_t gemm_nt_multi(cudaStream_t stream, int prio, int M, int N, int K, int npairs, const double* const* As,
                          int64_t lda, const double* const* Bs, int64_t ldb, double* C, int64_t ldc, int lower,
                          int small, const int* kflag, int kcount) {
  if (M <= 0 || N <= 0 || K <= 0) return cudaSuccess;
  if (npairs < 1 || npairs > 4) return cudaErrorInvalidValue;
  if ((lda & 1) || (ldb & 1)) return cudaErrorMisalignedAddress;
  for (int p = 0; p < npairs; ++p)
    if ((reinterpret_cast<uintptr_t>(As[p]) & 15) || (reinterpret_cast<uintptr_t>(Bs[p]) & 15))
      return cudaErrorMisalignedAddress;
  const bool narrow = gemm_narrow() != 0;
  const int bk = narrow ? 32 : gemm_bk();
  // every pair after the first starts on a fresh k tile: K must fill whole tiles
  if (npairs > 1 && K % bk) return cudaErrorInvalidValue;
  CUtensorMap tmA, tmB;
  if (!make_operand_map(&tmA, As[0], M, K, lda, bk) || !make_operand_map(&tmB, Bs[0], N, K, ldb, bk))
    return cudaErrorInvalidValue;
  ExtraPairs ex;
  memset(&ex, 0, sizeof ex);
  ex.npairs = npairs;
  ex.kflag = kflag;
  ex.kcount = kcount;
  if (kflag && (npairs != 1 || K % 64)) return cudaErrorInvalidValue;
  for (int p = 1; p < 4; ++p) {
    if (p < npairs) {
      if (!make_operand_map(&ex.a[p - 1], As[p], M, K, lda, bk) || !make_operand_map(&ex.b[p - 1], Bs[p], N, K, ldb, bk))
        return cudaErrorInvalidValue;
    } else {
      ex.a[p - 1] = tmA;
      ex.b[p - 1] = tmB;
    }
  }
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = prio;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cfg.stream = stream;
  if ((lower && M <= syrk64_max() && bk == CfgS64::BK) || (small && bk == CfgS64::BK)) {
    const int t64 = (M + 63) / 64;
    cfg.gridDim = lower ? dim3(t64 * (t64 + 1) / 2, 1, 1) : dim3(t64, (N + 63) / 64, 1);
    cfg.dynamicSmemBytes = CfgS64::SMEM_BYTES;
    ++launch_count();
    if (s64_warps() == 8) {  // 32 x 16 warp tiles: two warps per SM sub-partition
      cfg.blockDim = dim3(256, 1, 1);
      return cudaLaunchKernelEx(&cfg, gemm_nt_dmma_kernel<32, 16, CfgS64>, tmA, tmB, ex, C, ldc, M, N, K, lower);
    }
    cfg.blockDim = dim3(128, 1, 1);
    return cudaLaunchKernelEx(&cfg, gemm_nt_dmma_kernel<32, 32, CfgS64>, tmA, tmB, ex, C, ldc, M, N, K, lower);
  }
  const int tM = (M + 127) / 128, tN = narrow ? (N + 63) / 64 : (N + 127) / 128;
  cfg.gridDim = lower ? dim3(narrow ? tM * (tM + 1) : tM * (tM + 1) / 2, 1, 1) : dim3(tM, tN, 1);
  ++launch_count();
  if (narrow) {
    cfg.dynamicSmemBytes = CfgN64::SMEM_BYTES;
    if (gemm_narrow() == 2) {  // 8 warps of 32 x 32, 2 CTAs (16 warps) per SM
      cfg.blockDim = dim3(256, 1, 1);
      return cudaLaunchKernelEx(&cfg, gemm_nt_dmma_kernel<32, 32, CfgN64>, tmA, tmB, ex, C, ldc, M, N, K, lower);
    }
    cfg.blockDim = dim3(128, 1, 1);  // 4 warps of 64 x 32
    return cudaLaunchKernelEx(&cfg, gemm_nt_dmma_kernel<64, 32, CfgN64>, tmA, tmB, ex, C, ldc, M, N, K, lower);
  }
  if (bk == 32) return launch_variant<CfgK32>(cfg, tmA, tmB, ex, C, ldc, M, N, K, lower);
  return launch_variant<CfgK16>(cfg, tmA, tmB, ex, C, ldc, M, N, K, lower);
}

template <class G>
static cudaError_t set_attrs() {
  cudaError_t e = cudaFuncSetAttribute(gemm_nt_dmma_kernel<64, 32, G>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       G::SMEM_BYTES);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(gemm_nt_dmma_kernel<32, 32, G>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             G::SMEM_BYTES);
  return e;
}

cudaError_t gemm_init_attrs() {
  cudaError_t e = set_attrs<CfgK16>();
  if (e == cudaSuccess) e = set_attrs<CfgK32>();
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(gemm_nt_dmma_kernel<64, 32, CfgN64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             CfgN64::SMEM_BYTES);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(gemm_nt_dmma_kernel<32, 32, CfgN64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             CfgN64::SMEM_BYTES);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(gemm_nt_dmma_kernel<32, 32, CfgS64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             CfgS64::SMEM_BYTES);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(gemm_nt_dmma_kernel<32, 16, CfgS64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             CfgS64::SMEM_BYTES);
  return e;
}

}  // namespace stfk
