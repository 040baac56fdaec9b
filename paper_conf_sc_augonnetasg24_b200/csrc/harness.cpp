// include/stf_harness.h: seeded input generation on the device, direct tile-kernel
// entry points (kernel-level parity tests), kernel timing for the roofline, and
// debug timelines.  None of these is part of a factorisation.
#include <algorithm>
#include <climits>

#include "../../include/stf_harness.h"
#include "runtime_internal.hpp"

using namespace stfrt;

extern "C" {

int stf_fill_spd_tiles(int64_t n, int64_t nb, const stf_matrix_desc* A_desc, int ngpus, uint64_t seed) {
  g_err.clear();
  if (!A_desc || A_desc->kind != STF_DESC_TILED_2DBC || nb < 1 || n % nb || !A_desc->tiles)
    return fail(-4, "stf_fill_spd_tiles needs a TILED_2DBC descriptor");
  const int64_t T = n / nb;
  int cur = 0;
  cudaGetDevice(&cur);
  std::vector<int> devs;
  for (int64_t j = 0; j < T; ++j)
    for (int64_t i = j; i < T; ++i) {
      double* tp = A_desc->tiles[(size_t)(i + j * T)];
      if (!tp) continue;  // not held by this process (multi-process mode)
      int d = 0;
      if (!device_of(tp, &d)) return fail(-4, "tile (%lld,%lld) is not device memory", (long long)i, (long long)j);
      cudaSetDevice(d);
      CUDA_TRY(stfk::fill_spd(0, tp, nb, n, i * nb, j * nb, (int)nb, (int)nb, seed), "fill_spd");
      if (std::find(devs.begin(), devs.end(), d) == devs.end()) devs.push_back(d);
    }
  for (int d : devs) {
    cudaSetDevice(d);
    CUDA_TRY(cudaDeviceSynchronize(), "fill_spd sync");
  }
  cudaSetDevice(cur);
  (void)ngpus;
  return 0;
}

int stf_fill_spd_block(double* dst, int64_t ld, int64_t n, int64_t r0, int64_t c0, int64_t rows, int64_t cols,
                       uint64_t seed) {
  g_err.clear();
  if (!dst || ld < rows || rows < 0 || cols < 0) return fail(-4, "bad block arguments");
  CUDA_TRY(stfk::fill_spd(0, dst, ld, n, r0, c0, (int)rows, (int)cols, seed), "fill_spd");
  CUDA_TRY(cudaStreamSynchronize(0), "fill_spd sync");
  return 0;
}

int stf_kernel_gemm_nt(int64_t M, int64_t N, int64_t K, const double* A, int64_t lda, const double* B, int64_t ldb,
                       double* C, int64_t ldc, int lower) {
  g_err.clear();
  int dev = 0;
  cudaGetDevice(&dev);
  int r = ensure_kernel_attrs(dev);
  if (r) return r;
  if (lower && M != N) return fail(-4, "lower (SYRK) mode needs M == N");
  CUDA_TRY(stfk::gemm_nt(0, 0, (int)M, (int)N, (int)K, A, lda, B, ldb, C, ldc, lower), "gemm_nt");
  CUDA_TRY(cudaStreamSynchronize(0), "gemm_nt sync");
  return 0;
}

int stf_kernel_trsm(int64_t M, int64_t n, const double* L, int64_t ldl, double* B, int64_t ldb) {
  g_err.clear();
  int dev = 0;
  cudaGetDevice(&dev);
  int r = ensure_kernel_attrs(dev);
  if (r) return r;
  const int64_t trsm = ctx().opt.trsm;
  if (trsm == 3 && stfk::trsm_res_supported((int)n, L, ldl)) {
    CUDA_TRY(stfk::trsm_res_parts(0, 0, (int)M, (int)n, L, ldl, B, ldb, nullptr, (int)ctx().opt.trsm_res_split),
             "trsm (resident panel)");
    CUDA_TRY(cudaStreamSynchronize(0), "trsm sync");
    return 0;
  }
  if (trsm >= 2) {
    CUDA_TRY(stfk::trsm_panel(0, 0, (int)M, (int)n, L, ldl, B, ldb, (int)ctx().opt.trsm_rows), "trsm (row panel)");
    CUDA_TRY(cudaStreamSynchronize(0), "trsm sync");
    return 0;
  }
  if (trsm == 1) {
    int* ws = nullptr;
    CUDA_TRY(cudaMalloc(&ws, stfk::dataflow_ws_bytes((int)M, (int)n)), "ws alloc");
    cudaError_t e = stfk::trsm_tile(0, 0, (int)M, (int)n, L, ldl, B, ldb, ws);
    if (e == cudaSuccess) e = cudaStreamSynchronize(0);
    cudaFree(ws);
    CUDA_TRY(e, "trsm (dataflow)");
    return 0;
  }
  CUDA_TRY(stfk::trsm_rlt(0, 0, (int)M, (int)n, L, ldl, B, ldb), "trsm");
  CUDA_TRY(cudaStreamSynchronize(0), "trsm sync");
  return 0;
}

int stf_kernel_potrf(int64_t n, double* A, int64_t lda, int64_t* info) {
  g_err.clear();
  int dev = 0;
  cudaGetDevice(&dev);
  int r = ensure_kernel_attrs(dev);
  if (r) return r;
  unsigned long long* d_info = nullptr;
  CUDA_TRY(cudaMalloc(&d_info, sizeof *d_info), "info alloc");
  int* ws = nullptr;
  cudaError_t e = cudaMalloc(&ws, stfk::dataflow_ws_bytes((int)n, (int)n));
  if (e == cudaSuccess) e = stfk::info_reset(0, d_info);
  if (e == cudaSuccess)
    e = ctx().opt.dataflow ? stfk::potrf_tile(0, 0, (int)n, A, lda, 0, d_info, ws, nullptr, nullptr,
                                              (int)ctx().opt.potrf_ctas, -1, nullptr, (int)ctx().opt.potrf_split)
                           : stfk::potrf_lower(0, 0, (int)n, A, lda, 0, d_info);
  unsigned long long v = ULLONG_MAX;
  if (e == cudaSuccess) e = cudaMemcpy(&v, d_info, sizeof v, cudaMemcpyDeviceToHost);
  cudaFree(d_info);
  cudaFree(ws);
  if (e != cudaSuccess) return cuda_fail(e, "potrf");
  if (info) *info = (v == ULLONG_MAX) ? 0 : (int64_t)v;
  return 0;
}

// kind 4: one panel step of the critical chain, POTRF(k) -> TRSM(k+1,k) -> SYRK(k+1,k)
// on nb = M tiles, lowered as in a factorisation (one stream; with the pdl option
// the TRSM overlaps the POTRF through a programmatic capture edge), captured into a
// graph with the input restores in front and timing events around the chain.
static int bench_chain(int64_t M, int reps, double* avg_ms) {
  if (M % 64 || M > 1024) return fail(-4, "chain bench: M must be a multiple of 64, <= 1024");
  const Options& o = ctx().opt;
  const size_t bytes = (size_t)(M * M) * 8;
  double *A0 = nullptr, *B0 = nullptr, *C0 = nullptr, *A = nullptr, *B = nullptr, *Cm = nullptr;
  unsigned long long* info = nullptr;
  int* ws = nullptr;
  cudaStream_t s = nullptr;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  cudaGraph_t g = nullptr;
  cudaGraphExec_t ge = nullptr;
  cudaError_t e = cudaSuccess;
  int r = 0;
  auto step = [&](cudaError_t x) {
    if (e == cudaSuccess) e = x;
  };
  step(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  step(cudaEventCreate(&e0));
  step(cudaEventCreate(&e1));
  for (double** p : {&A0, &B0, &C0, &A, &B, &Cm}) step(cudaMalloc(p, bytes));
  step(cudaMalloc(&info, sizeof *info));
  step(cudaMalloc(&ws, stfk::dataflow_ws_bytes((int)M, (int)M)));
  if (e == cudaSuccess) {
    // A_kk, A_{k+1,k}, A_{k+1,k+1}: blocks of one SPD matrix of order 2M
    step(stfk::fill_spd(s, A0, M, 2 * M, 0, 0, (int)M, (int)M, 21));
    step(stfk::fill_spd(s, B0, M, 2 * M, M, 0, (int)M, (int)M, 21));
    step(stfk::fill_spd(s, C0, M, 2 * M, M, M, (int)M, (int)M, 21));
    step(stfk::dataflow_prepare((int)M, (int)M, true));
    step(cudaStreamSynchronize(s));
  }
  const bool pdl = o.pdl && o.dataflow && o.trsm == 3;
  if (e == cudaSuccess) step(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
  if (e == cudaSuccess) {
    step(cudaMemcpyAsync(A, A0, bytes, cudaMemcpyDeviceToDevice, s));
    step(cudaMemcpyAsync(B, B0, bytes, cudaMemcpyDeviceToDevice, s));
    step(cudaMemcpyAsync(Cm, C0, bytes, cudaMemcpyDeviceToDevice, s));
    step(stfk::info_reset(s, info));
    cudaGraphNode_t extra = capture_last_node(s);  // debug: an extra full dependency of the TRSM
    step(cudaEventRecordWithFlags(e0, s, cudaEventRecordExternal));
    const int nbk = (int)(M / 64);
    const int trig = pdl ? (int)std::max<int64_t>(0, nbk - pdl_lead_of(o.pdl_lead, M)) : -1;
    cudaGraphNode_t chain = nullptr;
    step(stfk::potrf_tile(s, 0, (int)M, A, M, 0, info, ws, nullptr, nullptr, (int)o.potrf_ctas, trig, &chain,
                          (int)o.potrf_split));
    cudaGraphNode_t pn = capture_last_node(s);
    if (chain) step(cudaStreamUpdateCaptureDependencies(s, &chain, 1, cudaStreamAddCaptureDependencies));
    if (pdl) {
      // one programmatic edge into the TRSM (see exec.cpp); debug: a second, full edge
      static const int dbg = getenv("STF_DEBUG_CHAIN_MODE") ? atoi(getenv("STF_DEBUG_CHAIN_MODE")) : 0;
      if (chain && !r) r = capture_drop_dependency(s, chain);
      if ((dbg & 2) && extra) step(cudaStreamUpdateCaptureDependencies(s, &extra, 1, cudaStreamAddCaptureDependencies));
      if (pn && !r) r = std::min(0, capture_make_programmatic(s, pn));
      int* kflag = ws + 2 + nbk * nbk;
      step(stfk::trsm_res(s, 0, (int)M, (int)M, A, M, B, M, nullptr, nullptr, ws + 2, nbk, kflag, trig));
      cudaGraphNode_t tn = capture_last_node(s);
      if (tn && !r) r = std::min(0, capture_make_programmatic(s, tn));
      const double* Bp = B;
      step(stfk::gemm_nt_multi(s, 0, (int)M, (int)M, (int)M, 1, &Bp, M, &Bp, M, Cm, M, 1, 0, kflag,
                               (int)(M / stfk::kTrsmResRows)));
    } else {
      step(stfk::trsm_res_parts(s, 0, (int)M, (int)M, A, M, B, M, nullptr, (int)o.trsm_res_split));
      step(stfk::gemm_nt(s, 0, (int)M, (int)M, (int)M, B, M, B, M, Cm, M, 1));
    }
    step(cudaEventRecordWithFlags(e1, s, cudaEventRecordExternal));
    cudaError_t ec = cudaStreamEndCapture(s, &g);
    step(ec);
  }
  if (e == cudaSuccess && !r && getenv("STF_DEBUG_CHAIN")) {  // edges of the captured chain graph
    size_t nn = 0;
    cudaGraphGetNodes(g, nullptr, &nn);
    std::vector<cudaGraphNode_t> nodes(nn);
    cudaGraphGetNodes(g, nodes.data(), &nn);
    for (size_t i = 0; i < nn; ++i) {
      cudaGraphNodeType ty;
      cudaGraphNodeGetType(nodes[i], &ty);
      size_t nd = 0;
      cudaGraphNodeGetDependencies_v2(nodes[i], nullptr, nullptr, &nd);
      std::vector<cudaGraphNode_t> d(nd);
      std::vector<cudaGraphEdgeData> ed(nd);
      cudaGraphNodeGetDependencies_v2(nodes[i], d.data(), ed.data(), &nd);
      fprintf(stderr, "node %zu type %d deps:", i, (int)ty);
      for (size_t k = 0; k < nd; ++k) {
        size_t j = std::find(nodes.begin(), nodes.end(), d[k]) - nodes.begin();
        fprintf(stderr, " %zu(type %d port %d)", j, (int)ed[k].type, (int)ed[k].from_port);
      }
      fprintf(stderr, "\n");
    }
  }
  if (e == cudaSuccess && !r) step(cudaGraphInstantiate(&ge, g, 0));
  double total = 0;
  for (int it = 0; it < reps + 1 && e == cudaSuccess && !r; ++it) {
    step(cudaGraphLaunch(ge, s));
    step(cudaStreamSynchronize(s));
    float ms = 0;
    step(cudaEventElapsedTime(&ms, e0, e1));
    if (it > 0) total += ms;
  }
  if (ge) cudaGraphExecDestroy(ge);
  if (g) cudaGraphDestroy(g);
  for (double* p : {A0, B0, C0, A, B, Cm}) cudaFree(p);
  cudaFree(info);
  cudaFree(ws);
  if (e0) cudaEventDestroy(e0);
  if (e1) cudaEventDestroy(e1);
  if (s) cudaStreamDestroy(s);
  if (r) return r;
  if (e != cudaSuccess) return cuda_fail(e, "chain bench");
  *avg_ms = total / reps;
  return 0;
}

int stf_bench_kernel(int kind, int64_t M, int64_t N, int64_t K, int reps, double* avg_ms) {
  g_err.clear();
  if (kind == 4 && M >= 1 && reps >= 1 && avg_ms) {
    int dev = 0;
    cudaGetDevice(&dev);
    int r = ensure_kernel_attrs(dev);
    return r ? r : bench_chain(M, reps, avg_ms);
  }
  if (kind < 0 || kind > 3 || M < 1 || reps < 1 || !avg_ms) return fail(-4, "bad stf_bench_kernel arguments");
  if (kind == 1 || kind == 3) N = M;
  if (kind == 2) K = N;
  if (kind == 3) K = M;
  if (N < 1 || K < 1) return fail(-4, "bad sizes");
  const int64_t ldm = M + (M & 1), ldn = N + (N & 1);
  int dev = 0;
  cudaGetDevice(&dev);
  int r = ensure_kernel_attrs(dev);
  if (r) return r;
  double *A = nullptr, *B = nullptr, *Cm = nullptr, *Src = nullptr;
  unsigned long long* info = nullptr;
  cudaStream_t s = nullptr;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  double total = 0;
  cudaError_t e = cudaSuccess;
  auto step = [&](cudaError_t x) {
    if (e == cudaSuccess) e = x;
  };
  const int64_t trsm = ctx().opt.trsm, dataflow = ctx().opt.dataflow;
  step(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  step(cudaEventCreate(&e0));
  step(cudaEventCreate(&e1));
  step(cudaMalloc(&A, (size_t)(ldm * K) * 8));
  step(cudaMalloc(&B, (size_t)(ldn * std::max(K, N)) * 8));
  step(cudaMalloc(&Cm, (size_t)(ldm * N) * 8));
  step(cudaMalloc(&Src, (size_t)(ldm * N) * 8));
  step(cudaMalloc(&info, sizeof *info));
  int* ws = nullptr;
  step(cudaMalloc(&ws, stfk::dataflow_ws_bytes((int)M, (int)N)));
  if (e == cudaSuccess) {
    // operands: SPD generator blocks (well scaled); L for TRSM = the lower part of an SPD block is fine
    step(stfk::fill_spd(s, A, ldm, M + K, 0, 0, (int)M, (int)K, 11));
    step(stfk::fill_spd(s, B, ldn, std::max(N, K), 0, 0, (int)N, (int)std::max(K, N), 12));
    step(stfk::fill_spd(s, Src, ldm, M, 0, 0, (int)M, (int)N, 13));
    step(cudaMemcpyAsync(Cm, Src, (size_t)(ldm * N) * 8, cudaMemcpyDeviceToDevice, s));
    step(stfk::info_reset(s, info));
    for (int it = 0; it < reps + 1 && e == cudaSuccess; ++it) {  // first launch = warm-up
      if (kind == 3 || kind == 2) step(cudaMemcpyAsync(Cm, Src, (size_t)(ldm * N) * 8, cudaMemcpyDeviceToDevice, s));
      step(cudaEventRecord(e0, s));
      switch (kind) {
        case 0: step(stfk::gemm_nt(s, 0, (int)M, (int)N, (int)K, A, ldm, B, ldn, Cm, ldm, 0)); break;
        case 1: step(stfk::gemm_nt(s, 0, (int)M, (int)M, (int)K, A, ldm, A, ldm, Cm, ldm, 1)); break;
        case 2:
          step(trsm == 3 && stfk::trsm_res_supported((int)N, Src, ldm)
                   ? stfk::trsm_res_parts(s, 0, (int)M, (int)N, Src, ldm, Cm, ldm, nullptr, (int)ctx().opt.trsm_res_split)
               : trsm >= 2 ? stfk::trsm_panel(s, 0, (int)M, (int)N, Src, ldm, Cm, ldm)
               : trsm == 1 ? stfk::trsm_tile(s, 0, (int)M, (int)N, Src, ldm, Cm, ldm, ws)
                           : stfk::trsm_rlt(s, 0, (int)M, (int)N, Src, ldm, Cm, ldm));
          break;
        case 3:
          step(dataflow ? stfk::potrf_tile(s, 0, (int)M, Cm, ldm, 0, info, ws, nullptr, nullptr,
                                           (int)ctx().opt.potrf_ctas, -1, nullptr, (int)ctx().opt.potrf_split)
                        : stfk::potrf_lower(s, 0, (int)M, Cm, ldm, 0, info));
          break;
      }
      step(cudaEventRecord(e1, s));
      step(cudaEventSynchronize(e1));
      float ms = 0;
      step(cudaEventElapsedTime(&ms, e0, e1));
      if (it > 0) total += ms;
    }
  }
  cudaFree(A);
  cudaFree(B);
  cudaFree(Cm);
  cudaFree(Src);
  cudaFree(info);
  cudaFree(ws);
  if (e0) cudaEventDestroy(e0);
  if (e1) cudaEventDestroy(e1);
  if (s) cudaStreamDestroy(s);
  if (e != cudaSuccess) return cuda_fail(e, "stf_bench_kernel");
  *avg_ms = total / reps;
  return 0;
}

int64_t stf_debug_last_trace(int64_t* out, int64_t cap_tasks) {
  Context& C = ctx();
  std::lock_guard<std::mutex> g(C.mu);
  const int64_t n = (int64_t)C.last_trace.size() / 7;
  if (out) std::copy(C.last_trace.begin(), C.last_trace.begin() + 7 * std::min(n, std::max<int64_t>(cap_tasks, 0)), out);
  return n;
}

int64_t stf_debug_potrf_trace(int64_t n, double* A, int64_t lda, int ctas, int64_t* trace, int64_t cap) {
  g_err.clear();
  int dev = 0;
  cudaGetDevice(&dev);
  int r = ensure_kernel_attrs(dev);
  if (r) return r;
  const int Nb = (int)((n + 63) / 64);
  const int64_t slots = 6 * Nb + 3 * (int64_t)Nb * Nb * Nb;  // >= 6 T + 3 * tasks
  unsigned long long *d_info = nullptr, *d_tr = nullptr;
  int* ws = nullptr;
  cudaError_t e = cudaMalloc(&d_info, sizeof *d_info);
  if (e == cudaSuccess) e = cudaMalloc(&d_tr, (size_t)slots * 8);
  if (e == cudaSuccess) e = cudaMemset(d_tr, 0, (size_t)slots * 8);
  if (e == cudaSuccess) e = cudaMalloc(&ws, stfk::dataflow_ws_bytes((int)n, (int)n));
  if (e == cudaSuccess) e = stfk::dataflow_prepare((int)n, (int)n, true);
  if (e == cudaSuccess) e = stfk::info_reset(0, d_info);
  if (e == cudaSuccess)
    e = stfk::potrf_tile(0, 0, (int)n, A, lda, 0, d_info, ws, nullptr, d_tr, ctas > 0 ? ctas : (int)ctx().opt.potrf_ctas,
                         -1, nullptr, (int)ctx().opt.potrf_split);
  if (e == cudaSuccess) e = cudaStreamSynchronize(0);
  const int64_t cnt = std::min<int64_t>(cap, slots);
  if (e == cudaSuccess && trace) e = cudaMemcpy(trace, d_tr, (size_t)cnt * 8, cudaMemcpyDeviceToHost);
  cudaFree(d_info);
  cudaFree(d_tr);
  cudaFree(ws);
  if (e != cudaSuccess) return cuda_fail(e, "potrf trace");
  return cnt;
}

int64_t stf_debug_trsm_trace(int64_t M, int64_t n, const double* L, int64_t ldl, double* B, int64_t ldb,
                             int64_t* trace, int64_t cap) {
  g_err.clear();
  if (M < 1 || !stfk::trsm_res_supported((int)n, L, ldl)) return fail(-4, "unsupported TRSM trace shape");
  int dev = 0;
  cudaGetDevice(&dev);
  int r = ensure_kernel_attrs(dev);
  if (r) return r;
  const int64_t slots = 6 * (n / 64);
  unsigned long long* d_tr = nullptr;
  cudaError_t e = cudaMalloc(&d_tr, (size_t)slots * 8);
  if (e == cudaSuccess) e = cudaMemset(d_tr, 0, (size_t)slots * 8);
  if (e == cudaSuccess) e = stfk::trsm_res(0, 0, (int)M, (int)n, L, ldl, B, ldb, nullptr, d_tr);
  if (e == cudaSuccess) e = cudaStreamSynchronize(0);
  const int64_t cnt = std::min<int64_t>(cap, slots);
  if (e == cudaSuccess && trace) e = cudaMemcpy(trace, d_tr, (size_t)cnt * 8, cudaMemcpyDeviceToHost);
  cudaFree(d_tr);
  if (e != cudaSuccess) return cuda_fail(e, "trsm trace");
  return cnt;
}

}  // extern "C"
