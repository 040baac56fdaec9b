// Lowering of an STF plan (plan.cpp) onto the device: buffers, CUDA streams and
// events (eager backend) or one CUDA graph per call
// configuration (graph backend), memoised across calls.
// See runtime_internal.hpp for the paper mechanisms this unit realises.
#include <algorithm>
#include <chrono>
#include <climits>
#include <cstdio>
#include <cstdlib>
#include <thread>

#include <nvtx3/nvToolsExt.h>

#include "runtime_internal.hpp"

namespace stfrt {

Exec::~Exec() {
  for (void* p : ipc_opened) cudaIpcCloseMemHandle(p);
  if (gexec) cudaGraphExecDestroy(gexec);
  if (graph) cudaGraphDestroy(graph);
  for (size_t t = 0; t < events.size(); ++t)
    if (events[t]) {
      cudaSetDevice(events_dev[t]);
      cudaEventDestroy(events[t]);
    }
  for (auto& ev : trace)
    if (ev) cudaEventDestroy(ev);
  for (auto& a : allocs) {
    cudaSetDevice(a.first);
    cudaFree(a.second);
  }
}

int ensure_kernel_attrs(int dev) {
  static std::mutex m;
  static std::vector<int> done;
  std::lock_guard<std::mutex> g(m);
  if (std::find(done.begin(), done.end(), dev) != done.end()) return 0;
  cudaError_t e = stfk::kernels_init(dev);
  if (e != cudaSuccess) return cuda_fail(e, "kernel attributes");
  done.push_back(dev);
  return 0;
}

bool device_of(const void* ptr, int* dev) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, ptr) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  if (a.type != cudaMemoryTypeDevice && a.type != cudaMemoryTypeManaged) return false;
  *dev = a.device;
  return true;
}

// page-locked (or registered) host memory: capturable async copies
bool host_pinned(const void* ptr) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, ptr) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeHost;
}

stf::PlanOptions call_plan_options(const Options& o, int64_t n, int64_t nb, int kind, int P, int Q, int nslots,
                                   int sms) {
  const int64_t T = n / nb;
  const bool colmajor = kind != STF_DESC_TILED_2DBC;
  stf::PlanOptions po;
  po.P = P;
  po.Q = Q;
  po.nslots = nslots;
  po.bulk_streams = (int)std::max<int64_t>(1, o.streams);
  po.crit_streams = kCritStreams;
  po.copy_streams = kCopyStreams;
  po.serial = o.serial != 0;
  po.stream_pool = (int)o.stream_pool;
  po.priority = o.priority != 0;
  po.prio_mode = (int)o.prio_mode;
  po.with_load = colmajor;
  po.with_store = colmajor;
  po.order_asap = o.order_asap != 0;
  po.lookahead = o.lookahead != 0;
  po.ooc_reorder = o.ooc_reorder != 0;
  po.dev_order = (int)o.dev_order;
  po.push = o.push != 0 && o.trsm >= 2;
  po.push_potrf = po.push && o.dataflow != 0;  // the dataflow POTRF kernel stores into replicas
  po.data_plane = po.push ? (int)o.push : 0;
  // merged tile updates need whole k tiles of 32 per operand pair (gemm_nt_multi)
  po.gemm_merge = (nb % 32 == 0) ? (int)o.gemm_merge : 0;
  // 4 updates per merged task on long factorisations (n = 65536, T = 64: +0.97% over none, +0.3%
  // over 2), 2 on shorter ones (n = 32768, T = 32: +0.47% vs +0.23% with 4;
  // profiles/r02/gemm_merge_sweep.txt)
  po.gemm_group = o.gemm_group > 0 ? (int)o.gemm_group : (T >= 48 ? 4 : 2);
  po.ooc_order = (int)o.ooc_order;
  // Scheduling model of the submission order (plan.cpp reorder_list), in units of
  // one nb^3 GEMM task's duration while `width` of them share the GPU: a tile
  // update has nb^2 / 8192 CTAs of 128 x 64 at 2 per SM, so about
  // width = SMs * 16384 / nb^2 run at once (2 at nb = 1024, 9 at nb = 512); a
  // PCIe tile copy (nb^2 * 8 B at ~54 GB/s) against 2 nb^3 flop at ~35 TFLOP/s per
  // width: copy_cost = 2592 / (width * nb) units; device copies ~free.
  po.sched_width = (int)o.sched_width;
  if (po.sched_width <= 0) po.sched_width = (int)std::min<int64_t>(64, std::max<int64_t>(1, (int64_t)sms * 16384 / (nb * nb)));
  po.copy_cost = kind == STF_DESC_HOST_COLMAJOR ? 2592.0 / ((double)po.sched_width * (double)nb) : 0.02;
  // Submission order (profiles/r01/submission_order.txt): with tiles of order
  // >= 512 the plan is re-submitted in simulated list-scheduling order - the panel
  // chain ahead of the bulk updates of its step, the transfers of a COLMAJOR call
  // next to the tasks that need them - for COLMAJOR calls (HOST n = 32768: 396 ->
  // 358 ms; n = 16384, nb = 512: 67 -> 58 ms) and for device tiles when T <= 16,
  // where the chain bounds the time (n = 8192: POTRF(1) starts 1.3 ms earlier,
  // nb = 512 +12%, nb = 1024 +2%; n = 16384, nb = 1024 +2%).  Device tiles with
  // T > 16 re-order only the last 8 panel steps, where the chain bounds the time
  // again (n = 32768: +0.2%; all steps: -0.3%; n = 65536 +-0).  nb = 256 keeps
  // program order (-12%).
  po.order_mode = o.order_mode >= 0 ? (int)o.order_mode : (nb >= 512 ? 2 : 0);
  po.order_tail = o.order_tail >= 0 ? o.order_tail : ((!colmajor && T > 16) ? 8 : 0);
  po.ooc_budget_pct = o.ooc_budget_pct > 0 ? (int)o.ooc_budget_pct : 60;
  if (kind == STF_DESC_HOST_COLMAJOR && nslots == 1 && o.mem_cap_tiles > 0 && o.mem_cap_tiles < T * (T + 1) / 2) {
    po.frames = o.mem_cap_tiles;  // NEXT-4: out-of-core plan over this many device frames
    // with three quarters of the tiles resident or more, wide blocks (90%) keep the
    // right-looking concurrency; below, eviction pressure favours 60% (n = 32768,
    // nb = 1024: F = 450 / 396 +2.1% / +2.0% at 90%, F = 264 -6%)
    if (o.ooc_budget_pct < 0 && 4 * po.frames >= 3 * (T * (T + 1) / 2)) po.ooc_budget_pct = 90;
  } else if (kind == STF_DESC_HOST_COLMAJOR && nslots == 1 && po.order_mode == 2 && po.ooc_reorder && o.host_stream &&
             o.lookahead && !o.serial && !o.stream_pool && T >= 16) {
    // T = 8 (n = 8192, nb = 1024): -1.5%, T = 16 +0.2%, T = 32 +2.7..5%.
    // In-core host call through the out-of-core builder with a frame per tile: its
    // 2D-blocked left-looking order consumes the tiles in the order they arrive
    // over PCIe; nothing is evicted, so a block may fill most of the frames
    // (n = 32768, nb = 1024: right-looking plan 357.6 ms, block budget 60% 352.7 ms,
    // 75..99% 345.8 ms; one block of all tiles would be the right-looking order).
    // lookahead = 0 (fence ablation), serial and the reduced stream pools keep the
    // right-looking builder, which implements them.
    po.frames = T * (T + 1) / 2;
    po.ooc_budget_pct = (int)o.host_stream_budget_pct;
  }
  return po;
}

// the node the capture of stream s would hang the next launch on (null when not capturing
// or when that is not exactly one node)
cudaGraphNode_t capture_last_node(cudaStream_t s) {
  cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
  const cudaGraphNode_t* deps = nullptr;
  size_t nd = 0;
  if (cudaStreamGetCaptureInfo_v3(s, &st, nullptr, nullptr, &deps, nullptr, &nd) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return (st == cudaStreamCaptureStatusActive && nd == 1) ? deps[0] : nullptr;
}
// Turn the capture edge from kernel node `from` (a current dependency of stream s)
// into a programmatic one: the next kernel captured on s may launch once every CTA
// of `from` has executed griddepcontrol.launch_dependents (or exited).  The other
// dependencies keep full-completion edges.  No-op (0) when `from` is not a
// dependency; 1 when the edge was converted; negative on error.
int capture_make_programmatic(cudaStream_t s, cudaGraphNode_t from) {
  cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
  const cudaGraphNode_t* deps = nullptr;
  const cudaGraphEdgeData* ed = nullptr;
  size_t nd = 0;
  CUDA_TRY(cudaStreamGetCaptureInfo_v3(s, &st, nullptr, nullptr, &deps, &ed, &nd), "capture info");
  if (st != cudaStreamCaptureStatusActive) return 0;
  std::vector<cudaGraphNode_t> d(deps, deps + nd);
  std::vector<cudaGraphEdgeData> e(nd);
  bool found = false;
  for (size_t i = 0; i < nd; ++i) {
    e[i] = ed ? ed[i] : cudaGraphEdgeData{};
    if (d[i] == from) {
      e[i].from_port = cudaGraphKernelNodePortProgrammatic;
      e[i].type = cudaGraphDependencyTypeProgrammatic;
      found = true;
    }
  }
  if (!found) return 0;
  CUDA_TRY(cudaStreamUpdateCaptureDependencies_v2(s, d.data(), e.data(), nd, cudaStreamSetCaptureDependencies),
           "programmatic capture edge");
  return 1;  // converted
}

// Remove node `from` from the current capture dependencies of stream s (no-op when absent).
int capture_drop_dependency(cudaStream_t s, cudaGraphNode_t from) {
  cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
  const cudaGraphNode_t* deps = nullptr;
  const cudaGraphEdgeData* ed = nullptr;
  size_t nd = 0;
  CUDA_TRY(cudaStreamGetCaptureInfo_v3(s, &st, nullptr, nullptr, &deps, &ed, &nd), "capture info");
  if (st != cudaStreamCaptureStatusActive) return 0;
  std::vector<cudaGraphNode_t> d;
  std::vector<cudaGraphEdgeData> e;
  for (size_t i = 0; i < nd; ++i)
    if (deps[i] != from) {
      d.push_back(deps[i]);
      e.push_back(ed ? ed[i] : cudaGraphEdgeData{});
    }
  if (d.size() == nd) return 0;
  CUDA_TRY(cudaStreamUpdateCaptureDependencies_v2(s, d.data(), e.data(), d.size(), cudaStreamSetCaptureDependencies),
           "capture drop edge");
  return 0;
}

// 64-block steps before its end at which a chain kernel releases its dependent (option
// pdl_lead; -1: nb / 128, at least 2 -- the chain step alone: lead 8 best at nb = 1024,
// 4 at nb = 512, profiles/r02/pdl_and_tail.txt)
int64_t pdl_lead_of(int64_t opt, int64_t nb) { return opt >= 0 ? opt : std::max<int64_t>(2, nb / 128); }

// ------------------------------------------------------------------ lowering
namespace {

struct Lowerer {
  Context& C;
  Exec& X;
  int cur_dev = -1;

  void set_dev(int d) {
    if (d != cur_dev) {
      cudaSetDevice(d);
      cur_dev = d;
    }
  }
  cudaStream_t stream_of(const stf::Task& t) { return C.slots[(size_t)t.slot].streams[(size_t)t.stream]; }
  // level 5 -> the device's greatest priority, each level below one step lower (clamped)
  int prio_of(const stf::Task& t) {
    int lo = 0, hi = 0;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);
    if (!X.opt.priority) return lo;
    const int v = hi + (5 - t.prio);
    return v > lo ? lo : v;
  }

  // replica destinations of a pushing task: each replica, or the multicast address of the tile
  stfk::Mirrors mirrors_of(const stf::Task& t) const {
    stfk::Mirrors mir{};
    if (t.nmir <= 0) return mir;
    if (X.mcs && X.mc_off[(size_t)t.out] >= 0) {
      mir.p[0] = reinterpret_cast<double*>(X.mcs->mcva) + X.mc_off[(size_t)t.out];
      mir.n = 1;
      mir.mc = 1;
      return mir;
    }
    for (int m = 0; m < t.nmir && m < 7; ++m) mir.p[m] = X.buf[(size_t)t.mir[m]];
    mir.n = t.nmir < 7 ? t.nmir : 7;
    return mir;
  }

  static cudaError_t trace_record(cudaEvent_t ev, cudaStream_t s) {
    cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
    cudaStreamIsCapturing(s, &st);
    return st == cudaStreamCaptureStatusActive ? cudaEventRecordWithFlags(ev, s, cudaEventRecordExternal)
                                               : cudaEventRecord(ev, s);
  }

  int body(const stf::Task& t, size_t tidx, cudaStream_t s, int prio) {
    const int64_t nb = X.nb;
    const uint64_t skip = (uint64_t)X.opt.debug_skip;
    if (skip & (1u << t.kind)) return 0;  // debug what-if timing only (results invalid)
    int* ws = X.task_ws.empty() ? nullptr : X.task_ws[tidx];
    const size_t tile_bytes = (size_t)(nb * nb) * sizeof(double);
    Slot& S = C.slots[(size_t)t.slot];
    switch (t.kind) {
      case stf::K_POTRF:
        if (X.opt.dataflow) {
          stfk::Mirrors mir = mirrors_of(t);  // fused push of L_kk (NEXT-3): final blocks also into the replicas
          // pdl: the chain CTA releases the dependent TRSM(k+1,k) pdl_lead 64-block steps before its end
          const int nbk = (int)((nb + 63) / 64);
          const int trig = X.opt.pdl ? (int)std::max<int64_t>(0, nbk - pdl_lead_of(X.opt.pdl_lead, nb)) : -1;
          cudaGraphNode_t chain = nullptr;
          CUDA_TRY(stfk::potrf_tile(s, prio, (int)nb, X.buf[(size_t)t.out], nb, (int64_t)t.k * nb, S.d_info, ws, &mir,
                                    nullptr, (int)X.opt.potrf_ctas, trig, &chain, (int)X.opt.potrf_split),
                   "POTRF launch");
          if (!X.cap_node.empty()) X.cap_node[tidx] = capture_last_node(s);  // the block-task launch
          if (chain) {
            // two launches (chain, then block tasks released by it): whatever follows on this
            // stream, and the successors waiting on its event, depend on both
            if (!X.cap_node2.empty()) X.cap_node2[tidx] = chain;
            CUDA_TRY(cudaStreamUpdateCaptureDependencies(s, &chain, 1, cudaStreamAddCaptureDependencies),
                     "POTRF join");
          }
        } else
          CUDA_TRY(stfk::potrf_lower(s, prio, (int)nb, X.buf[(size_t)t.out], nb, (int64_t)t.k * nb, S.d_info),
                   "POTRF launch");
        return 0;
      case stf::K_TRSM: {
        stfk::Mirrors mir = mirrors_of(t);
        if ((skip & (3u << 16)) && t.i != t.k + 1) {  // debug what-if: non-critical TRSM costed as a GEMM
          const int kk = (skip & (1u << 17)) ? (int)(nb / 2) : (int)nb;  // (half: triangular-GEMM flops)
          CUDA_TRY(stfk::gemm_nt(s, prio, (int)nb, (int)nb, kk, X.buf[(size_t)t.out], nb, X.buf[(size_t)t.in[0]],
                                 nb, X.buf[(size_t)t.out], nb, 0),
                   "TRSM what-if");
          return 0;
        }
        if (X.opt.pdl && X.opt.trsm == 3 && t.i == t.k + 1 &&
            stfk::trsm_res_supported((int)nb, X.buf[(size_t)t.in[0]], nb)) {
          // pdl: TRSM(k+1,k) in one resident-panel launch that reads the blocks of L_kk as
          // the dataflow POTRF(k) publishes them; captured behind POTRF(k) on the same
          // stream, the edge between the two becomes programmatic (the TRSM launches when
          // the POTRF triggers).  Without a same-stream POTRF(k) (another slot, eager
          // backend) L_kk is complete at launch and the flags are already final.
          const int64_t src = X.pdl_src.empty() ? -1 : X.pdl_src[tidx];
          const int nbk = (int)(nb / 64);
          const int* pflag = src >= 0 && X.task_ws[(size_t)src] ? X.task_ws[(size_t)src] + 2 : nullptr;
          if (pflag && !X.cap_node.empty() && X.cap_node[(size_t)src]) {
            // one programmatic edge, from the POTRF's last launch (a node with several
            // programmatic edges is not launched early: profiles/r02/pdl_and_tail.txt); the
            // chain launch of a two-launch POTRF is its ancestor through that edge, and the
            // TRSM reads L_kk through the progress flags, so its edge is dropped here
            if (X.cap_node2[(size_t)src]) {
              int r = capture_drop_dependency(s, X.cap_node2[(size_t)src]);
              if (r) return r;
            }
            int r = capture_make_programmatic(s, X.cap_node[(size_t)src]);
            if (r < 0) return r;
            X.pdl_edges += r;
          }
          // column-block counters for a SYRK(k+1,k) that overlaps this TRSM in turn
          int* kflag = pflag ? X.task_ws[(size_t)src] + 2 + nbk * nbk : nullptr;
          const int trig = kflag ? std::max(0, nbk - (int)pdl_lead_of(X.opt.pdl_lead, nb)) : -1;
          CUDA_TRY(stfk::trsm_res(s, prio, (int)nb, (int)nb, X.buf[(size_t)t.in[0]], nb, X.buf[(size_t)t.out], nb, &mir,
                                  nullptr, pflag, nbk, kflag, trig),
                   "TRSM launch");
          if (!X.cap_node.empty()) X.cap_node[tidx] = capture_last_node(s);
        } else if (X.opt.trsm == 3 &&
                   (t.i == t.k + 1 ||
                    X.n - t.k * nb <= (X.opt.trsm_res_tail >= 0 ? X.opt.trsm_res_tail : (nb >= 1024 ? 4096 : 8192))) &&
                   stfk::trsm_res_supported((int)nb, X.buf[(size_t)t.in[0]], nb)) {
          // the next panel's TRSM(k+1,k) is on the critical path, and near the end of the
          // factorisation every TRSM is latency-bound: the resident-panel kernel (16 rows per
          // CTA, 4x the CTAs of the row panel, solve overlapped with the updates)
          CUDA_TRY(stfk::trsm_res_parts(s, prio, (int)nb, (int)nb, X.buf[(size_t)t.in[0]], nb, X.buf[(size_t)t.out], nb,
                                        &mir, (int)X.opt.trsm_res_split),
                   "TRSM launch");
        } else if (X.opt.trsm >= 2 && t.i == t.k + 1) {
          // the next panel's TRSM(k+1,k) is on the critical path: one low-latency launch
          CUDA_TRY(stfk::trsm_panel(s, prio, (int)nb, (int)nb, X.buf[(size_t)t.in[0]], nb, X.buf[(size_t)t.out], nb, 32,
                                    &mir),
                   "TRSM launch");
        } else if (X.opt.trsm >= 2 && X.opt.trsm_split > 1 && nb % (64 * X.opt.trsm_split) == 0) {
          // Right-looking over `parts` column blocks of width w:
          //   X_p = B_p L_pp^-T (row-panel kernel);  B_{>p} -= X_p L_{>p,p}^T (full-rate GEMM kernel).
          // Only 1/parts of the TRSM flops stay in the substitution kernel (SM-time matters here,
          // not latency; the critical TRSM(k+1,k) takes the single-launch branch above).
          const int64_t parts = X.opt.trsm_split, w = nb / parts;
          const double* L = X.buf[(size_t)t.in[0]];
          double* B = X.buf[(size_t)t.out];
          for (int64_t pp = 0; pp < parts; ++pp) {
            stfk::Mirrors mp = mir;
            for (int m = 0; m < mp.n; ++m) mp.p[m] = mir.p[m] + pp * w * nb;
            CUDA_TRY(stfk::trsm_panel(s, prio, (int)nb, (int)w, L + pp * w * nb + pp * w, nb, B + pp * w * nb, nb,
                                      (int)X.opt.trsm_rows, &mp),
                     "TRSM launch");
            if (pp + 1 < parts)
              CUDA_TRY(stfk::gemm_nt(s, prio, (int)nb, (int)(nb - (pp + 1) * w), (int)w, B + pp * w * nb, nb,
                                     L + pp * w * nb + (pp + 1) * w, nb, B + (pp + 1) * w * nb, nb, 0),
                       "TRSM GEMM");
          }
        } else if (X.opt.trsm >= 2) {
          CUDA_TRY(stfk::trsm_panel(s, prio, (int)nb, (int)nb, X.buf[(size_t)t.in[0]], nb, X.buf[(size_t)t.out], nb,
                                    (int)X.opt.trsm_rows, &mir),
                   "TRSM launch");
        } else if (X.opt.trsm == 1)
          CUDA_TRY(stfk::trsm_tile(s, prio, (int)nb, (int)nb, X.buf[(size_t)t.in[0]], nb, X.buf[(size_t)t.out], nb, ws),
                   "TRSM launch");
        else
          CUDA_TRY(stfk::trsm_rlt(s, prio, (int)nb, (int)nb, X.buf[(size_t)t.in[0]], nb, X.buf[(size_t)t.out], nb),
                   "TRSM launch");
        return 0;
      }
      case stf::K_SYRK: {
        // pdl: SYRK(k+1,k) behind its overlapping TRSM(k+1,k) on the same stream reads
        // the k columns of L_{k+1,k} as the TRSM's CTAs publish them (programmatic edge)
        const int64_t src = X.pdl_src.empty() ? -1 : X.pdl_src[tidx];
        const int* kflag = nullptr;
        if (src >= 0) {
          const int nbk = (int)(nb / 64);
          kflag = X.task_ws[(size_t)X.pdl_src[(size_t)src]] + 2 + nbk * nbk;
          if (!X.cap_node.empty() && X.cap_node[(size_t)src]) {
            int r = capture_make_programmatic(s, X.cap_node[(size_t)src]);
            if (r < 0) return r;
            X.pdl_edges += r;
          }
        }
        const double* A = X.buf[(size_t)t.in[0]];
        CUDA_TRY(stfk::gemm_nt_multi(s, prio, (int)nb, (int)nb, (int)nb, 1, &A, nb, &A, nb, X.buf[(size_t)t.out], nb, 1,
                                     0, kflag, kflag ? (int)((nb + stfk::kTrsmResRows - 1) / stfk::kTrsmResRows) : 0),
                 "SYRK launch");
        return 0;
      }
      case stf::K_GEMM:
        if (t.nupd > 1) {  // merged GEMM(i,j,k) .. GEMM(i,j,k+nupd-1): one k sweep of nupd nb
          const double* As[4];
          const double* Bs[4];
          As[0] = X.buf[(size_t)t.in[0]];
          Bs[0] = X.buf[(size_t)t.in[1]];
          for (int u = 1; u < t.nupd; ++u) {
            As[u] = X.buf[(size_t)t.xin[2 * (u - 1)]];
            Bs[u] = X.buf[(size_t)t.xin[2 * (u - 1) + 1]];
          }
          CUDA_TRY(stfk::gemm_nt_multi(s, prio, (int)nb, (int)nb, (int)nb, t.nupd, As, nb, Bs, nb, X.buf[(size_t)t.out], nb,
                                       0, 0),
                   "GEMM launch");
        }
        else
          CUDA_TRY(stfk::gemm_nt(s, prio, (int)nb, (int)nb, (int)nb, X.buf[(size_t)t.in[0]], nb, X.buf[(size_t)t.in[1]],
                                 nb, X.buf[(size_t)t.out], nb, 0),
                   "GEMM launch");
        return 0;
      case stf::K_COPY:
        // Push of a finished tile into a consumer slot's replica on the producer's
        // copy stream (copy engine, no SMs).  One call for every slot pair: with
        // unified addressing and peer access enabled (stf_cholesky_init), a
        // cudaMemcpyDefault copy between two devices is a peer copy over NVLink,
        // between virtual slots of one device a device-to-device copy, and in both
        // cases a memcpy node when captured (cudaMemcpyPeerAsync is not
        // capturable: the capture falls back to eager).
        CUDA_TRY(cudaMemcpyAsync(X.buf[(size_t)t.out], X.buf[(size_t)t.in[0]], tile_bytes, cudaMemcpyDefault, s),
                 "replica copy");
        return 0;
      case stf::K_FENCE:
        return 0;  // ordering only: its waits (and event record) are the whole task
      case stf::K_LOAD:
      case stf::K_STORE: {
        const bool load = t.kind == stf::K_LOAD;
        double* tile = X.buf[(size_t)(load ? t.out : t.in[0])];
        const int64_t i = t.i, j = t.j;
        const bool upper = (X.uplo == 'U');
        // block of the caller matrix holding tile (i,j) of L: (i,j) for 'L', (j,i) transposed for 'U'
        double* blk = upper ? X.mat + (j * nb) + (i * nb) * X.ld : X.mat + (i * nb) + (j * nb) * X.ld;
        if (!upper) {
          if (load)
            CUDA_TRY(cudaMemcpy2DAsync(tile, nb * 8, blk, X.ld * 8, nb * 8, nb, cudaMemcpyDefault, s), "load tile");
          else
            CUDA_TRY(cudaMemcpy2DAsync(blk, X.ld * 8, tile, nb * 8, nb * 8, nb, cudaMemcpyDefault, s), "store tile");
          return 0;
        }
        const size_t scr_idx = (size_t)t.slot * kCopyStreams + (size_t)(t.stream % kCopyStreams);
        if (X.mat_dev >= 0 && X.mat_dev == S.device) {
          if (load)
            CUDA_TRY(stfk::transpose_copy(s, tile, nb, blk, X.ld, (int)nb, (int)nb), "load transpose");
          else
            CUDA_TRY(stfk::transpose_copy(s, blk, X.ld, tile, nb, (int)nb, (int)nb), "store transpose");
          return 0;
        }
        double* scr = X.scratch[scr_idx];
        if (load) {
          CUDA_TRY(cudaMemcpy2DAsync(scr, nb * 8, blk, X.ld * 8, nb * 8, nb, cudaMemcpyDefault, s), "load stage");
          CUDA_TRY(stfk::transpose_copy(s, tile, nb, scr, nb, (int)nb, (int)nb), "load transpose");
        } else {
          CUDA_TRY(stfk::transpose_copy(s, scr, nb, tile, nb, (int)nb, (int)nb), "store transpose");
          CUDA_TRY(cudaMemcpy2DAsync(blk, X.ld * 8, scr, nb * 8, nb * 8, nb, cudaMemcpyDefault, s), "store stage");
        }
        return 0;
      }
    }
    return fail(-101, "unknown task kind %d", t.kind);
  }

  // Enqueue every task in plan order.  Assumes all pool streams are ready
  // (forked from the origin when capturing).
  int issue() {
    const stf::Plan& P = X.plan;
    const int64_t launches0 = stfk::launch_count();
    // info reset on each slot's first stream
    for (size_t s = 0; s < C.slots.size() && s < (size_t)X.ngpus; ++s) {
      if (X.mp && (int)s != C.mp_me) continue;
      set_dev(C.slots[s].device);
      CUDA_TRY(stfk::info_reset(C.slots[s].streams[0], C.slots[s].d_info), "info reset");
    }
    // info reset must precede POTRFs on other streams of the slot: make every
    // stream of the slot wait for it
    for (size_t s = 0; s < C.slots.size() && s < (size_t)X.ngpus; ++s) {
      if (X.mp && (int)s != C.mp_me) continue;
      Slot& S = C.slots[s];
      set_dev(S.device);
      cudaEvent_t ev = C.fork_join[s * S.streams.size()];
      CUDA_TRY(cudaEventRecord(ev, S.streams[0]), "record info event");
      for (size_t k = 1; k < S.streams.size(); ++k) CUDA_TRY(cudaStreamWaitEvent(S.streams[k], ev, 0), "wait info event");
    }
    const int nt = (X.opt.graph || X.opt.threads <= 1) ? 1 : (int)std::min<int64_t>(X.opt.threads, X.ngpus);
    int r = 0;
    if (nt == 1) {
      r = issue_range(0, 1, nullptr);
    } else {
      // Multi-threaded eager submission (A26): thread w issues the
      // tasks of slots s with s % nt == w, in plan order.  A cross-thread
      // predecessor's event may be waited on only after its record was issued,
      // so each thread spins on the producer's `recorded` flag first; a thread
      // only ever waits on tasks earlier in plan order, so this cannot deadlock.
      std::unique_ptr<std::atomic<uint8_t>[]> recorded(new std::atomic<uint8_t>[P.tasks.size()]);
      for (size_t t = 0; t < P.tasks.size(); ++t) recorded[t].store(0, std::memory_order_relaxed);
      std::vector<int> rc((size_t)nt, 0);
      std::vector<std::string> err((size_t)nt);
      std::vector<std::thread> th;
      for (int w = 0; w < nt; ++w)
        th.emplace_back([&, w] {
          Lowerer L{C, X};
          rc[(size_t)w] = L.issue_range(w, nt, recorded.get());
          if (rc[(size_t)w]) {
            err[(size_t)w] = g_err;
            for (size_t t = 0; t < P.tasks.size(); ++t) recorded[t].store(1, std::memory_order_release);  // unblock peers
          }
        });
      for (auto& x : th) x.join();
      for (int w = 0; w < nt && !r; ++w)
        if (rc[(size_t)w]) {
          r = rc[(size_t)w];
          g_err = err[(size_t)w];
        }
    }
    if (r) return r;
    X.launches = stfk::launch_count() - launches0;
    return 0;
  }

  // Issue the tasks of the slots owned by submission thread w of nt (all tasks
  // when nt == 1) in plan order.
  int issue_range(int w, int nt, std::atomic<uint8_t>* recorded) {
    const stf::Plan& P = X.plan;
    for (size_t t = 0; t < P.tasks.size(); ++t) {
      const stf::Task& task = P.tasks[t];
      if (X.mp && task.slot != C.mp_me) continue;  // another process runs it
      if (task.slot % nt != w) continue;
      set_dev(C.slots[(size_t)task.slot].device);
      cudaStream_t s = stream_of(task);
      if (X.mp) {
        // inputs that are replicas here were written by another process: wait
        // (on the device, no host round trip) for the producer's flag
        // (every operand: in[] and, for a merged GEMM, the further pairs xin[])
        for (int a = 0; a < 2 + 2 * (task.nupd - 1); ++a) {
          const int64_t b = a < 2 ? task.in[a] : task.xin[a - 2];
          if (b >= 0 && P.buffers[(size_t)b].replica && task.kind != stf::K_COPY) {
            const CUresult cr = g_wait_value32((CUstream)s, (CUdeviceptr)(X.local_flags + X.flag_idx[(size_t)b]),
                                               X.epoch, CU_STREAM_WAIT_VALUE_GEQ);
            if (cr != CUDA_SUCCESS) return fail(-101, "cuStreamWaitValue32 failed (%d)", (int)cr);
          }
        }
      }
      for (const int64_t* q = P.graph.preds_begin((int64_t)t); q != P.graph.preds_end((int64_t)t); ++q) {
        const stf::Task& pt = P.tasks[(size_t)*q];
        if (pt.slot == task.slot && pt.stream == task.stream) continue;  // stream order suffices
        if (X.mp && pt.slot != C.mp_me) continue;  // cross-process: replica flags above
        if (recorded && pt.slot % nt != w)
          while (!recorded[*q].load(std::memory_order_acquire)) std::this_thread::yield();
        CUDA_TRY(cudaStreamWaitEvent(s, X.events[(size_t)*q], 0), "stream wait event");
      }
      // debug timeline: timing events (external record nodes when captured), no SM work
      if (!X.trace.empty()) CUDA_TRY(trace_record(X.trace[2 * t], s), "trace");
      const bool nv = X.opt.nvtx && !X.opt.graph;  // one NVTX range per task submission (eager)
      if (nv) {
        static const char* kn[] = {"POTRF", "TRSM", "SYRK", "GEMM", "COPY", "LOAD", "STORE", "FENCE"};
        char name[64];
        snprintf(name, sizeof name, "%s(%d,%d,%d)@%d", kn[task.kind & 7], task.i, task.j, task.k, task.slot);
        nvtxRangePushA(name);
      }
      int r = body(task, t, s, prio_of(task));
      if (nv) nvtxRangePop();
      if (r) return r;
      if (!X.trace.empty()) CUDA_TRY(trace_record(X.trace[2 * t + 1], s), "trace");
      if (X.mp) {  // publish remote replicas written by this task (COPY target, fused-push mirrors)
        auto signal = [&](int64_t b) -> int {
          const int dst = P.buffers[(size_t)b].slot;
          const CUresult cr = g_write_value32((CUstream)s, (CUdeviceptr)(X.peer_flags[(size_t)dst] + X.flag_idx[(size_t)b]),
                                              X.epoch, CU_STREAM_WRITE_VALUE_DEFAULT);
          return cr == CUDA_SUCCESS ? 0 : fail(-101, "cuStreamWriteValue32 failed (%d)", (int)cr);
        };
        if (task.kind == stf::K_COPY && (r = signal(task.out))) return r;
        for (int m = 0; m < task.nmir; ++m)
          if ((r = signal(task.mir[m]))) return r;
      }
      if (X.events[t]) CUDA_TRY(cudaEventRecord(X.events[t], s), "event record");
      if (recorded) recorded[t].store(1, std::memory_order_release);
    }
    return 0;
  }
};

// slots this process issues work on
bool slot_active(const Context& C, const Exec& X, int s) { return !X.mp || s == C.mp_me; }

// fork all pool streams of the participating slots from `origin` / join them back
int fork_streams(Context& C, Exec& X) {
  cudaSetDevice(C.origin_dev);
  cudaEvent_t fork = C.fork_join.back();
  CUDA_TRY(cudaEventRecord(fork, C.origin), "fork record");
  for (int s = 0; s < X.ngpus; ++s) {
    if (!slot_active(C, X, s)) continue;
    Slot& S = C.slots[(size_t)s];
    cudaSetDevice(S.device);
    for (cudaStream_t st : S.streams) CUDA_TRY(cudaStreamWaitEvent(st, fork, 0), "fork wait");
  }
  return 0;
}

int join_streams(Context& C, Exec& X) {
  for (int s = 0; s < X.ngpus; ++s) {
    if (!slot_active(C, X, s)) continue;
    Slot& S = C.slots[(size_t)s];
    cudaSetDevice(S.device);
    for (size_t k = 0; k < S.streams.size(); ++k) {
      cudaEvent_t ev = C.fork_join[(size_t)s * S.streams.size() + k];
      CUDA_TRY(cudaEventRecord(ev, S.streams[k]), "join record");
      cudaSetDevice(C.origin_dev);
      CUDA_TRY(cudaStreamWaitEvent(C.origin, ev, 0), "join wait");
      cudaSetDevice(S.device);
    }
  }
  cudaSetDevice(C.origin_dev);
  return 0;
}

// Multi-process mode: once every local task is done (after the join), all of
// this process's replica flags have been consumed; clear them for the next
// run.  Producers cannot publish the next run's tiles before the caller's
// barrier that follows stf_mp_potrf, so one constant flag value serves every
// run and the whole run (waits, writes, reset) can live in one CUDA graph.
int mp_reset_flags(Context& C, Exec& X) {
  if (!X.mp || !X.local_flag_count) return 0;
  cudaSetDevice(C.origin_dev);
  CUDA_TRY(cudaMemsetAsync(X.local_flags, 0, X.local_flag_count * sizeof(uint32_t), C.origin), "flag reset");
  return 0;
}

// fork + every task + join (+ flag reset) on the current capture / eager streams
int issue_all(Context& C, Exec& X) {
  X.pdl_edges = 0;
  int r = fork_streams(C, X);
  Lowerer L{C, X};
  if (!r) r = L.issue();
  if (!r) r = join_streams(C, X);
  if (!r) r = mp_reset_flags(C, X);
  return r;
}

int alloc_on(Exec& X, int dev, size_t bytes, double** out) {
  cudaSetDevice(dev);
  void* p = nullptr;
  cudaError_t e = cudaMalloc(&p, bytes);
  if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc (plan workspace)");
  X.allocs.push_back({dev, p});
  *out = static_cast<double*>(p);
  return 0;
}

}  // namespace

// Capture the whole DAG.  A capture the driver rejects (e.g. a multi-device
// topology it cannot express) falls back to the eager stream backend for this
// plan: same tasks, same edges, same results; graph_fallback = 1 is reported
// in the call's statistics.
int capture_graph(Context& C, Exec& X) {
  cudaSetDevice(C.origin_dev);
  int r = 0;
  cudaGraph_t g = nullptr;
  cudaError_t e = cudaStreamBeginCapture(C.origin, cudaStreamCaptureModeThreadLocal);
  if (e == cudaSuccess) {
    r = issue_all(C, X);
    cudaSetDevice(C.origin_dev);
    e = cudaStreamEndCapture(C.origin, &g);
  }
  if (r == 0 && e == cudaSuccess && g) {
    e = cudaGraphInstantiateWithFlags(&X.gexec, g, cudaGraphInstantiateFlagUseNodePriority);
    if (e == cudaSuccess) {
      X.graph = g;
      size_t nn = 0;
      cudaGraphGetNodes(g, nullptr, &nn);
      X.graph_nodes = (int64_t)nn;
    }
  }
  if (!X.gexec) {
    if (g) cudaGraphDestroy(g);
    if (r == -103) return r;  // out of memory is not a capture problem
    if (getenv("STF_DEBUG_CAPTURE")) fprintf(stderr, "stf: graph capture failed (%s / %s), eager lowering\n",
                                             cudaGetErrorString(e), g_err.c_str());
    cudaGetLastError();
    for (int d : C.devices) {  // drain anything a partial capture may have left behind
      cudaSetDevice(d);
      cudaDeviceSynchronize();
    }
    cudaGetLastError();
    g_err.clear();
    X.opt.graph = 0;
    X.graph_fallback = 1;
  }
  return 0;
}

int prepare(Context& C, Exec& X, const stf_matrix_desc* desc) {
  auto t0 = std::chrono::steady_clock::now();
  const int64_t T = X.n / X.nb;
  const bool colmajor = X.kind != STF_DESC_TILED_2DBC;
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, C.slots[0].device);
  stf::PlanOptions po = call_plan_options(X.opt, X.n, X.nb, X.kind, X.P, X.Q, X.ngpus, sms);
  stf::build_plan(X.plan, T, po);
  const stf::Plan& P = X.plan;
  const size_t tile_bytes = (size_t)(X.nb * X.nb) * sizeof(double);
  X.buf.assign(P.buffers.size(), nullptr);
  {
    std::vector<int> devs;
    for (int s = 0; s < X.ngpus; ++s)
      if (std::find(devs.begin(), devs.end(), C.slots[(size_t)s].device) == devs.end())
        devs.push_back(C.slots[(size_t)s].device);
    X.ndevices = (int)devs.size();
    X.peer_transfers = 0;
    for (const stf::Task& t : P.tasks) {
      if (t.kind == stf::K_COPY)
        X.peer_transfers += C.slots[(size_t)t.slot].device != C.slots[(size_t)t.k].device;
      for (int m = 0; m < t.nmir; ++m)
        X.peer_transfers += C.slots[(size_t)t.slot].device != C.slots[(size_t)P.buffers[(size_t)t.mir[m]].slot].device;
    }
  }
  // home tiles
  if (!colmajor) {
    for (size_t b = 0; b < (size_t)P.ntiles(); ++b) {
      const stf::Buffer& B = P.buffers[b];
      X.buf[b] = desc->tiles[(size_t)B.i + (size_t)B.j * (size_t)T];
    }
  } else {
    X.mat = desc->ptr;
    X.ld = desc->ld;
    X.mat_dev = (X.kind == STF_DESC_DEVICE_COLMAJOR) ? desc->device : -1;
  }
  if (X.mp) {
    // offsets and flag slots of every replica, identical in every process (same plan)
    X.rep_off.assign(P.buffers.size(), 0);
    X.flag_idx.assign(P.buffers.size(), -1);
    std::vector<size_t> used((size_t)X.ngpus, 0);
    for (size_t b = 0; b < P.buffers.size(); ++b) {
      const stf::Buffer& B = P.buffers[b];
      if (!B.replica) continue;
      X.flag_idx[b] = (int)used[(size_t)B.slot];
      X.rep_off[b] = (used[(size_t)B.slot]++) * (size_t)(X.nb * X.nb);
    }
    const int me = C.mp_me;
    const size_t cnt = used[(size_t)me];
    X.local_flag_count = cnt;
    if (cnt) {
      double* arena = nullptr;
      int r = alloc_on(X, C.slots[(size_t)me].device, cnt * tile_bytes, &arena);
      if (r) return r;
      X.local_arena = arena;
      double* fl = nullptr;
      r = alloc_on(X, C.slots[(size_t)me].device, (cnt * sizeof(uint32_t) + 7) / 8 * 8, &fl);
      if (r) return r;
      X.local_flags = reinterpret_cast<uint32_t*>(fl);
      CUDA_TRY(cudaMemset(X.local_flags, 0, cnt * sizeof(uint32_t)), "flag init");
      for (size_t b = 0; b < P.buffers.size(); ++b)
        if (P.buffers[b].replica && P.buffers[b].slot == me) X.buf[b] = arena + X.rep_off[b];
    }
    X.peer_arena.assign((size_t)X.ngpus, nullptr);
    X.peer_flags.assign((size_t)X.ngpus, nullptr);
  }
  // push = 2: the pushed tiles' replicas in one NVSwitch multicast slab (mcast.cpp)
  X.data_plane = P.opt.push ? 1 : 0;
  auto in_slab = [&](const stf::Buffer& B) {
    return X.mcs && B.replica && X.mc_off[(size_t)stf::Plan::tile_id(B.i, B.j)] >= 0;
  };
  if (P.opt.push && X.opt.push == 2 && !X.mp && X.ngpus >= 2 && X.ndevices == X.ngpus) {
    std::vector<int> devs;
    for (int s = 0; s < X.ngpus; ++s) devs.push_back(C.slots[(size_t)s].device);
    std::string why;
    if (mc_supported(devs, &why)) {
      X.mc_off.assign((size_t)P.ntiles(), -1);
      int64_t cnt = 0;
      for (const stf::Task& t : P.tasks)
        if (t.nmir > 0 && X.mc_off[(size_t)t.out] < 0) X.mc_off[(size_t)t.out] = (cnt++) * X.nb * X.nb;
      std::unique_ptr<McSlab> S(new McSlab());
      const int r = mc_create(*S, devs, (size_t)cnt * tile_bytes, &why);
      if (r == 0) {
        X.mcs = std::move(S);
        X.data_plane = 2;
        for (size_t b = 0; b < P.buffers.size(); ++b)
          if (in_slab(P.buffers[b]))
            X.buf[b] = reinterpret_cast<double*>(X.mcs->uc[(size_t)P.buffers[b].slot]) +
                       X.mc_off[(size_t)stf::Plan::tile_id(P.buffers[b].i, P.buffers[b].j)];
      } else if (r == -103) {
        return fail(-103, "multicast slab: %s", why.c_str());
      }
    }
    if (!X.mcs && getenv("STF_DEBUG_MC")) fprintf(stderr, "stf: push=2 keeps peer stores: %s\n", why.c_str());
  }
  // library-owned storage: per slot one arena for (COLMAJOR) home tiles + replicas
  for (int s = 0; s < X.ngpus && !X.mp; ++s) {
    size_t count = 0;
    for (size_t b = 0; b < P.buffers.size(); ++b) {
      const stf::Buffer& B = P.buffers[b];
      if (B.slot == s && (B.replica || colmajor) && !in_slab(B)) count++;
    }
    const size_t nscr = (colmajor && X.uplo == 'U') ? kCopyStreams : 0;
    if (count + nscr == 0) continue;
    double* arena = nullptr;
    int r = alloc_on(X, C.slots[(size_t)s].device, (count + nscr) * tile_bytes, &arena);
    if (r) return r;
    size_t used = 0;
    for (size_t b = 0; b < P.buffers.size(); ++b) {
      const stf::Buffer& B = P.buffers[b];
      if (B.slot == s && (B.replica || colmajor) && !in_slab(B)) X.buf[b] = arena + (used++) * (size_t)(X.nb * X.nb);
    }
    if (nscr) {
      X.scratch.resize((size_t)X.ngpus * kCopyStreams, nullptr);
      for (size_t k = 0; k < nscr; ++k) X.scratch[(size_t)s * kCopyStreams + k] = arena + (used++) * (size_t)(X.nb * X.nb);
    }
  }
  // dataflow-kernel workspaces (one private block per POTRF/TRSM task) and task tables
  X.task_ws.assign(P.tasks.size(), nullptr);
  if (X.opt.dataflow || X.opt.trsm == 1) {
    const size_t wsb = stfk::dataflow_ws_bytes((int)X.nb, (int)X.nb);
    for (int s = 0; s < X.ngpus; ++s) {
      if (X.mp && s != C.mp_me) continue;
      size_t cnt = 0;
      for (const auto& t : P.tasks) cnt += (t.slot == s && (t.kind == stf::K_POTRF || t.kind == stf::K_TRSM));
      if (!cnt) continue;
      double* arena = nullptr;
      int r = alloc_on(X, C.slots[(size_t)s].device, cnt * wsb, &arena);
      if (r) return r;
      char* base = reinterpret_cast<char*>(arena);
      size_t used = 0;
      for (size_t t = 0; t < P.tasks.size(); ++t) {
        const stf::Task& tk = P.tasks[t];
        if (tk.slot == s && (tk.kind == stf::K_POTRF || tk.kind == stf::K_TRSM))
          X.task_ws[t] = reinterpret_cast<int*>(base + (used++) * wsb);
      }
      cudaSetDevice(C.slots[(size_t)s].device);
      CUDA_TRY(stfk::dataflow_prepare((int)X.nb, (int)X.nb, true), "dataflow tables");
      CUDA_TRY(stfk::dataflow_prepare((int)X.nb, (int)X.nb, false), "dataflow tables");
    }
  }
  // pdl: TRSM(k+1,k) that follows its POTRF(k) on the same slot and stream
  X.pdl_src.assign(P.tasks.size(), -1);
  X.cap_node.assign(X.opt.graph && X.opt.pdl ? P.tasks.size() : 0, nullptr);
  X.cap_node2.assign(X.cap_node.size(), nullptr);
  if (X.opt.pdl && X.opt.dataflow && X.opt.trsm == 3) {
    std::vector<int64_t> potrf_of((size_t)T, -1);
    for (size_t t = 0; t < P.tasks.size(); ++t)
      if (P.tasks[t].kind == stf::K_POTRF) potrf_of[(size_t)P.tasks[t].k] = (int64_t)t;
    std::vector<int64_t> trsm_of((size_t)T, -1);
    for (size_t t = 0; t < P.tasks.size(); ++t) {
      const stf::Task& a = P.tasks[t];
      if (a.kind != stf::K_TRSM || a.i != a.k + 1) continue;
      const int64_t src = potrf_of[(size_t)a.k];
      if (src >= 0 && P.tasks[(size_t)src].slot == a.slot && P.tasks[(size_t)src].stream == a.stream &&
          X.nb % 64 == 0 && X.nb <= 1024) {
        X.pdl_src[t] = src;
        trsm_of[(size_t)a.k] = (int64_t)t;
      }
    }
    // SYRK(k+1,k) that follows such a TRSM(k+1,k) on the same slot and stream
    for (size_t t = 0; t < P.tasks.size(); ++t) {
      const stf::Task& a = P.tasks[t];
      if (a.kind != stf::K_SYRK || a.i != a.k + 1) continue;
      const int64_t src = trsm_of[(size_t)a.k];
      if (src >= 0 && P.tasks[(size_t)src].slot == a.slot && P.tasks[(size_t)src].stream == a.stream)
        X.pdl_src[t] = src;
    }
  }
  if (X.opt.debug_trace && X.ngpus == 1 && !X.mp) {
    cudaSetDevice(C.slots[0].device);
    X.trace.assign(P.tasks.size() * 2, nullptr);
    for (auto& ev : X.trace) CUDA_TRY(cudaEventCreate(&ev), "trace event");
  }
  // events only where a successor runs on another stream
  std::vector<int64_t> soff, succ;
  P.graph.build_successors(soff, succ);
  X.events.assign(P.tasks.size(), nullptr);
  X.events_dev.assign(P.tasks.size(), 0);
  for (size_t t = 0; t < P.tasks.size(); ++t) {
    const stf::Task& a = P.tasks[t];
    if (X.mp && a.slot != C.mp_me) continue;  // never issued here
    bool need = false;
    for (int64_t e = soff[t]; e < soff[t + 1] && !need; ++e) {
      const stf::Task& b = P.tasks[(size_t)succ[(size_t)e]];
      need = !(b.slot == a.slot && b.stream == a.stream);
    }
    if (need) {
      const int dev = C.slots[(size_t)a.slot].device;
      cudaSetDevice(dev);
      CUDA_TRY(cudaEventCreateWithFlags(&X.events[t], cudaEventDisableTiming), "cudaEventCreate");
      X.events_dev[t] = dev;
    }
  }
  if (X.opt.graph && !X.mp) {  // multi-process: captured by stf_mp_import, once peer replicas are mapped
    int r = capture_graph(C, X);
    if (r) return r;
  }
  X.build_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return 0;
}

// Point an existing plan at new caller storage (same shape) and refresh its graph.
int rebind(Context& C, Exec& X, const stf_matrix_desc* desc, const std::vector<uintptr_t>& ptrs) {
  auto t0 = std::chrono::steady_clock::now();
  const int64_t T = X.n / X.nb;
  if (X.kind == STF_DESC_TILED_2DBC) {
    for (size_t b = 0; b < (size_t)X.plan.ntiles(); ++b) {
      const stf::Buffer& B = X.plan.buffers[b];
      X.buf[b] = desc->tiles[(size_t)B.i + (size_t)B.j * (size_t)T];
    }
  } else {
    X.mat = desc->ptr;
    X.ld = desc->ld;
    X.mat_dev = (X.kind == STF_DESC_DEVICE_COLMAJOR) ? desc->device : -1;
  }
  X.key_ptrs = ptrs;
  X.key_ld = desc->ld;
  X.key_dev = desc->device;
  if (X.gexec) {
    cudaSetDevice(C.origin_dev);
    CUDA_TRY(cudaStreamBeginCapture(C.origin, cudaStreamCaptureModeThreadLocal), "begin capture");
    int r = issue_all(C, X);
    cudaSetDevice(C.origin_dev);
    cudaGraph_t g = nullptr;
    cudaError_t e = cudaStreamEndCapture(C.origin, &g);
    if (r || e != cudaSuccess) {
      if (g) cudaGraphDestroy(g);
      return r ? r : cuda_fail(e, "re-capture");
    }
    cudaGraphExecUpdateResultInfo ri;
    if (cudaGraphExecUpdate(X.gexec, g, &ri) == cudaSuccess) {
      X.updates++;
    } else {
      cudaGetLastError();
      cudaGraphExecDestroy(X.gexec);
      X.gexec = nullptr;
      CUDA_TRY(cudaGraphInstantiateWithFlags(&X.gexec, g, cudaGraphInstantiateFlagUseNodePriority), "graph instantiate");
    }
    if (X.graph) cudaGraphDestroy(X.graph);
    X.graph = g;
  }
  X.build_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  X.rebound = true;
  return 0;
}

// One factorisation.  Ordering contract (include/stf_cholesky.h): the call
// starts after all work the caller enqueued before it on the legacy default
// stream and on the calling thread's per-thread default stream of every
// participating device (events recorded there are waited on by the launch
// stream), and returns after all of its own work has completed.
int run(Context& C, Exec& X) {
  for (size_t d = 0; d < C.devices.size(); ++d) {
    bool used = false;
    for (int s = 0; s < X.ngpus && !used; ++s)
      used = slot_active(C, X, s) && C.slots[(size_t)s].device == C.devices[d];
    if (!used) continue;
    cudaSetDevice(C.devices[d]);
    CUDA_TRY(cudaEventRecord(C.caller_ev[2 * d], cudaStreamLegacy), "caller legacy-stream event");
    CUDA_TRY(cudaEventRecord(C.caller_ev[2 * d + 1], cudaStreamPerThread), "caller per-thread-stream event");
    cudaSetDevice(C.origin_dev);
    CUDA_TRY(cudaStreamWaitEvent(C.origin, C.caller_ev[2 * d], 0), "wait caller work");
    CUDA_TRY(cudaStreamWaitEvent(C.origin, C.caller_ev[2 * d + 1], 0), "wait caller work");
  }
  cudaSetDevice(C.origin_dev);
  CUDA_TRY(cudaEventRecord(C.t_start, C.origin), "timing start");
  if (X.opt.nvtx) nvtxRangePushA(X.opt.graph ? "stf_potrf graph launch" : "stf_potrf eager submission");
  if (X.opt.graph) {
    const cudaError_t ge = cudaGraphLaunch(X.gexec, C.origin);
    if (X.opt.nvtx) nvtxRangePop();
    CUDA_TRY(ge, "graph launch");
  } else {
    int r = issue_all(C, X);
    if (X.opt.nvtx) nvtxRangePop();
    if (r) return r;
  }
  cudaSetDevice(C.origin_dev);
  CUDA_TRY(cudaEventRecord(C.t_end, C.origin), "timing end");
  CUDA_TRY(cudaStreamSynchronize(C.origin), "factorisation sync");
  float ms = 0.f;
  CUDA_TRY(cudaEventElapsedTime(&ms, C.t_start, C.t_end), "timing elapsed");
  C.device_ms = ms;
  // info = min over slots (0 if none failed)
  unsigned long long best = ULLONG_MAX;
  for (int s = 0; s < X.ngpus; ++s) {
    if (!slot_active(C, X, s)) continue;
    unsigned long long v = 0;
    cudaSetDevice(C.slots[(size_t)s].device);
    CUDA_TRY(cudaMemcpy(&v, C.slots[(size_t)s].d_info, sizeof v, cudaMemcpyDeviceToHost), "info readback");
    best = std::min(best, v);
  }
  cudaSetDevice(C.origin_dev);
  return best == ULLONG_MAX ? 0 : (int)std::min<unsigned long long>(best, INT_MAX);
}

void fill_plan_stats(const stf::Plan& P, int64_t nb, stf_plan_stats* s) {
  *s = stf_plan_stats{};
  int64_t compute = 0;
  for (const auto& t : P.tasks) compute += (t.kind <= stf::K_GEMM);
  s->tasks = compute;
  s->transfers = P.ntransfers + P.npushed;
  s->edges = P.graph.nedges();
  s->transfer_bytes = (P.ntransfers + P.npushed) * nb * nb * 8;
  s->critical_path = P.critical_path;
  s->dag_tasks = (int64_t)P.tasks.size();
  s->host_loads = P.nloads;
  s->host_stores = P.nstores;
  s->frames = P.opt.frames;
  s->pushed = P.npushed;
  int64_t mx = 0;
  for (int64_t r : P.replicas_per_slot) mx = std::max(mx, r);
  s->replicas_max = mx;
  s->data_plane = P.opt.data_plane;
  s->merged_gemms = P.nmerged;
}

void fill_stats(const Exec& X, bool hit, stf_plan_stats* s) {
  fill_plan_stats(X.plan, X.nb, s);
  s->pdl_edges = X.pdl_edges;
  s->graph_nodes = X.graph_nodes;
  s->kernel_launches = X.launches;
  s->build_ms = hit ? 0.0 : X.build_ms;
  s->graph_reuse = hit ? 1 : 0;
  s->graph_fallback = X.graph_fallback;
  s->graph = X.opt.graph ? 1 : 0;
  s->devices = X.ndevices;
  s->slots = X.ngpus;
  s->peer_transfers = X.peer_transfers;
  s->data_plane = X.data_plane;
}

}  // namespace stfrt
