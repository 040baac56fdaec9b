// Runtime: context, per-slot stream pools, lowering of the STF plan onto CUDA
// streams + events (eager) or into one CUDA graph per call configuration
// (memoised), and the C ABI of include/stf_cholesky.h.
//
// Paper mechanisms realised here:
//   A4  Algorithm 2 prologue: for each task, wait on the
//       events of its STF predecessors that ran on other streams (enforce_stf),
//       allocation is done once per plan (replica arenas), update = COPY tasks.
//   A8  stream pools per device.
//   A9  stream backend: ordering with cudaStreamWaitEvent.
//   A10 graph backend: the whole DAG of one stf_potrf call (one epoch,
//       PAPER.md:166-172) captured into a CUDA graph; multi-stream capture keeps
//       the DAG's concurrency, and per-node priorities keep the look-ahead.
//   A11 memoisation of executable graphs across calls, keyed by the call
//       configuration.
//   A12 abstract events: a task's completion is an event only when a successor
//       runs on another stream; in a graph these become plain edges.
//   A13 finalize: synchronous completion + write-back.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <climits>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <list>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <atomic>
#include <vector>

#include "../../include/stf_cholesky.h"
#include "kernels/tile_ops.hpp"
#include "plan.hpp"

namespace {

thread_local std::string g_err;
thread_local stf::Plan g_dag_plan;  // the plan of the last stf_dag_build (stf_dag_tasks_io)

int fail(int code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}

int cuda_fail(cudaError_t e, const char* what) {
  cudaGetLastError();  // clear sticky-free errors
  if (e == cudaErrorMemoryAllocation) return fail(-103, "%s: %s", what, cudaGetErrorString(e));
  return fail(-101, "%s: %s", what, cudaGetErrorString(e));
}

#define CUDA_TRY(expr, what)                 \
  do {                                       \
    cudaError_t e_ = (expr);                 \
    if (e_ != cudaSuccess) return cuda_fail(e_, what); \
  } while (0)

int64_t env_int(const char* name, int64_t dflt) {
  const char* v = getenv(name);
  if (!v || !*v) return dflt;
  return strtoll(v, nullptr, 10);
}

struct Slot {
  int device = 0;
  std::vector<cudaStream_t> streams;
  unsigned long long* d_info = nullptr;
};

struct Options {
  int64_t dataflow = 1;  // POTRF tile kernel: 1 single-launch dataflow, 0 recursive (GEMM-based)
  int64_t trsm = 3;      // TRSM tile kernel: 3 resident panel, 2 row-panel, 1 dataflow, 0 recursive
  int64_t trsm_split = 4;  // row panel: non-critical TRSMs as `trsm_split` column blocks (panel + GEMM updates)
  int64_t graph = 1;
  int64_t streams = 32;
  int64_t serial = 0;
  int64_t priority = 1;
  int64_t grid_p = 0;
  int64_t lookahead = 1;
  int64_t threads = 8;  // eager backend: host submission threads (one per slot group)
  int64_t push = 0;     // fused push of TRSM outputs into consumer replicas (row-panel TRSM only)
  int64_t mem_cap_tiles = 0;  // HOST_COLMAJOR on one GPU: device tile frames (0 = whole matrix resident)
  int64_t ooc_order = -1;     // out-of-core program order: 0 tall super-columns, 1 2D-blocked, -1 auto
  int64_t host_stream = 1;    // HOST_COLMAJOR on one GPU, nb >= 512: out-of-core builder with all tiles as frames
  int64_t trsm_res_tail = 8192;  // trsm 3: every TRSM(i,k) resident-panel once the trailing order n - k nb <= this
  int64_t trsm_rows = 128;  // row panel: rows per CTA of the non-critical TRSM panels (32, 64 or 128)
};

// options that change the plan or its lowering (part of the memo key)
bool same_plan_options(const Options& a, int64_t a_graph, const Options& b) {
  return a.streams == b.streams && a.serial == b.serial && a_graph == b.graph && a.priority == b.priority &&
         a.dataflow == b.dataflow && a.trsm == b.trsm && a.trsm_split == b.trsm_split && a.push == b.push &&
         a.lookahead == b.lookahead && a.mem_cap_tiles == b.mem_cap_tiles && a.ooc_order == b.ooc_order && a.host_stream == b.host_stream && a.trsm_res_tail == b.trsm_res_tail &&
         a.trsm_rows == b.trsm_rows;
}

// A plan bound to physical buffers, plus its lowering artefacts.
struct Exec {
  // key
  int64_t n = 0, nb = 0;
  char uplo = 'L';
  int kind = 0, ngpus = 0, P = 1, Q = 1;
  Options opt;
  std::vector<uintptr_t> key_ptrs;
  int64_t key_ld = 0;
  int key_dev = 0;
  int64_t key_graph = 1;  // graph option requested when the plan was built (opt.graph may fall back to 0)

  stf::Plan plan;
  std::vector<double*> buf;           // buffer id -> device pointer
  std::vector<std::pair<int, void*>> allocs;  // (device, ptr) library-owned
  std::vector<double*> scratch;       // per (slot, copy stream): staging tile for 'U'
  std::vector<int*> task_ws;          // per task: dataflow-kernel workspace (POTRF/TRSM), else null
  std::vector<cudaEvent_t> events;    // per task, null if not needed
  std::vector<int> events_dev;
  cudaGraph_t graph = nullptr;
  cudaGraphExec_t gexec = nullptr;
  int64_t graph_nodes = 0;
  int graph_fallback = 0;  // capture failed, eager lowering used
  unsigned skip_mask = 0;  // STF_DEBUG_SKIP: task kinds whose kernels are not launched (timing what-ifs)
  std::vector<cudaEvent_t> trace;  // STF_DEBUG_TRACE: per task timing events at start / end (one GPU slot)
  int64_t updates = 0;     // successful cudaGraphExecUpdate re-binds
  bool rebound = false;
  int64_t launches = 0;
  double build_ms = 0;
  // caller matrix for COLMAJOR kinds
  double* mat = nullptr;
  int64_t ld = 0;
  int mat_dev = -1;  // -1: host
  // multi-process mode (one process per slot): replicas of slot s live in slot s's
  // arena at rep_off[b]; their readiness is a 32-bit flag (index flag_idx[b]) in
  // slot s's flag array, written by the remote producer after the transfer.
  bool mp = false;
  std::vector<size_t> rep_off;        // per buffer id (replicas), element offset in its slot's arena
  std::vector<int> flag_idx;          // per buffer id (replicas), index in its slot's flag array
  double* local_arena = nullptr;      // this slot's replica arena (exported)
  uint32_t* local_flags = nullptr;    // this slot's flags (exported)
  size_t local_flag_count = 0;
  std::vector<double*> peer_arena;    // per slot, IPC-mapped (null for self / no replicas)
  std::vector<uint32_t*> peer_flags;  // per slot, IPC-mapped
  std::vector<void*> ipc_opened;      // to cudaIpcCloseMemHandle
  uint32_t epoch = 1;  // multi-process: value a published replica flag carries (reset to 0 at run end)

  ~Exec() {
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
};

struct Context {
  std::mutex mu;
  bool inited = false;
  std::vector<Slot> slots;
  std::vector<int> devices;  // distinct physical devices
  Options opt;
  std::list<std::unique_ptr<Exec>> cache;  // MRU first
  stf_plan_stats last{};
  std::vector<int64_t> last_trace;  // STF_DEBUG_TRACE: (kind, i, j, k, stream, t0_ns, t1_ns) per task
  cudaStream_t origin = nullptr;  // capture / launch stream on slot 0's device
  int origin_dev = 0;
  std::vector<cudaEvent_t> fork_join;  // per slot-stream, for fork/join around a call
  cudaEvent_t t_start = nullptr, t_end = nullptr;  // timing events on `origin`
  double device_ms = 0;
  int mp_me = -1;  // multi-process mode: the slot this process owns (-1: single-process mode)
  std::unique_ptr<Exec> mp_exec;  // multi-process mode: the current plan
};

// CUDA driver stream memory operations (flag hand-off between processes, no SMs)
typedef CUresult (*PFN_wv32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
PFN_wv32 g_write_value32 = nullptr, g_wait_value32 = nullptr;
bool load_memops() {
  if (g_write_value32 && g_wait_value32) return true;
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint("cuStreamWriteValue32", &p, cudaEnableDefault, &q) == cudaSuccess &&
      q == cudaDriverEntryPointSuccess)
    g_write_value32 = reinterpret_cast<PFN_wv32>(p);
  if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &p, cudaEnableDefault, &q) == cudaSuccess &&
      q == cudaDriverEntryPointSuccess)
    g_wait_value32 = reinterpret_cast<PFN_wv32>(p);
  return g_write_value32 && g_wait_value32;
}

Context& ctx() {
  static Context c;
  return c;
}

constexpr int kCritStreams = 6;  // 0: panel chain, 1: its feeders, 2..5: other urgent tasks by row
constexpr int kCopyStreams = 2;
constexpr size_t kCacheMax = 4;

stf::PlanOptions plan_options(const Options& o, int P, int Q, int nslots, bool load, bool store) {
  stf::PlanOptions po;
  po.P = P;
  po.Q = Q;
  po.nslots = nslots;
  po.bulk_streams = (int)std::max<int64_t>(1, o.streams);
  po.crit_streams = kCritStreams;
  po.copy_streams = kCopyStreams;
  po.serial = o.serial != 0;
  po.priority = o.priority != 0;
  po.prio_mode = (int)env_int("STF_PRIO_MODE", 0);
  po.with_load = load;
  po.with_store = store;
  // submission in order of earliest start for plans with host/device transfers
  // (STF_ORDER_ASAP: -1 auto = COLMAJOR calls, 0 never, 1 always)
  po.order_asap = env_int("STF_ORDER_ASAP", 0) != 0;
  po.order_mode = (int)std::max<int64_t>(0, env_int("STF_ORDER_MODE", 0));
  po.order_tail = std::max<int64_t>(0, env_int("STF_ORDER_TAIL", 0));
  po.sched_width = (int)std::max<int64_t>(0, env_int("STF_SCHED_WIDTH", 0));  // 0: from nb (prepare)
  po.lookahead = o.lookahead != 0;
  po.ooc_reorder = env_int("STF_OOC_REORDER", 1) != 0;
  po.dev_order = (int)env_int("STF_DEV_ORDER", 0);
  po.ooc_budget_pct = (int)std::min<int64_t>(95, std::max<int64_t>(10, env_int("STF_OOC_BUDGET_PCT", 60)));
  po.push = o.push != 0 && o.trsm >= 2;
  return po;
}

// ------------------------------------------------------------------ lowering
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

  static cudaError_t trace_record(cudaEvent_t ev, cudaStream_t s) {
    cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
    cudaStreamIsCapturing(s, &st);
    return st == cudaStreamCaptureStatusActive ? cudaEventRecordWithFlags(ev, s, cudaEventRecordExternal)
                                               : cudaEventRecord(ev, s);
  }

  int body(const stf::Task& t, size_t tidx, cudaStream_t s, int prio) {
    const int64_t nb = X.nb;
    if (X.skip_mask & (1u << t.kind)) return 0;  // debug what-if timing only (results invalid)
    int* ws = X.task_ws.empty() ? nullptr : X.task_ws[tidx];
    const size_t tile_bytes = (size_t)(nb * nb) * sizeof(double);
    Slot& S = C.slots[(size_t)t.slot];
    switch (t.kind) {
      case stf::K_POTRF:
        if (X.opt.dataflow)
          CUDA_TRY(stfk::potrf_tile(s, prio, (int)nb, X.buf[(size_t)t.out], nb, (int64_t)t.k * nb, S.d_info, ws),
                   "POTRF launch");
        else
          CUDA_TRY(stfk::potrf_lower(s, prio, (int)nb, X.buf[(size_t)t.out], nb, (int64_t)t.k * nb, S.d_info),
                   "POTRF launch");
        return 0;
      case stf::K_TRSM: {
        stfk::Mirrors mir{};
        for (int m = 0; m < t.nmir && m < 7; ++m) mir.p[m] = X.buf[(size_t)t.mir[m]];
        mir.n = t.nmir < 7 ? t.nmir : 7;
        if ((X.skip_mask & (3u << 16)) && t.i != t.k + 1) {  // debug what-if: non-critical TRSM costed as a GEMM
          const int kk = (X.skip_mask & (1u << 17)) ? (int)(nb / 2) : (int)nb;   // (half: triangular-GEMM flops)
          CUDA_TRY(stfk::gemm_nt(s, prio, (int)nb, (int)nb, kk, X.buf[(size_t)t.out], nb, X.buf[(size_t)t.in[0]],
                                 nb, X.buf[(size_t)t.out], nb, 0),
                   "TRSM what-if");
          return 0;
        }
        if (X.opt.trsm == 3 && (t.i == t.k + 1 || X.n - t.k * nb <= X.opt.trsm_res_tail) &&
            stfk::trsm_res_supported((int)nb, X.buf[(size_t)t.in[0]], nb)) {
          // the next panel's TRSM(k+1,k) is on the critical path, and near the end of the
          // factorisation every TRSM is latency-bound: the resident-panel kernel (16 rows per
          // CTA, 4x the CTAs of the row panel, solve overlapped with the updates)
          CUDA_TRY(stfk::trsm_res(s, prio, (int)nb, (int)nb, X.buf[(size_t)t.in[0]], nb, X.buf[(size_t)t.out], nb, &mir),
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
      case stf::K_SYRK:
        CUDA_TRY(stfk::gemm_nt(s, prio, (int)nb, (int)nb, (int)nb, X.buf[(size_t)t.in[0]], nb, X.buf[(size_t)t.in[0]],
                               nb, X.buf[(size_t)t.out], nb, 1),
                 "SYRK launch");
        return 0;
      case stf::K_GEMM:
        CUDA_TRY(stfk::gemm_nt(s, prio, (int)nb, (int)nb, (int)nb, X.buf[(size_t)t.in[0]], nb, X.buf[(size_t)t.in[1]],
                               nb, X.buf[(size_t)t.out], nb, 0),
                 "GEMM launch");
        return 0;
      case stf::K_COPY: {
        const int dst_dev = C.slots[(size_t)t.k].device, src_dev = S.device;
        if (dst_dev == src_dev)
          CUDA_TRY(cudaMemcpyAsync(X.buf[(size_t)t.out], X.buf[(size_t)t.in[0]], tile_bytes, cudaMemcpyDeviceToDevice, s),
                   "replica copy");
        else
          CUDA_TRY(cudaMemcpyPeerAsync(X.buf[(size_t)t.out], dst_dev, X.buf[(size_t)t.in[0]], src_dev, tile_bytes, s),
                   "replica peer copy");
        return 0;
      }
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

  // Enqueue every task in program order.  Assumes all pool streams are ready
  // (forked from the origin when capturing).
  int issue() {
    const stf::Plan& P = X.plan;
    const int64_t launches0 = stfk::launch_count();
    // info reset on each slot's first stream
    for (size_t s = 0; s < C.slots.size() && s < (size_t)X.ngpus; ++s) {
      set_dev(C.slots[s].device);
      CUDA_TRY(stfk::info_reset(C.slots[s].streams[0], C.slots[s].d_info), "info reset");
    }
    // info reset must precede POTRFs on other streams of the slot: make every
    // stream of the slot wait for it
    for (size_t s = 0; s < C.slots.size() && s < (size_t)X.ngpus; ++s) {
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
      // tasks of slots s with s % nt == w, in program order.  A cross-thread
      // predecessor's event may be waited on only after its record was issued,
      // so each thread spins on the producer's `recorded` flag first; a thread
      // only ever waits on tasks earlier in program order, so this cannot deadlock.
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
  // when nt == 1) in program order.
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
        for (int a = 0; a < 2; ++a) {
          const int64_t b = task.in[a];
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
      int r = body(task, t, s, prio_of(task));
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

// fork all pool streams of the first ngpus slots from `origin` / join them back
int fork_streams(Context& C, int ngpus) {
  cudaSetDevice(C.origin_dev);
  cudaEvent_t fork = C.fork_join.back();
  CUDA_TRY(cudaEventRecord(fork, C.origin), "fork record");
  for (int s = 0; s < ngpus; ++s) {
    Slot& S = C.slots[(size_t)s];
    cudaSetDevice(S.device);
    for (cudaStream_t st : S.streams) CUDA_TRY(cudaStreamWaitEvent(st, fork, 0), "fork wait");
  }
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

int join_streams(Context& C, int ngpus) {
  for (int s = 0; s < ngpus; ++s) {
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

int alloc_on(Exec& X, int dev, size_t bytes, double** out) {
  cudaSetDevice(dev);
  void* p = nullptr;
  cudaError_t e = cudaMalloc(&p, bytes);
  if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc (plan workspace)");
  X.allocs.push_back({dev, p});
  *out = static_cast<double*>(p);
  return 0;
}

// Build plan + buffers + events (+ graph) for X (key fields already set).
// Capture the whole DAG.  A capture the driver rejects (e.g. a multi-device
// topology it cannot express) falls back to the eager stream backend for this
// plan: same tasks, same edges, same results.
int capture_graph(Context& C, Exec& X) {
  cudaSetDevice(C.origin_dev);
  int r = 0;
  cudaGraph_t g = nullptr;
  cudaError_t e = cudaStreamBeginCapture(C.origin, cudaStreamCaptureModeThreadLocal);
  if (e == cudaSuccess) {
    r = fork_streams(C, X.ngpus);
    Lowerer L{C, X};
    if (!r) r = L.issue();
    if (!r) r = join_streams(C, X.ngpus);
    if (!r) r = mp_reset_flags(C, X);
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
  stf::PlanOptions po = plan_options(X.opt, X.P, X.Q, X.ngpus, colmajor, colmajor);
  // Scheduling model of the submission order (plan.cpp reorder_list), in units of
  // one nb^3 GEMM task's duration while `width` of them share the GPU: a tile
  // update has nb^2 / 8192 CTAs of 128 x 64 at 2 per SM, so about
  // width = SMs * 16384 / nb^2 run at once (2 at nb = 1024, 9 at nb = 512); a
  // PCIe tile copy (nb^2 * 8 B at ~54 GB/s) against 2 nb^3 flop at ~35 TFLOP/s per
  // width: copy_cost = 2592 / (width * nb) units; device copies ~free.
  {
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, C.slots[0].device);
    if (po.sched_width <= 0)
      po.sched_width = (int)std::min<int64_t>(64, std::max<int64_t>(1, (int64_t)sms * 16384 / (X.nb * X.nb)));
    po.copy_cost = X.kind == STF_DESC_HOST_COLMAJOR ? 2592.0 / ((double)po.sched_width * (double)X.nb) : 0.02;
  }
  // Submission order (profiles/r01/submission_order.txt): with tiles of order
  // >= 512 the plan is re-submitted in simulated list-scheduling order - the panel
  // chain ahead of the bulk updates of its step, the transfers of a COLMAJOR call
  // next to the tasks that need them - for COLMAJOR calls (HOST n = 32768: 396 ->
  // 358 ms; n = 16384, nb = 512: 67 -> 58 ms) and for device tiles when T <= 16,
  // where the chain bounds the time (n = 8192: POTRF(1) starts 1.3 ms earlier,
  // nb = 512 +12%, nb = 1024 +2%; n = 16384, nb = 1024 +2%).  Device tiles with
  // T > 16 re-order only the last 8 panel steps, where the chain bounds the time
  // again (n = 32768: +0.2%; all steps: -0.3%; n = 65536 +-0).  nb = 256 keeps
  // program order (-12%).  STF_ORDER_MODE / STF_ORDER_TAIL override (mode 0
  // program order, 2 list; tail 0 = all steps); STF_ORDER_ASAP=1 selects the
  // earliest-start order instead.
  if (env_int("STF_ORDER_MODE", -1) < 0) po.order_mode = X.nb >= 512 ? 2 : 0;
  if (env_int("STF_ORDER_TAIL", -1) < 0) po.order_tail = (!colmajor && T > 16) ? 8 : 0;

  if (X.kind == STF_DESC_HOST_COLMAJOR && X.ngpus == 1 && X.opt.mem_cap_tiles > 0 &&
      X.opt.mem_cap_tiles < T * (T + 1) / 2) {
    po.frames = X.opt.mem_cap_tiles;  // NEXT-4: out-of-core plan over this many device frames
    // with three quarters of the tiles resident or more, wide blocks (90%) keep the
    // right-looking concurrency; below, eviction pressure favours 60% (n = 32768,
    // nb = 1024: F = 450 / 396 +2.1% / +2.0% at 90%, F = 264 -6%)
    if (env_int("STF_OOC_BUDGET_PCT", -1) < 0 && 4 * po.frames >= 3 * (T * (T + 1) / 2)) po.ooc_budget_pct = 90;
  }
  else if (X.kind == STF_DESC_HOST_COLMAJOR && X.ngpus == 1 && po.order_mode == 2 && po.ooc_reorder &&
           X.opt.host_stream && T >= 16) {  // T = 8 (n = 8192, nb = 1024): -1.5%, T = 16 +0.2%, T = 32 +2.7..5%
    // in-core host call through the out-of-core builder with a frame per tile: its
    // 2D-blocked left-looking order consumes the tiles in the order they arrive
    // over PCIe; nothing is evicted, so a block may fill most of the frames
    // (n = 32768, nb = 1024: right-looking plan 357.6 ms, block budget 60% 352.7 ms,
    // 75..99% 345.8 ms; one block of all tiles would be the right-looking order)
    po.frames = T * (T + 1) / 2;
    po.ooc_budget_pct = (int)std::min<int64_t>(99, std::max<int64_t>(10, env_int("STF_HOST_STREAM_BUDGET_PCT", 90)));
  }
  po.ooc_order = (int)X.opt.ooc_order;
  stf::build_plan(X.plan, T, po);
  const stf::Plan& P = X.plan;
  const size_t tile_bytes = (size_t)(X.nb * X.nb) * sizeof(double);
  X.buf.assign(P.buffers.size(), nullptr);
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
  // library-owned storage: per slot one arena for (COLMAJOR) home tiles + replicas
  for (int s = 0; s < X.ngpus && !X.mp; ++s) {
    size_t count = 0;
    for (size_t b = 0; b < P.buffers.size(); ++b) {
      const stf::Buffer& B = P.buffers[b];
      if (B.slot == s && (B.replica || colmajor)) count++;
    }
    const size_t nscr = (colmajor && X.uplo == 'U') ? kCopyStreams : 0;
    if (count + nscr == 0) continue;
    double* arena = nullptr;
    int r = alloc_on(X, C.slots[(size_t)s].device, (count + nscr) * tile_bytes, &arena);
    if (r) return r;
    size_t used = 0;
    for (size_t b = 0; b < P.buffers.size(); ++b) {
      const stf::Buffer& B = P.buffers[b];
      if (B.slot == s && (B.replica || colmajor)) X.buf[b] = arena + (used++) * (size_t)(X.nb * X.nb);
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
  if (getenv("STF_DEBUG_TRACE") && atoi(getenv("STF_DEBUG_TRACE")) && X.ngpus == 1 && !X.mp) {
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
    int r = fork_streams(C, X.ngpus);
    Lowerer L{C, X};
    if (!r) r = L.issue();
    if (!r) r = join_streams(C, X.ngpus);
    if (!r) r = mp_reset_flags(C, X);
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

int run(Context& C, Exec& X) {
  cudaSetDevice(C.origin_dev);
  CUDA_TRY(cudaEventRecord(C.t_start, C.origin), "timing start");
  if (X.opt.graph) {
    CUDA_TRY(cudaGraphLaunch(X.gexec, C.origin), "graph launch");
  } else {
    int r = fork_streams(C, X.ngpus);
    Lowerer L{C, X};
    if (!r) r = L.issue();
    if (!r) r = join_streams(C, X.ngpus);
    if (!r) r = mp_reset_flags(C, X);
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
    unsigned long long v = 0;
    cudaSetDevice(C.slots[(size_t)s].device);
    CUDA_TRY(cudaMemcpy(&v, C.slots[(size_t)s].d_info, sizeof v, cudaMemcpyDeviceToHost), "info readback");
    best = std::min(best, v);
  }
  cudaSetDevice(C.origin_dev);
  return best == ULLONG_MAX ? 0 : (int)std::min<unsigned long long>(best, INT_MAX);
}

void fill_stats(const Exec& X, bool hit, stf_plan_stats* s) {
  const stf::Plan& P = X.plan;
  int64_t compute = 0;
  for (const auto& t : P.tasks) compute += (t.kind <= stf::K_GEMM);
  s->tasks = compute;
  s->transfers = P.ntransfers + P.npushed;
  s->edges = P.graph.nedges();
  s->transfer_bytes = (P.ntransfers + P.npushed) * X.nb * X.nb * 8;
  s->critical_path = P.critical_path;
  s->graph_nodes = X.graph_nodes;
  s->kernel_launches = X.launches;
  s->build_ms = hit ? 0.0 : X.build_ms;
  s->graph_reuse = hit ? 1 : 0;
  s->dag_tasks = (int64_t)P.tasks.size();
  s->host_loads = P.nloads;
  s->host_stores = P.nstores;
  s->frames = P.opt.frames;
}

int choose_grid(int ngpus, int64_t grid_p, int* P, int* Q) {
  if (grid_p > 0) {
    if (ngpus % grid_p) return -1;
    *P = (int)grid_p;
    *Q = ngpus / (int)grid_p;
    return 0;
  }
  int best = 1;
  for (int p = 1; p * p <= ngpus; ++p)
    if (ngpus % p == 0) best = p;
  *P = best;
  *Q = ngpus / best;
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

// HOST_COLMAJOR calls on pageable memory are lowered eagerly onto the streams
// (pageable copies cannot be captured); STF_HOST_EAGER=1 forces the eager
// lowering for pinned memory too.  The eager path's speed depends on how the
// driver maps the ~40 streams onto its hardware queues (measured 350 to 388 ms
// at n = 32768 for the same plan), the captured graph does not (357 ms).
bool host_eager(const Context& C, const stf_matrix_desc* d, int64_t n, int64_t nb, int ngpus) {
  (void)C; (void)n; (void)nb; (void)ngpus;
  if (d->kind != STF_DESC_HOST_COLMAJOR) return false;
  return !host_pinned(d->ptr) || env_int("STF_HOST_EAGER", 0) != 0;
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

}  // namespace

// ====================================================================== C ABI
extern "C" {

const char* stf_last_error(void) { return g_err.c_str(); }

int stf_cholesky_init(int ngpus, const int* device_ids) {
  Context& C = ctx();
  std::lock_guard<std::mutex> g(C.mu);
  g_err.clear();
  if (C.inited) return fail(-104, "stf_cholesky_init called twice without stf_finalize");
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    return fail(-101, "no CUDA device available (%s)", cudaGetErrorString(e));
  }
  if (ngpus < 1 || ngpus > 64) return fail(-5, "ngpus=%d out of range", ngpus);
  C.opt.graph = env_int("STF_GRAPH", 1);
  C.opt.dataflow = env_int("STF_DATAFLOW", 1);
  C.opt.trsm = env_int("STF_TRSM", 3);
  C.opt.trsm_split = env_int("STF_TRSM_SPLIT", 4);
  C.opt.trsm_res_tail = env_int("STF_TRSM_RES_TAIL", 8192);
  C.opt.trsm_rows = env_int("STF_TRSM_ROWS", 128);
  C.opt.push = env_int("STF_PUSH", 0);
  C.opt.mem_cap_tiles = env_int("STF_MEM_CAP_TILES", 0);
  C.opt.ooc_order = env_int("STF_OOC_ORDER", -1);
  C.opt.host_stream = env_int("STF_HOST_STREAM", 1);
  C.opt.streams = env_int("STF_STREAMS", 32);
  C.opt.serial = env_int("STF_SERIAL", 0);
  C.opt.lookahead = env_int("STF_LOOKAHEAD", 1);
  C.opt.threads = env_int("STF_THREADS", 8);
  C.opt.priority = env_int("STF_PRIO", 1);
  C.opt.grid_p = 0;
  if (const char* gs = getenv("STF_GRID")) C.opt.grid_p = atoi(gs);
  C.slots.assign((size_t)ngpus, Slot{});
  C.devices.clear();
  for (int s = 0; s < ngpus; ++s) {
    const int d = device_ids ? device_ids[s] : s;
    if (d < 0 || d >= ndev) {
      C.slots.clear();
      return fail(-5, "device id %d of slot %d out of range (have %d)", d, s, ndev);
    }
    C.slots[(size_t)s].device = d;
    if (std::find(C.devices.begin(), C.devices.end(), d) == C.devices.end()) C.devices.push_back(d);
  }
  // peer access between distinct devices
  for (int a : C.devices)
    for (int b : C.devices) {
      if (a == b) continue;
      int can = 0;
      cudaDeviceCanAccessPeer(&can, a, b);
      if (can) {
        cudaSetDevice(a);
        cudaError_t pe = cudaDeviceEnablePeerAccess(b, 0);
        if (pe != cudaSuccess && pe != cudaErrorPeerAccessAlreadyEnabled) {
          cudaGetLastError();
          return cuda_fail(pe, "enable peer access");
        }
        cudaGetLastError();
      }
    }
  for (int d : C.devices) {
    int r = ensure_kernel_attrs(d);
    if (r) return r;
  }
  // stream pools: sized for the largest configuration (crit + bulk + copy)
  const int nstreams = kCritStreams + (int)std::max<int64_t>(1, C.opt.streams) + kCopyStreams;
  int lo = 0, hi = 0;
  for (auto& S : C.slots) {
    cudaSetDevice(S.device);
    cudaDeviceGetStreamPriorityRange(&lo, &hi);
    S.streams.resize((size_t)nstreams);
    for (int k = 0; k < nstreams; ++k) {
      const int pr = (k < kCritStreams) ? hi : lo;
      CUDA_TRY(cudaStreamCreateWithPriority(&S.streams[(size_t)k], cudaStreamNonBlocking, pr), "stream create");
    }
    CUDA_TRY(cudaMalloc(&S.d_info, sizeof(unsigned long long)), "info alloc");
  }
  C.origin_dev = C.slots[0].device;
  cudaSetDevice(C.origin_dev);
  CUDA_TRY(cudaStreamCreateWithFlags(&C.origin, cudaStreamNonBlocking), "origin stream");
  C.fork_join.assign((size_t)ngpus * (size_t)nstreams + 1, nullptr);
  for (size_t k = 0; k < C.fork_join.size(); ++k) {
    const int dev = (k + 1 == C.fork_join.size()) ? C.origin_dev : C.slots[k / (size_t)nstreams].device;
    cudaSetDevice(dev);
    CUDA_TRY(cudaEventCreateWithFlags(&C.fork_join[k], cudaEventDisableTiming), "fork/join event");
  }
  cudaSetDevice(C.origin_dev);
  CUDA_TRY(cudaEventCreate(&C.t_start), "timing event");
  CUDA_TRY(cudaEventCreate(&C.t_end), "timing event");
  C.inited = true;
  return 0;
}

static void release_all(Context& C) {
  C.cache.clear();
  C.mp_exec.reset();
  C.mp_me = -1;
  for (size_t k = 0; k < C.fork_join.size(); ++k)
    if (C.fork_join[k]) cudaEventDestroy(C.fork_join[k]);
  C.fork_join.clear();
  for (auto& S : C.slots) {
    cudaSetDevice(S.device);
    for (auto st : S.streams) cudaStreamDestroy(st);
    if (S.d_info) cudaFree(S.d_info);
  }
  C.slots.clear();
  if (C.t_start) cudaEventDestroy(C.t_start);
  if (C.t_end) cudaEventDestroy(C.t_end);
  C.t_start = C.t_end = nullptr;
  if (C.origin) {
    cudaSetDevice(C.origin_dev);
    cudaStreamDestroy(C.origin);
    C.origin = nullptr;
  }
  C.inited = false;
}

int stf_finalize(void) {
  Context& C = ctx();
  std::lock_guard<std::mutex> g(C.mu);
  g_err.clear();
  if (!C.inited) return fail(-100, "stf_finalize: library not initialised");
  for (int d : C.devices) {
    cudaSetDevice(d);
    cudaDeviceSynchronize();
  }
  release_all(C);
  return 0;
}

int stf_set_option(const char* name, int64_t value) {
  Context& C = ctx();
  std::lock_guard<std::mutex> g(C.mu);
  g_err.clear();
  if (!name) return fail(-105, "option name is NULL");
  std::string n(name);
  if (n == "graph") C.opt.graph = value != 0;
  else if (n == "dataflow") C.opt.dataflow = value != 0;
  else if (n == "trsm") {
    if (value < 0 || value > 3)
      return fail(-105, "trsm must be 0 (recursive), 1 (dataflow), 2 (row panel) or 3 (resident panel)");
    C.opt.trsm = value;
  }
  else if (n == "streams") {
    if (value < 1 || value > 64) return fail(-105, "streams must be in [1, 64]");
    const int have = C.inited ? (int)C.slots[0].streams.size() - kCritStreams - kCopyStreams : 64;
    if (value > have) return fail(-105, "streams=%lld exceeds the pool created at init (%d)", (long long)value, have);
    C.opt.streams = value;
  } else if (n == "serial") C.opt.serial = value != 0;
  else if (n == "lookahead") C.opt.lookahead = value != 0;
  else if (n == "trsm_split") {
    if (value < 1 || value > 16) return fail(-105, "trsm_split must be in [1, 16]");
    C.opt.trsm_split = value;
  }
  else if (n == "trsm_res_tail") {
    if (value < 0) return fail(-105, "trsm_res_tail must be >= 0");
    C.opt.trsm_res_tail = value;
  }
  else if (n == "trsm_rows") {
    if (value != 32 && value != 64 && value != 128) return fail(-105, "trsm_rows must be 32, 64 or 128");
    C.opt.trsm_rows = value;
  }
  else if (n == "push") C.opt.push = value != 0;
  else if (n == "mem_cap_tiles") {
    if (value != 0 && value < 3) return fail(-105, "mem_cap_tiles must be 0 (no cap) or >= 3 (a GEMM holds 3 tiles)");
    C.opt.mem_cap_tiles = value;
  }
  else if (n == "ooc_order") {
    if (value < -1 || value > 1)
      return fail(-105, "ooc_order must be -1 (auto), 0 (tall super-columns) or 1 (2D-blocked)");
    C.opt.ooc_order = value;
  }
  else if (n == "host_stream") C.opt.host_stream = value != 0;
  else if (n == "threads") {
    if (value < 1 || value > 64) return fail(-105, "threads must be in [1, 64]");
    C.opt.threads = value;
  }
  else if (n == "priority") C.opt.priority = value != 0;
  else if (n == "grid_p") {
    if (value < 0) return fail(-105, "grid_p must be >= 0");
    C.opt.grid_p = value;
  } else return fail(-105, "unknown option '%s'", name);
  return 0;
}

int stf_get_option(const char* name, int64_t* value) {
  Context& C = ctx();
  std::lock_guard<std::mutex> g(C.mu);
  g_err.clear();
  if (!name || !value) return fail(-105, "NULL argument");
  std::string n(name);
  if (n == "graph") *value = C.opt.graph;
  else if (n == "dataflow") *value = C.opt.dataflow;
  else if (n == "trsm") *value = C.opt.trsm;
  else if (n == "streams") *value = C.opt.streams;
  else if (n == "serial") *value = C.opt.serial;
  else if (n == "lookahead") *value = C.opt.lookahead;
  else if (n == "trsm_split") *value = C.opt.trsm_split;
  else if (n == "trsm_res_tail") *value = C.opt.trsm_res_tail;
  else if (n == "trsm_rows") *value = C.opt.trsm_rows;
  else if (n == "push") *value = C.opt.push;
  else if (n == "mem_cap_tiles") *value = C.opt.mem_cap_tiles;
  else if (n == "ooc_order") *value = C.opt.ooc_order;
  else if (n == "host_stream") *value = C.opt.host_stream;
  else if (n == "threads") *value = C.opt.threads;
  else if (n == "priority") *value = C.opt.priority;
  else if (n == "grid_p") *value = C.opt.grid_p;
  else return fail(-105, "unknown option '%s'", name);
  return 0;
}

int stf_potrf(int64_t n, int64_t nb, char uplo, stf_matrix_desc* A_desc, int ngpus) {
  Context& C = ctx();
  std::lock_guard<std::mutex> g(C.mu);
  g_err.clear();
  // argument checks first (LAPACK order), then runtime state
  if (n < 0) return fail(-1, "n=%lld < 0", (long long)n);
  if (nb < 2 || (nb & 1) || (n > 0 && n % nb != 0) || nb > 16384)
    return fail(-2, "nb=%lld must be even, >= 2, <= 16384 and divide n=%lld", (long long)nb, (long long)n);
  const char up = (uplo == 'l') ? 'L' : (uplo == 'u') ? 'U' : uplo;
  if (up != 'L' && up != 'U') return fail(-3, "uplo='%c' must be 'L' or 'U'", uplo);
  if (!A_desc) return fail(-4, "A_desc is NULL");
  if (A_desc->kind != STF_DESC_TILED_2DBC && A_desc->kind != STF_DESC_DEVICE_COLMAJOR &&
      A_desc->kind != STF_DESC_HOST_COLMAJOR)
    return fail(-4, "unknown descriptor kind %d", A_desc->kind);
  if (A_desc->kind == STF_DESC_TILED_2DBC && up != 'L') return fail(-3, "uplo='U' requires a COLMAJOR descriptor");
  if (A_desc->kind != STF_DESC_TILED_2DBC) {
    if (!A_desc->ptr && n > 0) return fail(-4, "descriptor ptr is NULL");
    if (A_desc->ld < std::max<int64_t>(1, n)) return fail(-4, "ld=%lld < max(1,n)", (long long)A_desc->ld);
  } else {
    if (!A_desc->tiles && n > 0) return fail(-4, "descriptor tiles table is NULL");
    if (A_desc->p < 1 || A_desc->q < 1 || (int64_t)A_desc->p * A_desc->q != ngpus)
      return fail(-4, "grid %dx%d does not match ngpus=%d", A_desc->p, A_desc->q, ngpus);
  }
  if (ngpus < 1) return fail(-5, "ngpus=%d < 1", ngpus);
  if (!C.inited) return fail(-100, "stf_potrf: call stf_cholesky_init first");
  if (ngpus > (int)C.slots.size()) return fail(-5, "ngpus=%d exceeds the %zu initialised slots", ngpus, C.slots.size());
  if (n == 0) return 0;

  int P = A_desc->p, Q = A_desc->q;
  if (A_desc->kind != STF_DESC_TILED_2DBC) {
    if (choose_grid(ngpus, C.opt.grid_p, &P, &Q)) return fail(-4, "grid_p does not divide ngpus");
    if (A_desc->kind == STF_DESC_DEVICE_COLMAJOR) {
      int d = -1;
      if (!device_of(A_desc->ptr, &d) || d != A_desc->device)
        return fail(-4, "DEVICE_COLMAJOR ptr is not device memory of device %d", A_desc->device);
    }
  }
  const int64_t T = n / nb;
  if (A_desc->kind == STF_DESC_HOST_COLMAJOR && ngpus > 1 && C.opt.mem_cap_tiles > 0)
    return fail(-105, "mem_cap_tiles (out-of-core) supports HOST_COLMAJOR calls on one GPU");
  // tile residency check (TILED_2DBC): every lower tile on its owner's device
  std::vector<uintptr_t> ptrs;
  if (A_desc->kind == STF_DESC_TILED_2DBC) {
    ptrs.reserve((size_t)(T * (T + 1) / 2));
    for (int64_t j = 0; j < T; ++j)
      for (int64_t i = j; i < T; ++i) {
        const double* tp = A_desc->tiles[(size_t)(i + j * T)];
        const int own = (int)((i % P) * Q + (j % Q));
        int d = -1;
        if (!tp || !device_of(tp, &d) || d != C.slots[(size_t)own].device)
          return fail(-4, "tile (%lld,%lld) is not device memory on slot %d (device %d)", (long long)i, (long long)j,
                      own, C.slots[(size_t)own].device);
        if (reinterpret_cast<uintptr_t>(tp) & 15) return fail(-4, "tile (%lld,%lld) not 16-byte aligned", (long long)i, (long long)j);
        ptrs.push_back(reinterpret_cast<uintptr_t>(tp));
      }
  }
  // memo lookup
  Exec* X = nullptr;
  bool hit = false;
  for (auto it = C.cache.begin(); it != C.cache.end(); ++it) {
    Exec& e = **it;
    if (e.n == n && e.nb == nb && e.uplo == up && e.kind == A_desc->kind && e.ngpus == ngpus && e.P == P &&
        e.Q == Q && same_plan_options(e.opt, e.key_graph, C.opt) && e.key_ptrs == ptrs &&
        (A_desc->kind == STF_DESC_TILED_2DBC ||
         (e.mat == A_desc->ptr && e.key_ld == A_desc->ld && e.key_dev == A_desc->device))) {
      C.cache.splice(C.cache.begin(), C.cache, it);
      X = C.cache.front().get();
      hit = true;
      break;
    }
  }
  int reuse = hit ? 1 : 0;
  if (!X) {
    // NEXT-2: a plan of the same shape bound to other caller
    // pointers is re-bound: same plan, workspaces and events; the graph is
    // re-captured and applied to the existing executable graph with
    // cudaGraphExecUpdate (falls back to a fresh instantiation if rejected).
    for (auto it = C.cache.begin(); it != C.cache.end(); ++it) {
      Exec& e = **it;
      const bool pageable = A_desc->kind == STF_DESC_HOST_COLMAJOR && !host_pinned(A_desc->ptr);
      if (e.n == n && e.nb == nb && e.uplo == up && e.kind == A_desc->kind && e.ngpus == ngpus && e.P == P &&
          e.Q == Q && same_plan_options(e.opt, e.key_graph, C.opt) && (e.gexec == nullptr) == (e.opt.graph == 0) &&
          !(pageable && e.gexec)) {
        int r = rebind(C, e, A_desc, ptrs);
        if (r) return r;
        C.cache.splice(C.cache.begin(), C.cache, it);
        X = C.cache.front().get();
        reuse = 2;
        break;
      }
    }
  }
  if (!X) {
    while (C.cache.size() >= kCacheMax) C.cache.pop_back();
    std::unique_ptr<Exec> e(new Exec());
    e->n = n;
    e->nb = nb;
    e->uplo = up;
    e->kind = A_desc->kind;
    e->ngpus = ngpus;
    e->P = P;
    e->Q = Q;
    e->opt = C.opt;
    e->key_graph = C.opt.graph;
    e->key_ptrs = ptrs;
    e->key_ld = A_desc->ld;
    e->key_dev = A_desc->device;
    if (host_eager(C, A_desc, n, nb, ngpus)) e->opt.graph = 0;
    if (const char* sk = getenv("STF_DEBUG_SKIP")) {
      std::string v(sk);
      const char* names[] = {"potrf", "trsm", "syrk", "gemm", "copy", "trsm_as_gemm", "trsm_as_half_gemm"};
      const unsigned bits[] = {1u << 0, 1u << 1, 1u << 2, 1u << 3, 1u << 4, 1u << 16, 1u << 17};
      size_t pos = 0;
      while (pos <= v.size()) {  // comma-separated list of exact names
        size_t end = v.find(',', pos);
        if (end == std::string::npos) end = v.size();
        const std::string item = v.substr(pos, end - pos);
        for (unsigned k = 0; k < 7; ++k)
          if (item == names[k]) e->skip_mask |= bits[k];
        pos = end + 1;
      }
    }
    int r = prepare(C, *e, A_desc);
    if (r == -103 && !C.cache.empty()) {  // out of memory: drop memoised plans and retry once
      C.cache.clear();
      e.reset(new Exec());
      e->n = n; e->nb = nb; e->uplo = up; e->kind = A_desc->kind; e->ngpus = ngpus; e->P = P; e->Q = Q;
      e->opt = C.opt; e->key_graph = C.opt.graph; e->key_ptrs = ptrs; e->key_ld = A_desc->ld; e->key_dev = A_desc->device;
      if (host_eager(C, A_desc, n, nb, ngpus)) e->opt.graph = 0;
      g_err.clear();
      r = prepare(C, *e, A_desc);
    }
    if (r) return r;
    C.cache.push_front(std::move(e));
    X = C.cache.front().get();
  }
  int info = run(C, *X);
  fill_stats(*X, hit, &C.last);
  C.last.device_ms = C.device_ms;
  C.last.graph_reuse = reuse;
  C.last_trace.clear();
  if (!X->trace.empty() && info >= 0) {  // debug timeline of this call (run() has synchronised)
    const auto& tasks = X->plan.tasks;
    cudaSetDevice(C.slots[0].device);
    for (size_t t = 0; t < tasks.size(); ++t) {
      const stf::Task& k = tasks[t];
      float a = 0.f, b = 0.f;  // ms since the first task's start event
      if (cudaEventElapsedTime(&a, X->trace[0], X->trace[2 * t]) != cudaSuccess ||
          cudaEventElapsedTime(&b, X->trace[0], X->trace[2 * t + 1]) != cudaSuccess) {
        cudaGetLastError();
        a = b = -1.f;
      }
      const int64_t rec[7] = {k.kind, k.i, k.j, k.k, k.stream, (int64_t)(a * 1e6), (int64_t)(b * 1e6)};
      C.last_trace.insert(C.last_trace.end(), rec, rec + 7);
    }
  }
  if (info < 0) {
    // a failed call leaves device state unknown: drop the plan
    C.cache.remove_if([&](const std::unique_ptr<Exec>& p) { return p.get() == X; });
  }
  return info;
}

int64_t stf_debug_last_trace(int64_t* out, int64_t cap_tasks) {
  Context& C = ctx();
  std::lock_guard<std::mutex> g(C.mu);
  const int64_t n = (int64_t)C.last_trace.size() / 7;
  if (out)
    std::copy(C.last_trace.begin(), C.last_trace.begin() + 7 * std::min(n, std::max<int64_t>(cap_tasks, 0)), out);
  return n;
}

int stf_last_stats(stf_plan_stats* out) {
  Context& C = ctx();
  std::lock_guard<std::mutex> g(C.mu);
  if (!out) return fail(-105, "NULL stats pointer");
  *out = C.last;
  return 0;
}

int stf_dag_tasks_io(int64_t cap_tasks, int64_t* io) {
  g_err.clear();
  const stf::Plan& plan = g_dag_plan;
  for (size_t t = 0; t < plan.tasks.size() && (int64_t)t < cap_tasks; ++t) {
    io[3 * t] = plan.tasks[t].in[0];
    io[3 * t + 1] = plan.tasks[t].in[1];
    io[3 * t + 2] = plan.tasks[t].out;
  }
  return (int)std::min<size_t>(plan.buffers.size(), INT_MAX);
}

int stf_dag_build(int64_t T, int p, int q, int64_t cap, int64_t* edges, int64_t cap_tasks, int32_t* kinds,
                  int64_t* ijk, stf_plan_stats* stats) {
  g_err.clear();
  if (T < 0) return fail(-1, "T < 0");
  if (p < 1 || q < 1) return fail(-4, "bad grid %dx%d", p, q);
  Options o;
  o.priority = 1;
  o.push = ctx().opt.push;            // the DAG options the next stf_potrf would use
  o.lookahead = ctx().opt.lookahead;
  stf::Plan& plan = g_dag_plan;
  auto t0 = std::chrono::steady_clock::now();
  // with "mem_cap_tiles" set and one slot: the out-of-core plan of a HOST_COLMAJOR call
  const bool ooc = ctx().opt.mem_cap_tiles > 0 && p * q == 1 && ctx().opt.mem_cap_tiles < T * (T + 1) / 2;
  stf::PlanOptions po = plan_options(o, p, q, p * q, ooc, ooc);
  if (ooc) po.frames = ctx().opt.mem_cap_tiles;
  po.ooc_order = (int)ctx().opt.ooc_order;
  stf::build_plan(plan, T, po);
  double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  int64_t e = 0;
  for (int64_t t = 0; t < plan.graph.ntasks(); ++t)
    for (const int64_t* x = plan.graph.preds_begin(t); x != plan.graph.preds_end(t); ++x, ++e)
      if (edges && e < cap) {
        edges[2 * e] = *x;
        edges[2 * e + 1] = t;
      }
  for (size_t t = 0; t < plan.tasks.size() && (int64_t)t < cap_tasks; ++t) {
    if (kinds) kinds[t] = plan.tasks[t].kind;
    if (ijk) {
      ijk[3 * t] = plan.tasks[t].i;
      ijk[3 * t + 1] = plan.tasks[t].j;
      ijk[3 * t + 2] = plan.tasks[t].k;
    }
  }
  if (stats) {
    int64_t compute = 0;
    for (const auto& t : plan.tasks) compute += (t.kind <= stf::K_GEMM);
    stats->tasks = compute;
    stats->transfers = plan.ntransfers + plan.npushed;
    stats->edges = plan.graph.nedges();
    stats->transfer_bytes = 0;
    stats->critical_path = plan.critical_path;
    stats->graph_nodes = 0;
    stats->kernel_launches = 0;
    stats->build_ms = ms;
    stats->device_ms = 0;
    stats->graph_reuse = 0;
    stats->dag_tasks = (int64_t)plan.tasks.size();
    stats->host_loads = plan.nloads;
    stats->host_stores = plan.nstores;
    stats->frames = plan.opt.frames;
  }
  return 0;
}

int64_t stf_infer_edges(int64_t ntasks, const int32_t* nacc, const int64_t* data, const int32_t* modes, int64_t cap,
                        int64_t* edges) {
  g_err.clear();
  if (ntasks < 0 || (ntasks > 0 && (!nacc || !data || !modes))) return fail(-4, "bad arguments");
  stf::TaskGraph G(0);
  int64_t off = 0;
  std::vector<stf::Access> acc;
  for (int64_t t = 0; t < ntasks; ++t) {
    acc.clear();
    for (int32_t a = 0; a < nacc[t]; ++a) {
      const int32_t m = modes[off + a];
      if (m < 1 || m > 3) return fail(-4, "bad access mode %d", m);
      acc.push_back(stf::Access{data[off + a], (uint8_t)m});
    }
    off += nacc[t];
    G.submit(acc.data(), (int)acc.size());
  }
  int64_t e = 0;
  for (int64_t t = 0; t < ntasks; ++t)
    for (const int64_t* x = G.preds_begin(t); x != G.preds_end(t); ++x, ++e)
      if (edges && e < cap) {
        edges[2 * e] = *x;
        edges[2 * e + 1] = t;
      }
  return e;
}

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
  if (ctx().opt.trsm == 3 && stfk::trsm_res_supported((int)n, L, ldl)) {
    CUDA_TRY(stfk::trsm_res(0, 0, (int)M, (int)n, L, ldl, B, ldb), "trsm (resident panel)");
    CUDA_TRY(cudaStreamSynchronize(0), "trsm sync");
    return 0;
  }
  if (ctx().opt.trsm >= 2) {
    CUDA_TRY(stfk::trsm_panel(0, 0, (int)M, (int)n, L, ldl, B, ldb, (int)ctx().opt.trsm_rows), "trsm (row panel)");
    CUDA_TRY(cudaStreamSynchronize(0), "trsm sync");
    return 0;
  }
  if (ctx().opt.trsm == 1) {
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
    e = ctx().opt.dataflow ? stfk::potrf_tile(0, 0, (int)n, A, lda, 0, d_info, ws)
                           : stfk::potrf_lower(0, 0, (int)n, A, lda, 0, d_info);
  unsigned long long v = ULLONG_MAX;
  if (e == cudaSuccess) e = cudaMemcpy(&v, d_info, sizeof v, cudaMemcpyDeviceToHost);
  cudaFree(d_info);
  cudaFree(ws);
  if (e != cudaSuccess) return cuda_fail(e, "potrf");
  if (info) *info = (v == ULLONG_MAX) ? 0 : (int64_t)v;
  return 0;
}

// ---------------------------------------------------------------- multi-process mode
namespace {
struct MpBlob {
  int32_t magic;
  int32_t slot;
  int64_t count;  // replicas (and flags) of this slot
  cudaIpcMemHandle_t arena;
  cudaIpcMemHandle_t flags;
};
constexpr int32_t kMpMagic = 0x53544650;  // "STFP"
}  // namespace

int stf_mp_init(int rank, int world, int device) {
  if (world < 1 || rank < 0 || rank >= world) return fail(-5, "bad rank %d / world %d", rank, world);
  if (!load_memops()) return fail(-101, "CUDA stream memory operations unavailable");
  std::vector<int> devs((size_t)world, device);
  int r = stf_cholesky_init(world, devs.data());
  if (r) return r;
  Context& C = ctx();
  std::lock_guard<std::mutex> g(C.mu);
  C.mp_me = rank;
  return 0;
}

int64_t stf_mp_blob_size(void) { return (int64_t)sizeof(MpBlob); }

int stf_mp_prepare(int64_t n, int64_t nb, const stf_matrix_desc* A_desc, void* blob) {
  Context& C = ctx();
  std::lock_guard<std::mutex> g(C.mu);
  g_err.clear();
  if (C.mp_me < 0) return fail(-100, "stf_mp_prepare: call stf_mp_init first");
  if (n < 1 || nb < 2 || (nb & 1) || n % nb || nb > 16384) return fail(-2, "bad n / nb");
  if (!A_desc || A_desc->kind != STF_DESC_TILED_2DBC || !A_desc->tiles) return fail(-4, "TILED_2DBC descriptor required");
  const int world = (int)C.slots.size();
  if ((int64_t)A_desc->p * A_desc->q != world) return fail(-4, "grid %dx%d != world %d", A_desc->p, A_desc->q, world);
  if (C.opt.lookahead == 0) return fail(-105, "lookahead=0 (fence tasks) is not supported in multi-process mode");
  const int64_t T = n / nb;
  const int P = A_desc->p, Q = A_desc->q, me = C.mp_me;
  for (int64_t j = 0; j < T; ++j)
    for (int64_t i = j; i < T; ++i) {
      if ((int)((i % P) * Q + (j % Q)) != me) continue;
      const double* tp = A_desc->tiles[(size_t)(i + j * T)];
      int d = -1;
      if (!tp || !device_of(tp, &d) || d != C.slots[(size_t)me].device)
        return fail(-4, "own tile (%lld,%lld) is not device memory on this process's device", (long long)i,
                    (long long)j);
    }
  std::unique_ptr<Exec> e(new Exec());
  e->n = n;
  e->nb = nb;
  e->kind = STF_DESC_TILED_2DBC;
  e->ngpus = world;
  e->P = P;
  e->Q = Q;
  e->opt = C.opt;
  e->opt.threads = 1;  // one slot per process: one submission thread
  e->mp = true;
  int r = prepare(C, *e, A_desc);
  if (r) return r;
  MpBlob b{};
  b.magic = kMpMagic;
  b.slot = me;
  b.count = (int64_t)e->local_flag_count;
  if (e->local_flag_count) {
    CUDA_TRY(cudaIpcGetMemHandle(&b.arena, e->local_arena), "cudaIpcGetMemHandle(arena)");
    CUDA_TRY(cudaIpcGetMemHandle(&b.flags, e->local_flags), "cudaIpcGetMemHandle(flags)");
  }
  if (blob) memcpy(blob, &b, sizeof b);
  C.mp_exec = std::move(e);
  return 0;
}

int stf_mp_import(const void* blobs) {
  Context& C = ctx();
  std::lock_guard<std::mutex> g(C.mu);
  g_err.clear();
  if (!C.mp_exec) return fail(-100, "stf_mp_import: call stf_mp_prepare first");
  Exec& X = *C.mp_exec;
  const MpBlob* B = static_cast<const MpBlob*>(blobs);
  for (int s = 0; s < X.ngpus; ++s) {
    if (B[s].magic != kMpMagic || B[s].slot != s) return fail(-4, "blob %d is not slot %d's", s, s);
    if (s == C.mp_me || B[s].count == 0) continue;
    void *pa = nullptr, *pf = nullptr;
    CUDA_TRY(cudaIpcOpenMemHandle(&pa, B[s].arena, cudaIpcMemLazyEnablePeerAccess), "cudaIpcOpenMemHandle(arena)");
    X.ipc_opened.push_back(pa);
    CUDA_TRY(cudaIpcOpenMemHandle(&pf, B[s].flags, cudaIpcMemLazyEnablePeerAccess), "cudaIpcOpenMemHandle(flags)");
    X.ipc_opened.push_back(pf);
    X.peer_arena[(size_t)s] = static_cast<double*>(pa);
    X.peer_flags[(size_t)s] = static_cast<uint32_t*>(pf);
  }
  for (size_t b = 0; b < X.plan.buffers.size(); ++b) {
    const stf::Buffer& Bf = X.plan.buffers[b];
    if (Bf.replica && Bf.slot != C.mp_me) X.buf[b] = X.peer_arena[(size_t)Bf.slot] + X.rep_off[b];
  }
  if (X.opt.graph) return capture_graph(C, X);
  return 0;
}

int stf_mp_potrf(void) {
  Context& C = ctx();
  std::lock_guard<std::mutex> g(C.mu);
  g_err.clear();
  if (!C.mp_exec) return fail(-100, "stf_mp_potrf: call stf_mp_prepare / stf_mp_import first");
  int info = run(C, *C.mp_exec);
  fill_stats(*C.mp_exec, false, &C.last);
  C.last.device_ms = C.device_ms;
  return info;
}

int stf_bench_kernel(int kind, int64_t M, int64_t N, int64_t K, int reps, double* avg_ms) {
  g_err.clear();
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
  auto step = [&](cudaError_t x) { if (e == cudaSuccess) e = x; };
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
          step(ctx().opt.trsm == 3 && stfk::trsm_res_supported((int)N, Src, ldm)
                   ? stfk::trsm_res(s, 0, (int)M, (int)N, Src, ldm, Cm, ldm)
               : ctx().opt.trsm >= 2 ? stfk::trsm_panel(s, 0, (int)M, (int)N, Src, ldm, Cm, ldm)
               : ctx().opt.trsm == 1 ? stfk::trsm_tile(s, 0, (int)M, (int)N, Src, ldm, Cm, ldm, ws)
                                     : stfk::trsm_rlt(s, 0, (int)M, (int)N, Src, ldm, Cm, ldm));
          break;
        case 3:
          step(ctx().opt.dataflow ? stfk::potrf_tile(s, 0, (int)M, Cm, ldm, 0, info, ws)
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
  cudaFree(A); cudaFree(B); cudaFree(Cm); cudaFree(Src); cudaFree(info); cudaFree(ws);
  if (e0) cudaEventDestroy(e0);
  if (e1) cudaEventDestroy(e1);
  if (s) cudaStreamDestroy(s);
  if (e != cudaSuccess) return cuda_fail(e, "stf_bench_kernel");
  *avg_ms = total / reps;
  return 0;
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
  if (e == cudaSuccess) e = stfk::potrf_tile(0, 0, (int)n, A, lda, 0, d_info, ws, d_tr, ctas);
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
