// Shared state of the runtime units (not part of the C ABI):
//   api.cpp      C ABI of include/stf_cholesky.h: context, options, stf_potrf, DAG introspection
//   exec.cpp     plan -> device buffers -> CUDA streams/events (eager) or one CUDA graph (memoised)
//   mp.cpp       one process per GPU (stf_mp_*): CUDA-IPC replicas, device-side flags
//   harness.cpp  include/stf_harness.h: tile-kernel entry points, kernel timing, debug traces
//
// Paper mechanisms realised by these units:
//   A4  Algorithm 2 prologue: each task waits on the events of
//       its STF predecessors that ran on other streams; allocation is done once per
//       plan (replica arenas); the MSI update is a COPY task or a fused push.
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
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <atomic>
#include <cstdint>
#include <list>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/stf_cholesky.h"
#include "kernels/tile_ops.hpp"
#include "plan.hpp"

namespace stfrt {

// ------------------------------------------------------------------ errors
extern thread_local std::string g_err;
int fail(int code, const char* fmt, ...);
int cuda_fail(cudaError_t e, const char* what);

#define CUDA_TRY(expr, what)                               \
  do {                                                     \
    cudaError_t e_ = (expr);                               \
    if (e_ != cudaSuccess) return ::stfrt::cuda_fail(e_, what); \
  } while (0)

// ------------------------------------------------------------------ options
// Every knob that changes a plan or its lowering is an option: read once from
// the environment at stf_cholesky_init (STF_<NAME>), settable with
// stf_set_option, and part of the memo key (same_plan_options), so a plan or
// graph built under one setting is never reused under another.
struct Options {
  int64_t dataflow = 1;        // POTRF tile kernel: 1 single-launch dataflow, 0 recursive
  int64_t trsm = 3;            // TRSM tile kernel: 3 resident panel, 2 row panel, 1 dataflow, 0 recursive
  int64_t trsm_split = 4;      // non-critical row-panel TRSMs: column blocks (panel + GEMM updates)
  int64_t graph = 1;           // 1 whole-DAG CUDA graph, 0 eager streams + events
  int64_t streams = 32;        // bulk compute streams per slot
  int64_t serial = 0;          // 1: every task of a slot on one stream in program order
  int64_t priority = 1;        // graded stream priorities (critical path high)
  int64_t grid_p = 0;          // rows P of the P x Q grid for COLMAJOR kinds (0 auto)
  int64_t lookahead = 1;       // 0: FENCE task closes each panel step (ablation)
  int64_t threads = 8;         // eager backend: host submission threads
  int64_t push = 0;            // data plane: 0 COPY tasks, 1 fused epilogue push, 2 fused push via NVSwitch multicast
  int64_t mem_cap_tiles = 0;   // HOST_COLMAJOR on one GPU: device tile frames (0 = no cap)
  int64_t ooc_order = -1;      // out-of-core program order: 0 tall, 1 2D-blocked, -1 auto
  int64_t host_stream = 1;     // HOST_COLMAJOR on one GPU, nb >= 512, T >= 16: frame-per-tile OOC builder
  int64_t trsm_res_tail = -1;   // -1 auto: 4096 at nb >= 1024 (n = 8192 +7%), else 8192 (nb = 512 +6%)  // trsm 3: resident panel for every TRSM once n - k nb <= this
  int64_t trsm_rows = 128;     // row panel: rows per CTA (32, 64, 128)
  int64_t trsm_res_split = 2;  // resident-panel TRSMs in 2 (or 4) column parts with GEMMs between; 1 = one launch
  int64_t gemm_merge = 2;      // D > 0: merged tile updates for tiles >= D columns right of the panel
  int64_t gemm_group = -1;     // updates per merged GEMM task (2..4; -1 auto: 4 when T >= 48, else 2)
  int64_t order_mode = -1;     // submission order: 0 program, 2 list scheduling, -1 auto (nb >= 512 -> 2)
  int64_t order_tail = -1;     // order_mode 2: re-order only the last steps (0 all, -1 auto)
  int64_t order_asap = 0;      // earliest-start submission order (order_mode 0 only)
  int64_t sched_width = 0;     // list-scheduling model width (0: from nb and the SM count)
  int64_t prio_mode = 0;       // priority level assignment variant
  int64_t ooc_reorder = 1;     // re-submit out-of-core plans in list-scheduling order
  int64_t dev_order = 0;       // device-resident plans: 1 2D-blocked left-looking program order
  int64_t ooc_budget_pct = -1; // out-of-core block budget in % of the frames (-1 auto: 60, 90 from 3/4)
  int64_t host_stream_budget_pct = 90;  // host_stream block budget
  int64_t host_eager = 0;      // 1: HOST_COLMAJOR calls on pinned memory lowered eagerly
  int64_t stream_pool = 0;     // 0 default pool; 1 one compute + one copy stream per slot; 2 one stream (ablations)
  int64_t pdl = 1;             // programmatic dependent launch: TRSM(k+1,k) overlaps POTRF(k) (graph backend)
  int64_t potrf_split = 1;     // POTRF tile as two launches (chain + few block tasks, then 2-per-SM block tasks)
  int64_t potrf_ctas = 0;      // CTAs of a POTRF tile launch (0: 3 per 64-block column, 16..96)
  int64_t pdl_lead = -1;       // pdl: the POTRF lets its TRSM start this many 64-block steps before its end (-1: nb / 128)
  int64_t debug_skip = 0;      // bit mask of task kinds not launched (timing what-ifs; results invalid)
  int64_t debug_trace = 0;     // timing events around every task (one slot)
  int64_t nvtx = 0;            // NVTX range per task submission (eager backend; the graph launch is one range)
};

struct OptDesc {
  const char* name;
  const char* env;  // environment variable read at init
  int64_t Options::*field;
  int64_t lo, hi;
  bool plan_key;  // part of the memo key
};
const std::vector<OptDesc>& option_table();
// validate one value (range + special rules); returns 0 or -105 (with g_err)
int check_option(const OptDesc& d, int64_t v, int pool_streams);
bool same_plan_options(const Options& a, const Options& b);
// parse "potrf,trsm,..." or an integer into the debug_skip mask
int64_t parse_skip(const char* s);

// ------------------------------------------------------------------ state
struct Slot {
  int device = 0;
  std::vector<cudaStream_t> streams;
  unsigned long long* d_info = nullptr;
};

// NVSwitch multicast slab (mcast.cpp): one multicast object bound on every device of a call
struct McSlab {
  CUmemGenericAllocationHandle mc = 0;
  size_t size = 0;
  std::vector<int> devs;
  std::vector<CUmemGenericAllocationHandle> phys;  // per device: its physical copy
  std::vector<CUdeviceptr> uc;                     // per device: its mapping of its copy
  std::vector<char> bound;
  CUdeviceptr mcva = 0;                            // the multicast mapping
  ~McSlab();
};
bool mc_supported(const std::vector<int>& devs, std::string* why);
int mc_create(McSlab& S, const std::vector<int>& devs, size_t bytes, std::string* why);

constexpr int kCritStreams = 6;  // 0: panel chain, 1: its feeders, 2..5: other urgent tasks by row
constexpr int kCopyStreams = 2;
constexpr size_t kCacheMax = 4;

// A plan bound to physical buffers, plus its lowering artefacts.
// Stream-capture helpers for programmatic dependent launch (exec.cpp): the single
// node a capturing stream's next launch would depend on (else null), and turning
// the capture edge from kernel node `from` into a programmatic one.
cudaGraphNode_t capture_last_node(cudaStream_t s);
int capture_make_programmatic(cudaStream_t s, cudaGraphNode_t from);
int capture_drop_dependency(cudaStream_t s, cudaGraphNode_t from);
int64_t pdl_lead_of(int64_t opt, int64_t nb);

struct Exec {
  // key
  int64_t n = 0, nb = 0;
  char uplo = 'L';
  int kind = 0, ngpus = 0, P = 1, Q = 1;
  Options opt;              // options the plan was built with (opt.graph may fall back to 0)
  Options key_opt;          // options at build time (memo key)
  std::vector<uintptr_t> key_ptrs;
  int64_t key_ld = 0;
  int key_dev = 0;

  stf::Plan plan;
  std::vector<double*> buf;                   // buffer id -> device pointer
  std::vector<std::pair<int, void*>> allocs;  // (device, ptr) library-owned
  std::vector<double*> scratch;               // per (slot, copy stream): staging tile for 'U'
  std::vector<int*> task_ws;                  // per task: dataflow-kernel workspace (POTRF/TRSM), else null
  std::vector<int64_t> pdl_src;               // per task: TRSM(k+1,k) -> index of POTRF(k) it may overlap, else -1
  std::vector<cudaGraphNode_t> cap_node;      // per task: its last captured node (POTRFs with a pdl consumer)
  std::vector<cudaGraphNode_t> cap_node2;     // per task: a POTRF's chain node (its first launch)
  int64_t pdl_edges = 0;                      // programmatic capture edges of the last capture
  std::vector<cudaEvent_t> events;            // per task, null if not needed
  std::vector<int> events_dev;
  cudaGraph_t graph = nullptr;
  cudaGraphExec_t gexec = nullptr;
  int64_t graph_nodes = 0;
  int graph_fallback = 0;            // capture failed, eager lowering used
  std::vector<cudaEvent_t> trace;    // debug_trace: per task timing events at start / end (one slot)
  int64_t updates = 0;               // successful cudaGraphExecUpdate re-binds
  bool rebound = false;
  int64_t launches = 0;
  double build_ms = 0;
  int ndevices = 1;                  // distinct CUDA devices spanned by the slots of the call
  int data_plane = 0;                // 0 COPY tasks, 1 fused push (peer stores), 2 fused push via multicast
  std::unique_ptr<McSlab> mcs;       // push = 2: the multicast slab (null when not eligible)
  std::vector<int64_t> mc_off;       // per home tile: element offset of its replicas in the slab (-1: none)
  int64_t peer_transfers = 0;        // COPY tasks / pushes whose endpoints are distinct devices
  // caller matrix for COLMAJOR kinds
  double* mat = nullptr;
  int64_t ld = 0;
  int mat_dev = -1;  // -1: host
  // multi-process mode (one process per slot): replicas of slot s live in slot s's
  // arena at rep_off[b]; their readiness is a 32-bit flag (index flag_idx[b]) in
  // slot s's flag array, written by the remote producer after the transfer.
  bool mp = false;
  std::vector<size_t> rep_off;
  std::vector<int> flag_idx;
  double* local_arena = nullptr;
  uint32_t* local_flags = nullptr;
  size_t local_flag_count = 0;
  std::vector<double*> peer_arena;
  std::vector<uint32_t*> peer_flags;
  std::vector<void*> ipc_opened;
  uint32_t epoch = 1;

  ~Exec();
};

struct Context {
  std::mutex mu;
  bool inited = false;
  std::vector<Slot> slots;
  std::vector<int> devices;  // distinct physical devices
  Options opt;
  std::list<std::unique_ptr<Exec>> cache;  // MRU first
  stf_plan_stats last{};
  std::vector<int64_t> last_trace;  // debug_trace: (kind, i, j, k, stream, t0_ns, t1_ns) per task
  cudaStream_t origin = nullptr;    // capture / launch stream on slot 0's device
  int origin_dev = 0;
  std::vector<cudaEvent_t> fork_join;  // per slot-stream, for fork/join around a call
  std::vector<cudaEvent_t> caller_ev;  // per device: caller's default-stream work, waited on by origin
  cudaEvent_t t_start = nullptr, t_end = nullptr;  // timing events on `origin`
  double device_ms = 0;
  int mp_me = -1;                  // multi-process mode: the slot this process owns
  std::unique_ptr<Exec> mp_exec;   // multi-process mode: the current plan
};

Context& ctx();

// ------------------------------------------------------------------ exec.cpp
// PlanOptions of a call: the one function both stf_potrf (prepare) and
// stf_dag_build_call use, so the introspected plan is the executed one.
stf::PlanOptions call_plan_options(const Options& o, int64_t n, int64_t nb, int kind, int P, int Q, int nslots,
                                   int sms);
int prepare(Context& C, Exec& X, const stf_matrix_desc* desc);
int rebind(Context& C, Exec& X, const stf_matrix_desc* desc, const std::vector<uintptr_t>& ptrs);
int capture_graph(Context& C, Exec& X);
int run(Context& C, Exec& X);
void fill_stats(const Exec& X, bool hit, stf_plan_stats* s);
void fill_plan_stats(const stf::Plan& P, int64_t nb, stf_plan_stats* s);
int ensure_kernel_attrs(int dev);
bool device_of(const void* ptr, int* dev);
bool host_pinned(const void* ptr);

// ------------------------------------------------------------------ mp.cpp
bool load_memops();
typedef CUresult (*PFN_wv32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
extern PFN_wv32 g_write_value32, g_wait_value32;

}  // namespace stfrt
