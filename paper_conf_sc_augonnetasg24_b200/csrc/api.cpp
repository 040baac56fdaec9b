// C ABI of include/stf_cholesky.h: the library context ("a
// context as entry point"), options, stf_potrf with its memoised plans
// (PAPER.md:166-174), statistics and host-only DAG introspection (the STF rule,
// PAPER.md:144).  Lowering lives in exec.cpp, the multi-process mode in mp.cpp,
// harness entry points (include/stf_harness.h) in harness.cpp.
#include <algorithm>
#include <chrono>
#include <climits>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "runtime_internal.hpp"

namespace stfrt {

thread_local std::string g_err;
thread_local stf::Plan g_dag_plan;  // the plan of the last stf_dag_build* on this thread (stf_dag_tasks_io)

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
  cudaGetLastError();  // clear non-sticky errors
  if (e == cudaErrorMemoryAllocation) return fail(-103, "%s: %s", what, cudaGetErrorString(e));
  return fail(-101, "%s: %s", what, cudaGetErrorString(e));
}

Context& ctx() {
  static Context c;
  return c;
}

const std::vector<OptDesc>& option_table() {
  static const std::vector<OptDesc> t = {
      {"dataflow", "STF_DATAFLOW", &Options::dataflow, 0, 1, true},
      {"trsm", "STF_TRSM", &Options::trsm, 0, 3, true},
      {"trsm_split", "STF_TRSM_SPLIT", &Options::trsm_split, 1, 16, true},
      {"graph", "STF_GRAPH", &Options::graph, 0, 1, true},
      {"streams", "STF_STREAMS", &Options::streams, 1, 64, true},
      {"serial", "STF_SERIAL", &Options::serial, 0, 1, true},
      {"priority", "STF_PRIO", &Options::priority, 0, 1, true},
      {"grid_p", "STF_GRID", &Options::grid_p, 0, 64, false},  // the grid itself is part of the key
      {"lookahead", "STF_LOOKAHEAD", &Options::lookahead, 0, 1, true},
      {"threads", "STF_THREADS", &Options::threads, 1, 64, false},  // eager submission only
      {"push", "STF_PUSH", &Options::push, 0, 2, true},
      {"mem_cap_tiles", "STF_MEM_CAP_TILES", &Options::mem_cap_tiles, 0, INT64_MAX, true},
      {"ooc_order", "STF_OOC_ORDER", &Options::ooc_order, -1, 1, true},
      {"host_stream", "STF_HOST_STREAM", &Options::host_stream, 0, 1, true},
      {"trsm_res_tail", "STF_TRSM_RES_TAIL", &Options::trsm_res_tail, -1, INT64_MAX, true},
      {"trsm_rows", "STF_TRSM_ROWS", &Options::trsm_rows, 32, 128, true},
      {"trsm_res_split", "STF_TRSM_RES_SPLIT", &Options::trsm_res_split, 1, 4, true},
      {"gemm_merge", "STF_GEMM_MERGE", &Options::gemm_merge, 0, 64, true},
      {"gemm_group", "STF_GEMM_GROUP", &Options::gemm_group, -1, 4, true},
      {"order_mode", "STF_ORDER_MODE", &Options::order_mode, -1, 2, true},
      {"order_tail", "STF_ORDER_TAIL", &Options::order_tail, -1, INT64_MAX, true},
      {"order_asap", "STF_ORDER_ASAP", &Options::order_asap, 0, 1, true},
      {"sched_width", "STF_SCHED_WIDTH", &Options::sched_width, 0, 64, true},
      {"prio_mode", "STF_PRIO_MODE", &Options::prio_mode, 0, 3, true},
      {"ooc_reorder", "STF_OOC_REORDER", &Options::ooc_reorder, 0, 1, true},
      {"dev_order", "STF_DEV_ORDER", &Options::dev_order, 0, 1, true},
      {"ooc_budget_pct", "STF_OOC_BUDGET_PCT", &Options::ooc_budget_pct, -1, 95, true},
      {"host_stream_budget_pct", "STF_HOST_STREAM_BUDGET_PCT", &Options::host_stream_budget_pct, 10, 99, true},
      {"host_eager", "STF_HOST_EAGER", &Options::host_eager, 0, 1, true},
      {"stream_pool", "STF_STREAM_POOL", &Options::stream_pool, 0, 2, true},
      {"pdl", "STF_PDL", &Options::pdl, 0, 1, true},
      {"pdl_lead", "STF_PDL_LEAD", &Options::pdl_lead, -1, 1024, true},
      {"potrf_split", "STF_POTRF_SPLIT", &Options::potrf_split, 0, 1, true},
      {"potrf_ctas", "STF_POTRF_CTAS", &Options::potrf_ctas, 0, 1024, true},
      {"debug_skip", "STF_DEBUG_SKIP", &Options::debug_skip, 0, INT64_MAX, true},
      {"debug_trace", "STF_DEBUG_TRACE", &Options::debug_trace, 0, 1, true},
      {"nvtx", "STF_NVTX", &Options::nvtx, 0, 1, false},
  };
  return t;
}

int check_option(const OptDesc& d, int64_t v, int pool_streams) {
  const std::string n(d.name);
  if (v < d.lo || v > d.hi)
    return fail(-105, "option %s=%lld out of range [%lld, %lld]", d.name, (long long)v, (long long)d.lo,
                (long long)d.hi);
  if (n == "mem_cap_tiles" && v != 0 && v < 3)
    return fail(-105, "mem_cap_tiles must be 0 (no cap) or >= 3 (a GEMM holds 3 tiles)");
  if (n == "trsm_rows" && v != 32 && v != 64 && v != 128) return fail(-105, "trsm_rows must be 32, 64 or 128");
  if (n == "ooc_budget_pct" && v != -1 && v < 10) return fail(-105, "ooc_budget_pct must be -1 (auto) or in [10, 95]");
  if (n == "order_mode" && v == 1) return fail(-105, "order_mode must be -1 (auto), 0 (program) or 2 (list)");
  if (n == "trsm_res_split" && v == 3) return fail(-105, "trsm_res_split must be 1, 2 or 4");
  if (n == "gemm_group" && v >= 0 && v < 2) return fail(-105, "gemm_group must be -1 (auto) or 2..4");
  if (n == "streams" && pool_streams > 0 && v > pool_streams)
    return fail(-105, "streams=%lld exceeds the pool created at init (%d)", (long long)v, pool_streams);
  return 0;
}

bool same_plan_options(const Options& a, const Options& b) {
  for (const OptDesc& d : option_table())
    if (d.plan_key && a.*(d.field) != b.*(d.field)) return false;
  return true;
}

int64_t parse_skip(const char* s) {
  if (!s || !*s) return 0;
  char* end = nullptr;
  const long long iv = strtoll(s, &end, 10);
  if (end && *end == 0) return iv;
  static const char* names[] = {"potrf", "trsm", "syrk", "gemm", "copy", "trsm_as_gemm", "trsm_as_half_gemm"};
  static const int64_t bits[] = {1 << 0, 1 << 1, 1 << 2, 1 << 3, 1 << 4, 1 << 16, 1 << 17};
  int64_t m = 0;
  std::string v(s);
  size_t pos = 0;
  while (pos <= v.size()) {  // comma-separated list of exact names
    size_t e = v.find(',', pos);
    if (e == std::string::npos) e = v.size();
    const std::string item = v.substr(pos, e - pos);
    for (unsigned k = 0; k < 7; ++k)
      if (item == names[k]) m |= bits[k];
    pos = e + 1;
  }
  return m;
}

namespace {

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

// options from the environment (STF_<NAME>), validated like stf_set_option
int options_from_env(Options& o) {
  for (const OptDesc& d : option_table()) {
    const char* v = getenv(d.env);
    if (!v || !*v) continue;
    const int64_t x = (std::string(d.name) == "debug_skip") ? parse_skip(v) : strtoll(v, nullptr, 10);
    int r = check_option(d, x, 0);
    if (r) return fail(-105, "environment %s: %s", d.env, g_err.c_str());
    o.*(d.field) = x;
  }
  return 0;
}

void release_all(Context& C) {
  C.cache.clear();
  C.mp_exec.reset();
  C.mp_me = -1;
  for (size_t k = 0; k < C.fork_join.size(); ++k)
    if (C.fork_join[k]) cudaEventDestroy(C.fork_join[k]);
  C.fork_join.clear();
  for (auto ev : C.caller_ev)
    if (ev) cudaEventDestroy(ev);
  C.caller_ev.clear();
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

int pool_streams(const Context& C) {
  return C.inited && !C.slots.empty() ? (int)C.slots[0].streams.size() - kCritStreams - kCopyStreams : 0;
}

}  // namespace
}  // namespace stfrt

using namespace stfrt;

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
  Options o;
  if (int r = options_from_env(o)) return r;
  C.opt = o;
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
  // peer access between distinct devices: every transfer and fused push is a
  // device-to-device write over NVLink, so a pair without peer access is an
  // error here (fail fast) rather than a staged copy or a hang later
  for (int a : C.devices)
    for (int b : C.devices) {
      if (a == b) continue;
      int can = 0;
      cudaDeviceCanAccessPeer(&can, a, b);
      if (!can) {
        C.slots.clear();
        return fail(-101, "no peer access from device %d to device %d (NVLink P2P required)", a, b);
      }
      cudaSetDevice(a);
      cudaError_t pe = cudaDeviceEnablePeerAccess(b, 0);
      if (pe != cudaSuccess && pe != cudaErrorPeerAccessAlreadyEnabled) {
        C.slots.clear();
        return cuda_fail(pe, "enable peer access");
      }
      cudaGetLastError();
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
  // two per device (legacy and per-thread default stream of the caller)
  C.caller_ev.assign(2 * C.devices.size(), nullptr);
  for (size_t k = 0; k < C.caller_ev.size(); ++k) {
    cudaSetDevice(C.devices[k / 2]);
    CUDA_TRY(cudaEventCreateWithFlags(&C.caller_ev[k], cudaEventDisableTiming), "caller event");
  }
  cudaSetDevice(C.origin_dev);
  CUDA_TRY(cudaEventCreate(&C.t_start), "timing event");
  CUDA_TRY(cudaEventCreate(&C.t_end), "timing event");
  C.inited = true;
  return 0;
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
  for (const OptDesc& d : option_table())
    if (!strcmp(d.name, name)) {
      if (int r = check_option(d, value, pool_streams(C))) return r;
      C.opt.*(d.field) = value;
      return 0;
    }
  return fail(-105, "unknown option '%s'", name);
}

int stf_get_option(const char* name, int64_t* value) {
  Context& C = ctx();
  std::lock_guard<std::mutex> g(C.mu);
  g_err.clear();
  if (!name || !value) return fail(-105, "NULL argument");
  for (const OptDesc& d : option_table())
    if (!strcmp(d.name, name)) {
      *value = C.opt.*(d.field);
      return 0;
    }
  return fail(-105, "unknown option '%s'", name);
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
  if (C.mp_me >= 0) return fail(-100, "stf_potrf: library initialised in multi-process mode (use stf_mp_potrf)");
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
  if (A_desc->kind == STF_DESC_HOST_COLMAJOR && C.opt.mem_cap_tiles > 0 && C.opt.mem_cap_tiles < T * (T + 1) / 2 &&
      !C.opt.lookahead)
    return fail(-105, "lookahead=0 (per-step fences) is not available for out-of-core plans");
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
        if (reinterpret_cast<uintptr_t>(tp) & 15)
          return fail(-4, "tile (%lld,%lld) not 16-byte aligned", (long long)i, (long long)j);
        ptrs.push_back(reinterpret_cast<uintptr_t>(tp));
      }
  }
  const bool pageable = A_desc->kind == STF_DESC_HOST_COLMAJOR && !host_pinned(A_desc->ptr);
  auto same_shape = [&](const Exec& e) {
    return e.n == n && e.nb == nb && e.uplo == up && e.kind == A_desc->kind && e.ngpus == ngpus && e.P == P &&
           e.Q == Q && same_plan_options(e.key_opt, C.opt);
  };
  // memo lookup
  Exec* X = nullptr;
  bool hit = false;
  for (auto it = C.cache.begin(); it != C.cache.end(); ++it) {
    Exec& e = **it;
    if (same_shape(e) && e.key_ptrs == ptrs &&
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
      if (same_shape(e) && (e.gexec == nullptr) == (e.opt.graph == 0) && !(pageable && e.gexec)) {
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
    auto make = [&]() {
      std::unique_ptr<Exec> e(new Exec());
      e->n = n;
      e->nb = nb;
      e->uplo = up;
      e->kind = A_desc->kind;
      e->ngpus = ngpus;
      e->P = P;
      e->Q = Q;
      e->opt = C.opt;
      e->key_opt = C.opt;
      e->key_ptrs = ptrs;
      e->key_ld = A_desc->ld;
      e->key_dev = A_desc->device;
      // pageable host memory cannot be captured: eager lowering
      if (A_desc->kind == STF_DESC_HOST_COLMAJOR && (pageable || C.opt.host_eager)) e->opt.graph = 0;
      return e;
    };
    std::unique_ptr<Exec> e = make();
    int r = prepare(C, *e, A_desc);
    if (r == -103 && !C.cache.empty()) {  // out of memory: drop memoised plans and retry once
      C.cache.clear();
      e = make();
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

int64_t stf_dag_tasks_io2(int64_t cap_tasks, int64_t* io2) {
  g_err.clear();
  const stf::Plan& plan = g_dag_plan;
  for (size_t t = 0; t < plan.tasks.size() && (int64_t)t < cap_tasks; ++t)
    for (int u = 0; u < 6; ++u) io2[6 * t + u] = plan.tasks[t].xin[u];
  return plan.nmerged;
}

int64_t stf_dag_tasks_mirrors(int64_t cap_tasks, int64_t* mir) {
  g_err.clear();
  const stf::Plan& plan = g_dag_plan;
  int64_t total = 0;
  for (size_t t = 0; t < plan.tasks.size(); ++t) {
    const stf::Task& k = plan.tasks[t];
    total += k.nmir;
    if ((int64_t)t < cap_tasks && mir) {
      mir[8 * t] = k.nmir;
      for (int m = 0; m < 7; ++m) mir[8 * t + 1 + m] = m < k.nmir ? k.mir[m] : -1;
    }
  }
  return total;
}

}  // extern "C"

namespace {
void export_plan(const stf::Plan& plan, int64_t cap, int64_t* edges, int64_t cap_tasks, int32_t* kinds, int64_t* ijk) {
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
}
}  // namespace

extern "C" {

int stf_dag_build(int64_t T, int p, int q, int64_t cap, int64_t* edges, int64_t cap_tasks, int32_t* kinds,
                  int64_t* ijk, stf_plan_stats* stats) {
  g_err.clear();
  if (T < 0) return fail(-1, "T < 0");
  if (p < 1 || q < 1) return fail(-4, "bad grid %dx%d", p, q);
  if (ctx().opt.mem_cap_tiles > 0 && p * q == 1 && ctx().opt.mem_cap_tiles < T * (T + 1) / 2 && !ctx().opt.lookahead)
    return fail(-105, "lookahead=0 (per-step fences) is not available for out-of-core plans");
  // the current options; "order_mode" / "order_tail" auto mean program order here
  // (stf_dag_build_call resolves them as a call would), no host_stream plan
  Options o;
  {
    std::lock_guard<std::mutex> g(ctx().mu);
    o = ctx().opt;
  }
  if (o.order_mode < 0) o.order_mode = 0;
  if (o.order_tail < 0) o.order_tail = 0;
  o.host_stream = 0;
  stf::Plan& plan = g_dag_plan;
  auto t0 = std::chrono::steady_clock::now();
  // with "mem_cap_tiles" set and one slot: the out-of-core plan of a HOST_COLMAJOR call
  const bool ooc = o.mem_cap_tiles > 0 && p * q == 1 && o.mem_cap_tiles < T * (T + 1) / 2;
  // nb = 1024 on 148 SMs for the scheduling model (list-scheduling width 2)
  stf::PlanOptions po = call_plan_options(o, std::max<int64_t>(T, 1) * 1024, 1024,
                                          ooc ? STF_DESC_HOST_COLMAJOR : STF_DESC_TILED_2DBC, p, q, p * q, 148);
  stf::build_plan(plan, T, po);
  const double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  export_plan(plan, cap, edges, cap_tasks, kinds, ijk);
  if (stats) {
    fill_plan_stats(plan, 0, stats);
    stats->build_ms = ms;
  }
  return 0;
}

int stf_dag_build_call(int64_t n, int64_t nb, int kind, int ngpus, int p, int q, int sms, int64_t cap, int64_t* edges,
                       int64_t cap_tasks, int32_t* kinds, int64_t* ijk, stf_plan_stats* stats) {
  g_err.clear();
  if (n < 1 || nb < 2 || n % nb) return fail(-2, "bad n / nb");
  if (kind < STF_DESC_TILED_2DBC || kind > STF_DESC_HOST_COLMAJOR) return fail(-4, "bad descriptor kind");
  if (ngpus < 1 || p < 1 || q < 1 || p * q != ngpus) return fail(-4, "bad grid %dx%d for %d slots", p, q, ngpus);
  Options o;
  {
    std::lock_guard<std::mutex> g(ctx().mu);
    o = ctx().opt;
  }
  const int64_t T = n / nb;
  if (kind == STF_DESC_HOST_COLMAJOR && o.mem_cap_tiles > 0 && o.mem_cap_tiles < T * (T + 1) / 2 && !o.lookahead)
    return fail(-105, "lookahead=0 (per-step fences) is not available for out-of-core plans");
  stf::Plan& plan = g_dag_plan;
  auto t0 = std::chrono::steady_clock::now();
  stf::PlanOptions po = call_plan_options(o, n, nb, kind, p, q, ngpus, sms > 0 ? sms : 148);
  stf::build_plan(plan, T, po);
  const double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  export_plan(plan, cap, edges, cap_tasks, kinds, ijk);
  if (stats) {
    fill_plan_stats(plan, nb, stats);
    stats->build_ms = ms;
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

}  // extern "C"
