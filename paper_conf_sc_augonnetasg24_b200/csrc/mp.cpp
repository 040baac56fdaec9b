// Multi-process mode (include/stf_cholesky.h stf_mp_*): one process per GPU,
// the launch model of torchrun.  Every process builds the same plan (the STF
// DAG of PAPER.md:144 is deterministic) and lowers only its own slot's tasks;
// the replicas it consumes (the MSI copies of PAPER.md:210-216) live in its own
// arena, exported with CUDA IPC.  A producer writes a replica over NVLink (copy
// engine into the IPC-mapped arena, or the TRSM epilogue's peer stores) and then
// a 32-bit flag with cuStreamWriteValue32; the consumer's stream waits on it with
// cuStreamWaitValue32: device-side hand-off, no host round trip, no SMs.
#include <cstring>

#include "runtime_internal.hpp"

namespace stfrt {

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

}  // namespace stfrt

using namespace stfrt;

extern "C" {

int stf_mp_init(int rank, int world, int device) {
  g_err.clear();
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
  e->key_opt = e->opt;
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

}  // extern "C"
