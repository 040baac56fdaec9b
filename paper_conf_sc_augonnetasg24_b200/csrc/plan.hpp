// Cholesky task generator + 2D block-cyclic placement + MSI-lite replicas +
// stream assignment (§8 rows a1-a3, a5, a7).
//
// Program order (right-looking tiled Cholesky, ref. [17] PAPER.md:495; one
// logical datum per tile):
//   for k: POTRF(k)                      A_kk:rw
//          for i>k: TRSM(i,k)            A_kk:r  A_ik:rw
//          for i>k: SYRK(i,k)            A_ik:r  A_ii:rw
//                   for k<j<i: GEMM(i,j,k)  A_ik:r  A_jk:r  A_ij:rw
// Placement (owner computes): the task runs on the owner
// of the tile it writes; owner(i,j) = (i mod P)*Q + (j mod Q).
// Coherency (asynchronous MSI): every tile has a home
// instance on its owner; a read on another slot needs a valid replica there.
// If the replica is missing or stale (tile version changed), a COPY task is
// emitted in program order just before the reader: it reads the home tile and
// writes the replica datum, so the same STF rule orders it after the tile's
// last writer and before every later writer of the replica (WAR).  Cholesky
// tiles are final when first read remotely, so each replica is copied once.
// Optional LOAD (tile <- caller matrix) and STORE (caller matrix <- tile) tasks
// implement the COLMAJOR descriptors and the write-back of PAPER.md:146-148.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "stf_core.hpp"

namespace stf {

enum Kind : int32_t { K_POTRF = 0, K_TRSM = 1, K_SYRK = 2, K_GEMM = 3, K_COPY = 4, K_LOAD = 5, K_STORE = 6, K_FENCE = 7 };

struct Task {
  int32_t kind;
  int32_t i, j, k;   // tile indices (COPY/LOAD/STORE: tile (i,j); COPY: k = destination slot)
  int32_t slot;      // executing slot (COPY: source slot, push model)
  int32_t prio;      // urgency level 0..5 (5 = critical path); >= 4 runs on the high-priority streams
  int32_t stream;    // index into the slot's stream pool (see Lowering in runtime.cpp)
  int64_t in[2];     // buffer ids read (-1 if unused)
  int64_t out;       // buffer id written
  int32_t nmir;      // fused push (NEXT-3): replica buffers written by the same kernel
  int64_t mir[7];
  int32_t nupd = 1;           // merged GEMM: tile updates k, k+1, .., k+nupd-1 in one task
  int64_t xin[6] = {-1, -1, -1, -1, -1, -1};  // their operands after the first: (L_i,k+u, L_j,k+u), u = 1..3
};

struct PlanOptions {
  int P = 1, Q = 1;
  int nslots = 1;
  int bulk_streams = 8;
  int crit_streams = 2;
  int copy_streams = 2;
  bool serial = false;     // all compute tasks of a slot on stream 0 (program order)
  int stream_pool = 0;     // 1: one compute + one copy stream per slot; 2: one stream per slot (ablations)
  bool priority = true;
  int prio_mode = 0;       // level assignment variant (0 default; see plan.cpp)
  bool with_load = false;  // LOAD tasks first (COLMAJOR descriptors)
  bool with_store = false; // STORE tasks (write-back) at the end of program order
  bool store_own_stream = true;  // STOREs on the other copy stream than the slot's LOADs
  bool order_asap = false;  // re-submit the tasks in order of earliest start (see plan.cpp);
                            // the runtime sets it for COLMAJOR calls (LOAD/STORE tasks)
  int order_mode = 0;       // 2: re-submit in simulated list-scheduling order (plan.cpp reorder_list)
  int64_t order_tail = 0;   // order_mode 2: re-order only the last order_tail panel steps (0: all)
  int sched_width = 3;      // order_mode 2: compute tasks a GPU slot runs at a time in the model
                            // (the runtime derives it from nb and the SM count)
  double copy_cost = 0;     // order_asap: a tile copy in GEMM-tile times (0: 2.7, nb = 1024)
  bool lookahead = true;   // false: a FENCE task (RW on every tile) closes each panel step, so
                           // step k+1 starts only when step k is complete (ablation, NEXT-1)
  bool push = false;       // TRSM(i,k) writes L_ik into its consumers' replicas itself (fused
                           // push, NEXT-3) instead of COPY tasks at the first remote read
  int data_plane = 0;      // requested data plane (statistics): 0 COPY, 1 fused push, 2 multicast
  int gemm_merge = 0;      // D > 0: the updates of a tile from a group of gemm_group consecutive panels
  int gemm_group = 2;      // g G .. g G + G - 1 become one task at step g G + G - 1 when the tile is at
                           // least D columns right of that panel (one K = G nb sweep)
  bool push_potrf = false; // with push: POTRF(k) also writes L_kk into the replicas of the
                           // slots running TRSM(i,k) (the dataflow POTRF kernel's epilogue)
  int64_t frames = 0;      // > 0 (one slot, with_load/with_store): memory-capped out-of-core
                           // plan (NEXT-4) over this many device tile frames; see plan.cpp
  bool ooc_reorder = true;  // order_mode 2 also re-orders out-of-core plans (loads by simulated start)
  int ooc_budget_pct = 60;  // 2D order: % of the frames a block (triangle + row chunk) may fill
  int dev_order = 0;        // device-resident plans: 0 right-looking program order, 1 2D-blocked left-looking
  int ooc_order = -1;      // out-of-core program order: 0 tall super-columns, 1 2D-blocked,
                           // -1 auto: 2D-blocked if re-ordered, else while fewer than half
                           // the tiles fit (plan.cpp)
};

// A "buffer" is one physical nb x nb tile instance: home tiles are buffers
// 0..NT-1 (lower tile (i,j) -> i*(i+1)/2 + j), replicas follow.  In an
// out-of-core plan the buffers are the device frames instead (i = j = -1):
// tiles move between the caller's host matrix and frames by LOAD/STORE tasks.
struct Buffer {
  int32_t i, j, slot;
  bool replica;
};

struct Plan {
  int64_t T = 0;
  PlanOptions opt;
  std::vector<Task> tasks;
  std::vector<Buffer> buffers;
  TaskGraph graph;
  int64_t ntransfers = 0;     // COPY tasks
  int64_t npushed = 0;        // replicas written by fused push
  int64_t nmerged = 0;        // merged GEMM tasks (two tile updates each)
  int64_t nloads = 0;         // LOAD tasks (caller matrix -> device tile)
  int64_t nstores = 0;        // STORE tasks (device tile -> caller matrix)
  int64_t critical_path = 0;  // longest chain counted in compute tasks
  std::vector<int64_t> replicas_per_slot;

  int owner(int64_t i, int64_t j) const { return (int)((i % opt.P) * opt.Q + (j % opt.Q)); }
  static int64_t tile_id(int64_t i, int64_t j) { return i * (i + 1) / 2 + j; }
  int64_t ntiles() const { return T * (T + 1) / 2; }
};

// Build the full plan (tasks, DAG, replicas, stream assignment).  Pure host code.
void build_plan(Plan& plan, int64_t T, const PlanOptions& opt);

// Number of pool streams a slot needs for `opt`.
int streams_per_slot(const PlanOptions& opt);

}  // namespace stf
