// Cholesky plan construction; see plan.hpp for the model and citations.
#include "plan.hpp"

#include <algorithm>
#include <cstdlib>
#include <climits>
#include <queue>
#include <set>
#include <utility>
#include <vector>

namespace stf {

int streams_per_slot(const PlanOptions& opt) {
  if (opt.stream_pool == 2) return 1;
  if (opt.stream_pool == 1) return 2;
  if (opt.serial) return 1 + opt.copy_streams;
  return opt.crit_streams + opt.bulk_streams + opt.copy_streams;
}

namespace {

// High-priority streams: the panel chain POTRF(k) -> TRSM(k+1,k) -> SYRK(k+1,k)
// (level 5) alone on stream 0, so stream order never puts a chain task behind
// another task (measured at n = 8192: POTRF(1) started 1.06 ms after SYRK(1,0)
// while it queued behind the bulk TRSMs sharing its stream); the tasks that feed
// the next chain TRSM(k+2,k+1) - TRSM(k+2,k) and GEMM(k+2,k+1,k) - alone on
// stream 1; the other urgent tasks (level 4: TRSM(i,k), the next column's
// updates) on streams 2.. by row.
template <class TaskLike>
int crit_stream(const TaskLike& t, int crit_streams) {
  if (crit_streams <= 1 || t.prio >= 5) return 0;
  const bool feeds_chain = t.i == t.k + 2 && (t.kind == K_TRSM || (t.kind == K_GEMM && t.j == t.k + 1));
  if (crit_streams == 2 || feeds_chain) return 1;
  return 2 + (int)(t.i % (crit_streams - 2));
}

struct Builder {
  Plan& p;
  const int64_t T;
  const int G;
  std::vector<int64_t> version;      // per home tile
  std::vector<int64_t> rep_buffer;   // (tile * G + slot) -> buffer id or -1
  std::vector<int64_t> rep_version;  // version the replica holds

  Builder(Plan& plan, int64_t T_) : p(plan), T(T_), G(plan.opt.nslots) {
    const int64_t NT = p.ntiles();
    version.assign((size_t)NT, 0);
    rep_buffer.assign((size_t)(NT * G), -1);
    rep_version.assign((size_t)(NT * G), -1);
  }

  int copy_stream(int dst_slot) const {
    if (p.opt.stream_pool) return p.opt.stream_pool == 1 ? 1 : 0;
    const int base = p.opt.serial ? 1 : p.opt.crit_streams + p.opt.bulk_streams;
    return base + dst_slot % p.opt.copy_streams;
  }

  int compute_stream(const Task& t) const {
    if (p.opt.serial || p.opt.stream_pool) return 0;
    if (p.opt.priority && t.prio >= 4) return crit_stream(t, p.opt.crit_streams);
    return p.opt.crit_streams + (int)((t.i * T + t.j) % p.opt.bulk_streams);
  }

  std::vector<std::vector<Access>> accs;  // per task, for a re-ordered re-submission

  void submit(Task t, const Access* acc, int nacc) {
    p.graph.submit(acc, nacc);
    p.tasks.push_back(t);
    accs.emplace_back(acc, acc + nacc);
  }

  // buffer to read tile (i,j) from on `slot`, emitting a COPY if needed
  int64_t read_buffer(int64_t i, int64_t j, int slot) {
    const int64_t d = Plan::tile_id(i, j);
    const int own = p.owner(i, j);
    if (own == slot) return d;
    const size_t r = (size_t)(d * G + slot);
    if (rep_buffer[r] < 0) {
      rep_buffer[r] = (int64_t)p.buffers.size();
      p.buffers.push_back(Buffer{(int32_t)i, (int32_t)j, slot, true});
      p.replicas_per_slot[(size_t)slot]++;
    }
    if (rep_version[r] != version[(size_t)d]) {
      Task c{K_COPY, (int32_t)i, (int32_t)j, slot, own, 1, copy_stream(slot), {d, -1}, rep_buffer[r]};
      Access acc[2] = {{d, READ}, {rep_buffer[r], WRITE}};
      submit(c, acc, 2);
      p.ntransfers++;
      rep_version[r] = version[(size_t)d];
    }
    return rep_buffer[r];
  }

  // slots (other than the owner) whose tasks read the final L_ik: SYRK(i,k) on
  // owner(i,i), GEMM(i,j,k) on owner(i,j) (k<j<i), GEMM(r,i,k) on owner(r,i) (r>i)
  std::vector<int> consumers_of_panel_tile(int64_t i, int64_t k) const {
    std::vector<int> s;
    auto add = [&](int g) {
      if (g != p.owner(i, k) && std::find(s.begin(), s.end(), g) == s.end()) s.push_back(g);
    };
    add(p.owner(i, i));
    for (int64_t j = k + 1; j < i; ++j) add(p.owner(i, j));
    for (int64_t r = i + 1; r < T; ++r) add(p.owner(r, i));
    std::sort(s.begin(), s.end());
    return s;
  }

  // slots (other than the owner) whose TRSM(i,k), i > k, read the final L_kk
  std::vector<int> consumers_of_diag_tile(int64_t k) const {
    std::vector<int> s;
    for (int64_t i = k + 1; i < T; ++i) {
      const int g = p.owner(i, k);
      if (g != p.owner(k, k) && std::find(s.begin(), s.end(), g) == s.end()) s.push_back(g);
    }
    std::sort(s.begin(), s.end());
    return s;
  }

  int64_t replica_buffer(int64_t i, int64_t j, int slot) {
    const int64_t d = Plan::tile_id(i, j);
    const size_t r = (size_t)(d * G + slot);
    if (rep_buffer[r] < 0) {
      rep_buffer[r] = (int64_t)p.buffers.size();
      p.buffers.push_back(Buffer{(int32_t)i, (int32_t)j, slot, true});
      p.replicas_per_slot[(size_t)slot]++;
    }
    return rep_buffer[r];
  }

  void compute(int32_t kind, int64_t i, int64_t j, int64_t k, int prio, int64_t ra, int64_t rb, int64_t wi,
               int64_t wj, int nupd = 1, const int64_t* xk = nullptr) {
    const int slot = p.owner(wi, wj);
    const int64_t w = Plan::tile_id(wi, wj);
    int64_t in0 = ra >= 0 ? read_buffer(ra / T, ra % T, slot) : -1;
    int64_t in1 = rb >= 0 ? read_buffer(rb / T, rb % T, slot) : -1;
    Task t{kind, (int32_t)i, (int32_t)j, (int32_t)k, slot, prio, 0, {in0, in1}, w};
    if (nupd > 1) {  // merged GEMM: the operands of updates k+1 .. k+nupd-1
      t.nupd = nupd;
      for (int u = 0; u < 2 * (nupd - 1); ++u) t.xin[u] = read_buffer(xk[u] / T, xk[u] % T, slot);
      p.nmerged++;
    }
    t.stream = compute_stream(t);
    Access acc[3 + 6 + 7];
    int n = 0;
    if (in0 >= 0) acc[n++] = {in0, READ};
    if (in1 >= 0) acc[n++] = {in1, READ};
    for (int u = 0; u < 2 * (t.nupd - 1); ++u) acc[n++] = {t.xin[u], READ};
    acc[n++] = {w, RW};
    std::vector<int> cons;
    if (kind == K_TRSM && p.opt.push) cons = consumers_of_panel_tile(wi, wj);
    if (kind == K_POTRF && p.opt.push && p.opt.push_potrf) cons = consumers_of_diag_tile(wi);
    for (int g : cons) {
      const int64_t rb2 = replica_buffer(wi, wj, g);
      t.mir[t.nmir++] = rb2;
      acc[n++] = {rb2, WRITE};
    }
    submit(t, acc, n);
    version[(size_t)w]++;
    for (int g : cons) {  // the pushed replicas hold the new version: no COPY at their reads
      rep_version[(size_t)(w * G + g)] = version[(size_t)w];
      p.npushed++;
    }
  }

  void run() {
    const int64_t NT = p.ntiles();
    p.buffers.clear();
    for (int64_t i = 0; i < T; ++i)
      for (int64_t j = 0; j <= i; ++j) p.buffers.push_back(Buffer{(int32_t)i, (int32_t)j, p.owner(i, j), false});
    (void)NT;
    if (p.opt.with_load) {
      // tile columns in order, the order in which the panel steps need them (tile
      // rows first measured 4% slower end to end)
      for (int64_t j = 0; j < T; ++j)
        for (int64_t i = j; i < T; ++i) {
          const int own = p.owner(i, j);
          const int64_t w = Plan::tile_id(i, j);
          Task t{K_LOAD, (int32_t)i, (int32_t)j, 0, own, 0, copy_stream(own), {-1, -1}, w};
          Access acc[1] = {{w, WRITE}};
          submit(t, acc, 1);
          p.nloads++;
          version[(size_t)w]++;
        }
    }
    auto key = [&](int64_t i, int64_t j) { return i * T + j; };
    // Priority levels 0..5 (5 = most urgent), by how soon the written tile feeds a
    // panel: POTRF, the next panel's TRSM and SYRK are on the critical path (5);
    // the other TRSMs and the next column's GEMMs gate the next panel (4); later
    // columns decay with their distance d = column - k.
    const bool prio = p.opt.priority;
    const int mode = p.opt.prio_mode;
    auto level = [&](int64_t d) -> int {
      if (mode == 3) return d <= 1 ? 4 : 0;                                  // two levels
      if (mode == 2) return d <= 1 ? 4 : d == 2 ? 3 : d == 3 ? 2 : d <= 5 ? 1 : 0;  // faster decay
      return d <= 1 ? 4 : d == 2 ? 3 : d <= 4 ? 2 : d <= 8 ? 1 : 0;
    };
    auto P = [&](int lv) { return prio ? lv : 0; };
    // merged GEMMs: the updates of tile (i, j) from panels gG .. gG+G-1 become one
    // task at step gG+G-1 when the tile is at least D columns right of that panel
    const int64_t D = p.opt.lookahead ? p.opt.gemm_merge : 0, G = std::max(1, std::min(4, p.opt.gemm_group));
    auto merged = [&](int64_t j, int64_t k) {  // update k of column j belongs to a merged group
      const int64_t last = k / G * G + G - 1;
      return D > 0 && G > 1 && last < j && j >= last + D;
    };
    for (int64_t k = 0; k < T; ++k) {
      compute(K_POTRF, k, k, k, P(5), -1, -1, k, k);
      for (int64_t i = k + 1; i < T; ++i)
        compute(K_TRSM, i, k, k, P(i == k + 1 || mode == 1 ? 5 : 4), key(k, k), -1, i, k);
      for (int64_t i = k + 1; i < T; ++i) {
        compute(K_SYRK, i, i, k, P(i == k + 1 ? 5 : level(i - k)), key(i, k), -1, i, i);
        for (int64_t j = k + 1; j < i; ++j) {
          if (!merged(j, k)) {
            compute(K_GEMM, i, j, k, P(level(j - k)), key(i, k), key(j, k), i, j);
          } else if (k % G == G - 1) {  // the group's last panel: all G updates now
            const int64_t f = k - G + 1;
            int64_t x[6];
            for (int64_t u = 1; u < G; ++u) {
              x[2 * (u - 1)] = key(i, f + u);
              x[2 * (u - 1) + 1] = key(j, f + u);
            }
            compute(K_GEMM, i, j, f, P(level(j - k)), key(i, f), key(j, f), i, j, (int)G, x);
          }
        }      }
      if (!p.opt.lookahead && k + 1 < T) {
        std::vector<Access> acc;
        for (int64_t d = 0; d < p.ntiles(); ++d) acc.push_back({d, RW});
        Task f{K_FENCE, (int32_t)k, (int32_t)k, (int32_t)k, 0, 1, 0, {-1, -1}, -1};
        submit(f, acc.data(), (int)acc.size());
      }
    }
    if (p.opt.with_store)
      for (int64_t j = 0; j < T; ++j)
        for (int64_t i = j; i < T; ++i) store(i, j);
  }

  // the same tasks in another program order (dev_order 1): seq holds
  // (kind, i, j, k) in any order in which every tile receives its updates
  // k = 0, 1, ... and then its TRSM, so the STF rule infers the same DAG
  template <class Seq>
  void run_seq(const Seq& seq) {
    p.buffers.clear();
    for (int64_t i = 0; i < T; ++i)
      for (int64_t j = 0; j <= i; ++j) p.buffers.push_back(Buffer{(int32_t)i, (int32_t)j, p.owner(i, j), false});
    auto key = [&](int64_t i, int64_t j) { return i * T + j; };
    const bool prio = p.opt.priority;
    auto level = [&](int64_t d) -> int { return d <= 1 ? 4 : d == 2 ? 3 : d <= 4 ? 2 : d <= 8 ? 1 : 0; };
    auto P = [&](int lv) { return prio ? lv : 0; };
    for (const auto& c : seq) {
      const int64_t i = c.i, j = c.j, k = c.k;
      if (c.kind == K_POTRF) compute(K_POTRF, k, k, k, P(5), -1, -1, k, k);
      else if (c.kind == K_TRSM) compute(K_TRSM, i, k, k, P(i == k + 1 ? 5 : 4), key(k, k), -1, i, k);
      else if (c.kind == K_SYRK) compute(K_SYRK, i, i, k, P(i == k + 1 ? 5 : level(i - k)), key(i, k), -1, i, i);
      else compute(K_GEMM, i, j, k, P(level(j - k)), key(i, k), key(j, k), i, j);
    }
  }

  // write-back of the final tile (i, j); on the other copy stream than the slot's
  // loads, so a write-back starts as soon as its tile is final instead of queueing
  // behind every load
  void store(int64_t i, int64_t j) {
    const int own = p.owner(i, j);
    const int64_t d = Plan::tile_id(i, j);
    Task t{K_STORE, (int32_t)i, (int32_t)j, 0, own, 0, copy_stream(own + (p.opt.store_own_stream ? 1 : 0)),
           {d, -1}, -1};
    Access acc[1] = {{d, READ}};
    submit(t, acc, 1);
    p.nstores++;
  }
};

}  // namespace

// ------------------------------------------------------------------ NEXT-4
// Memory-capped (out-of-core) plan: the matrix stays in the
// caller's host memory and only `F` device tile frames exist.  The STF rule
// does all the synchronisation: each frame is a logical datum (a compute task
// accesses the frame holding its tile with the tile's mode), each host tile is
// another one; LOAD(tile -> frame f) reads the host tile and writes frame f,
// STORE(frame f -> tile) reads frame f and writes the host tile.  Reusing a
// frame therefore waits for the previous occupant's readers (WAR) and writer
// (WAW), and a reload waits for the eviction's write-back (RAW).
//
// Program order.  Any order in which every task follows the tasks whose
// outputs it reads gives the same DAG up to frame edges and bit-identical
// results (each tile still receives its updates k = 0, 1, ... in order).  For
// traffic the plan uses a left-looking super-column order: columns are taken
// in blocks [j0, j1] whose tiles fit in about half of the frames; the block
// first receives all updates from columns k < j0 (k outer, so each panel tile
// L_ik is loaded once per block), then is factored right-looking inside.
// Each tile is written back once; reads of earlier panels cost about
// 8 nb^2 bytes per w*2 nb^3 flops for a block of width w.
// Eviction is Belady's (furthest next use in program order), never a frame the
// current task uses.
namespace {
struct OocBuilder {
  Plan& p;
  const int64_t T;
  const int64_t F;
  struct CT {
    int32_t kind, i, j, k, prio;
    int64_t r0, r1, w;  // tile ids read (or -1) and written
  };
  std::vector<CT> seq;
  std::vector<std::vector<Access>> accs;  // per task, for a re-ordered re-submission

  OocBuilder(Plan& plan, int64_t T_, int64_t F_) : p(plan), T(T_), F(F_) {}

  int64_t id(int64_t i, int64_t j) const { return Plan::tile_id(i, j); }

  // updates from column k to columns j0..j1.  Column j0 is the next to be
  // factored: its updates are critical (high-priority streams), so they are not
  // queued behind the wider block's updates in the bulk streams' FIFO order.
  void emit_updates_from(int64_t k, int64_t j0, int64_t j1) {
    for (int64_t j = j0; j <= j1; ++j) {
      const int d = (int)(j - j0);
      seq.push_back({K_SYRK, (int32_t)j, (int32_t)j, (int32_t)k, d == 0 ? 5 : d == 1 ? 3 : 2, id(j, k), -1, id(j, j)});
      for (int64_t i = j + 1; i < T; ++i)
        seq.push_back({K_GEMM, (int32_t)i, (int32_t)j, (int32_t)k, d == 0 ? 4 : d == 1 ? 2 : 1, id(i, k), id(j, k),
                       id(i, j)});
    }
  }

  void make_sequence() {
    int64_t j0 = 0;
    while (j0 < T) {
      // widest block whose tiles use at most half the frames (at least one column)
      int64_t j1 = j0, used = T - j0;
      while (j1 + 1 < T && used + (T - j1 - 1) <= F / 2) used += T - (++j1);
      for (int64_t k = 0; k < j0; ++k) emit_updates_from(k, j0, j1);
      for (int64_t j = j0; j <= j1; ++j) {
        seq.push_back({K_POTRF, (int32_t)j, (int32_t)j, (int32_t)j, 5, -1, -1, id(j, j)});
        for (int64_t i = j + 1; i < T; ++i)
          seq.push_back({K_TRSM, (int32_t)i, (int32_t)j, (int32_t)j, i == j + 1 ? 5 : 4, id(j, j), -1, id(i, j)});
        if (j < j1) emit_updates_from(j, j + 1, j1);
      }
      j0 = j1 + 1;
    }
  }

  // 2D-blocked order (ooc_order 1).  A tall super-column of width w re-reads
  // about 1/w panel tiles per update; when the trailing column alone fills the
  // budget, w is 1.  Here the block [j0, j1] is processed in row chunks of
  // height r: the diagonal triangle first (all updates from k < j0, then
  // factored right-looking inside), then each chunk of rows below it: updates
  // from k < j0 (k outer: r + w panel tiles per k for r w GEMMs), then its
  // TRSMs against the block's diagonal and the block-internal updates.  Every
  // tile still receives its updates k = 0, 1, ... in order and then its TRSM,
  // so L is bit-identical.  (w, r) minimise 1/w + 1/r under
  // w(w+1)/2 + r w <= 3F/5 (the other frames stream panel tiles; 3/5 gave
  // the fewest loads over F = 33..396 at T = 32 among 30..70%, and time within
  // 3% of the best of 40..80% at F = 33, 66, 132); a single
  // chunk is the tall super-column.
  void choose_block(int64_t j0, int64_t& w_out, int64_t& r_out) const {
    const int64_t B = std::max<int64_t>(F * p.opt.ooc_budget_pct / 100, 1);
    double best = 1e30;
    w_out = 1;
    r_out = T - j0 - 1;
    for (int64_t w = 1; w <= T - j0; ++w) {
      const int64_t rest = T - j0 - w;  // rows below the block
      const int64_t tri = w * (w + 1) / 2;
      if (tri > B && w > 1) break;
      int64_t r = rest == 0 ? 0 : std::min(rest, std::max<int64_t>((B - tri) / w, 1));
      const double cost = 1.0 / (double)w + (rest > 0 ? 1.0 / (double)r : 0.0);
      if (cost < best - 1e-12) {
        best = cost;
        w_out = w;
        r_out = r;
      }
    }
  }

  void make_sequence_2d() {
    int64_t j0 = 0;
    while (j0 < T) {
      int64_t w, r;
      choose_block(j0, w, r);
      const int64_t j1 = j0 + w - 1;
      // diagonal triangle of the block
      for (int64_t k = 0; k < j0; ++k)
        for (int64_t j = j0; j <= j1; ++j) {
          const int d = (int)(j - j0);
          seq.push_back({K_SYRK, (int32_t)j, (int32_t)j, (int32_t)k, d == 0 ? 5 : d == 1 ? 3 : 2, id(j, k), -1, id(j, j)});
          for (int64_t i = j + 1; i <= j1; ++i)
            seq.push_back({K_GEMM, (int32_t)i, (int32_t)j, (int32_t)k, d == 0 ? 4 : d == 1 ? 2 : 1, id(i, k), id(j, k),
                           id(i, j)});
        }
      for (int64_t j = j0; j <= j1; ++j) {
        seq.push_back({K_POTRF, (int32_t)j, (int32_t)j, (int32_t)j, 5, -1, -1, id(j, j)});
        for (int64_t i = j + 1; i <= j1; ++i)
          seq.push_back({K_TRSM, (int32_t)i, (int32_t)j, (int32_t)j, i == j + 1 ? 5 : 4, id(j, j), -1, id(i, j)});
        for (int64_t jj = j + 1; jj <= j1; ++jj) {
          seq.push_back({K_SYRK, (int32_t)jj, (int32_t)jj, (int32_t)j, jj == j + 1 ? 5 : 3, id(jj, j), -1, id(jj, jj)});
          for (int64_t i = jj + 1; i <= j1; ++i)
            seq.push_back({K_GEMM, (int32_t)i, (int32_t)jj, (int32_t)j, jj == j + 1 ? 4 : 2, id(i, j), id(jj, j),
                           id(i, jj)});
        }
      }
      // row chunks below it
      for (int64_t i0 = j1 + 1; i0 < T; i0 += r) {
        const int64_t i1 = std::min(T - 1, i0 + r - 1);
        for (int64_t k = 0; k < j0; ++k)
          for (int64_t j = j0; j <= j1; ++j)
            for (int64_t i = i0; i <= i1; ++i)
              seq.push_back({K_GEMM, (int32_t)i, (int32_t)j, (int32_t)k, j == j0 ? 2 : 1, id(i, k), id(j, k), id(i, j)});
        for (int64_t j = j0; j <= j1; ++j) {
          for (int64_t i = i0; i <= i1; ++i)
            seq.push_back({K_TRSM, (int32_t)i, (int32_t)j, (int32_t)j, 4, id(j, j), -1, id(i, j)});
          for (int64_t jj = j + 1; jj <= j1; ++jj)
            for (int64_t i = i0; i <= i1; ++i)
              seq.push_back({K_GEMM, (int32_t)i, (int32_t)jj, (int32_t)j, jj == j + 1 ? 2 : 1, id(i, j), id(jj, j),
                             id(i, jj)});
        }
      }
      j0 = j1 + 1;
    }
  }

  void run(int crit_streams, int bulk_streams, int load_stream, int store_stream, bool serial, bool priority,
           int order) {
    if (order == 1)
      make_sequence_2d();
    else
      make_sequence();
    const int64_t NT = p.ntiles();
    p.buffers.clear();
    for (int64_t f = 0; f < F; ++f) p.buffers.push_back(Buffer{-1, -1, 0, false});
    auto host = [&](int64_t t) { return F + t; };  // datum id of the caller's copy of tile t
    // next-use bookkeeping for Belady
    std::vector<std::vector<int64_t>> uses((size_t)NT);
    for (size_t q = 0; q < seq.size(); ++q)
      for (int64_t t : {seq[q].r0, seq[q].r1, seq[q].w})
        if (t >= 0) uses[(size_t)t].push_back((int64_t)q);
    std::vector<size_t> ptr((size_t)NT, 0);
    const int64_t kNever = INT64_MAX;
    auto next_use = [&](int64_t t, int64_t after) -> int64_t {
      auto& u = uses[(size_t)t];
      size_t& k = ptr[(size_t)t];
      while (k < u.size() && u[k] <= after) ++k;
      return k < u.size() ? u[k] : kNever;
    };
    std::vector<int64_t> frame_of((size_t)NT, -1), tile_in((size_t)F, -1);
    std::vector<char> dirty((size_t)F, 0);
    std::set<std::pair<int64_t, int64_t>> resident;  // (next use, tile)
    std::vector<int64_t> key((size_t)NT, 0);
    std::vector<int64_t> free_frames;
    for (int64_t f = F - 1; f >= 0; --f) free_frames.push_back(f);
    int32_t ij[2];
    auto tile_ij = [&](int64_t t) {
      int64_t i = 0;
      while ((i + 1) * (i + 2) / 2 <= t) ++i;
      ij[0] = (int32_t)i;
      ij[1] = (int32_t)(t - i * (i + 1) / 2);
    };
    auto store = [&](int64_t f) {
      tile_ij(tile_in[(size_t)f]);
      Task s{K_STORE, ij[0], ij[1], 0, 0, 0, store_stream, {f, -1}, -1};
      Access acc[2] = {{f, READ}, {host(tile_in[(size_t)f]), WRITE}};
      p.graph.submit(acc, 2);
      accs.emplace_back(acc, acc + 2);
      p.tasks.push_back(s);
      p.nstores++;
      dirty[(size_t)f] = 0;
    };
    auto compute_stream = [&](const CT& c) -> int {
      if (serial) return 0;
      if (priority && c.prio >= 4) return crit_stream(c, crit_streams);
      return crit_streams + (int)((c.i * T + c.j) % bulk_streams);
    };
    for (size_t q = 0; q < seq.size(); ++q) {
      const CT& c = seq[q];
      const int64_t need[3] = {c.r0, c.r1, c.w};
      for (int a = 0; a < 3; ++a) {
        const int64_t t = need[a];
        if (t < 0 || frame_of[(size_t)t] >= 0) continue;
        int64_t f;
        if (!free_frames.empty()) {
          f = free_frames.back();
          free_frames.pop_back();
        } else {
          // furthest next use among residents the current task does not touch
          // (F >= 3 guarantees one: a task touches at most 3 tiles; build_plan rejects F < 3)
          auto it = resident.end();
          do {
            --it;
          } while (it != resident.begin() &&
                   (it->second == need[0] || it->second == need[1] || it->second == need[2]));
          const int64_t v = it->second;
          resident.erase(it);
          f = frame_of[(size_t)v];
          if (dirty[(size_t)f]) store(f);
          frame_of[(size_t)v] = -1;
          tile_in[(size_t)f] = -1;
        }
        tile_ij(t);
        Task l{K_LOAD, ij[0], ij[1], 0, 0, priority ? c.prio : 0, load_stream, {-1, -1}, f};
        Access acc[2] = {{host(t), READ}, {f, WRITE}};
        p.graph.submit(acc, 2);
        accs.emplace_back(acc, acc + 2);
        p.tasks.push_back(l);
        p.nloads++;
        frame_of[(size_t)t] = f;
        tile_in[(size_t)f] = t;
        key[(size_t)t] = -1;  // inserted below with its next use
      }
      // the task itself
      Task t{c.kind, c.i, c.j, c.k, 0, priority ? c.prio : 0, 0,
             {c.r0 >= 0 ? frame_of[(size_t)c.r0] : -1, c.r1 >= 0 ? frame_of[(size_t)c.r1] : -1},
             frame_of[(size_t)c.w]};
      t.stream = compute_stream(c);
      Access acc[3];
      int n = 0;
      if (t.in[0] >= 0) acc[n++] = {t.in[0], READ};
      if (t.in[1] >= 0) acc[n++] = {t.in[1], READ};
      acc[n++] = {t.out, RW};
      p.graph.submit(acc, n);
      accs.emplace_back(acc, acc + n);
      p.tasks.push_back(t);
      dirty[(size_t)t.out] = 1;
      // refresh the next-use keys of the tiles just used
      for (int a = 0; a < 3; ++a) {
        const int64_t x = need[a];
        if (x < 0) continue;
        if (key[(size_t)x] >= 0) resident.erase({key[(size_t)x], x});
        key[(size_t)x] = next_use(x, (int64_t)q);
        resident.insert({key[(size_t)x], x});
      }
    }
    // write back what is still dirty
    for (int64_t f = 0; f < F; ++f)
      if (tile_in[(size_t)f] >= 0 && dirty[(size_t)f]) store(f);
  }
};
}  // namespace

// Submission order by earliest start.  The CUDA graph executor (and the eager
// stream queues) only look a bounded distance ahead in submission order, so a
// task submitted far behind tasks that wait on late transfers starts late even
// when its own inputs are ready (measured: with the loads first and the
// write-backs last, the first compute of a HOST_COLMAJOR call started 30 ms in
// and the first write-back 256 ms in).  The tasks are re-submitted in the order
// of their earliest start in a model with unlimited compute, one transfer at a
// time per copy stream (a tile copy = copy_cost GEMM-tile times) and unit-ish
// compute costs; ties keep program order.  Any topological order of the DAG
// re-submitted through the STF rule yields the same DAG (conflicting accesses
// keep their relative order), so only the stream-order chains change.
static void reorder_asap(Plan& plan, const std::vector<std::vector<Access>>& accs, int64_t ndata) {
  const size_t n = plan.tasks.size();
  const double copy_cost = plan.opt.copy_cost > 0 ? plan.opt.copy_cost : 2.7;
  auto cost = [&](const Task& t) -> double {
    switch (t.kind) {
      case K_POTRF: return 5.0;
      case K_TRSM: return 2.0;
      case K_SYRK:
      case K_GEMM: return 1.0;
      case K_COPY:
      case K_LOAD:
      case K_STORE: return copy_cost;
      default: return 0.01;
    }
  };
  std::vector<double> start(n, 0.0), fin(n, 0.0);
  std::vector<double> qfree;  // per (slot, stream) for transfers
  for (size_t t = 0; t < n; ++t) {
    const Task& k = plan.tasks[t];
    double s0 = 0.0;
    for (const int64_t* q = plan.graph.preds_begin((int64_t)t); q != plan.graph.preds_end((int64_t)t); ++q)
      s0 = std::max(s0, fin[(size_t)*q]);
    if (k.kind == K_COPY || k.kind == K_LOAD || k.kind == K_STORE) {
      const size_t key = (size_t)k.slot * 64 + (size_t)k.stream;
      if (qfree.size() <= key) qfree.resize(key + 1, 0.0);
      s0 = std::max(s0, qfree[key]);
      qfree[key] = s0 + cost(k);
    }
    start[t] = s0;
    fin[t] = s0 + cost(k);
  }
  std::vector<size_t> ord(n);
  for (size_t t = 0; t < n; ++t) ord[t] = t;
  std::stable_sort(ord.begin(), ord.end(), [&](size_t a, size_t b) { return start[a] < start[b]; });
  std::vector<Task> tasks(n);
  TaskGraph g(ndata);
  for (size_t r = 0; r < n; ++r) {
    tasks[r] = plan.tasks[ord[r]];
    g.submit(accs[ord[r]].data(), (int)accs[ord[r]].size());
  }
  plan.tasks.swap(tasks);
  plan.graph = std::move(g);
}

// Submission order by simulated list scheduling (order_mode 2): each GPU slot
// runs at most `width` compute tasks at a time, transfers one at a time per copy
// stream; among ready compute tasks the one with the longest remaining path
// (bottom level, in the cost units of reorder_asap) starts first.  Tasks are
// re-submitted in order of simulated start, so the bounded look-ahead of the
// graph executor / stream queues sees the tasks the GPU will run next - the
// panel chain before the bulk updates of the same step.  A topological order,
// so the DAG is unchanged (see reorder_asap).
static void reorder_list(Plan& plan, const std::vector<std::vector<Access>>& accs, int64_t ndata, int width,
                         int64_t tail_steps) {
  const size_t n = plan.tasks.size();
  // tail_steps > 0: only the tasks from POTRF(T - tail_steps) on (a suffix of the
  // program order) are re-ordered; the prefix keeps program order
  size_t first = 0;
  if (tail_steps > 0 && tail_steps < plan.T)
    for (size_t t = 0; t < n; ++t)
      if (plan.tasks[t].kind == K_POTRF && plan.tasks[t].k == plan.T - tail_steps) {
        first = t;
        break;
      }
  const double copy_cost = plan.opt.copy_cost > 0 ? plan.opt.copy_cost : 2.7;
  auto is_copy = [](int32_t k) { return k == K_COPY || k == K_LOAD || k == K_STORE; };
  auto cost = [&](const Task& t) -> double {
    switch (t.kind) {
      case K_POTRF: return 5.0;
      case K_TRSM: return 2.0;
      case K_SYRK:
      case K_GEMM: return 1.0;
      case K_COPY:
      case K_LOAD:
      case K_STORE: return copy_cost;
      default: return 0.01;
    }
  };
  std::vector<int64_t> soff, succ;
  plan.graph.build_successors(soff, succ);
  std::vector<double> bl(n, 0.0);
  for (size_t t = n; t-- > 0;) {
    double m = 0.0;
    for (int64_t e = soff[t]; e < soff[t + 1]; ++e) m = std::max(m, bl[(size_t)succ[(size_t)e]]);
    bl[t] = cost(plan.tasks[t]) + m;
  }
  std::vector<int64_t> npred(n, 0);
  for (size_t t = 0; t < n; ++t) npred[t] = plan.graph.preds_end((int64_t)t) - plan.graph.preds_begin((int64_t)t);
  int nslots = 1;
  for (const Task& t : plan.tasks) nslots = std::max(nslots, t.slot + 1);
  auto cmp_ready = [&](size_t a, size_t b) { return bl[a] < bl[b] || (bl[a] == bl[b] && a > b); };
  std::vector<std::priority_queue<size_t, std::vector<size_t>, decltype(cmp_ready)>> ready;
  for (int s = 0; s < nslots; ++s) ready.emplace_back(cmp_ready);
  std::vector<int> busy((size_t)nslots, 0);
  typedef std::pair<double, size_t> Ev;  // (finish time, task)
  std::priority_queue<Ev, std::vector<Ev>, std::greater<Ev>> events;
  std::vector<double> qfree;
  std::vector<double> start(n, 0.0);
  double now = 0.0;
  auto release = [&](size_t t) {
    const Task& k = plan.tasks[t];
    if (is_copy(k.kind)) {
      const size_t key = (size_t)k.slot * 64 + (size_t)k.stream;
      if (qfree.size() <= key) qfree.resize(key + 1, 0.0);
      start[t] = std::max(now, qfree[key]);
      qfree[key] = start[t] + cost(k);
      events.push(Ev(qfree[key], t));
    } else {
      ready[(size_t)k.slot].push(t);
    }
  };
  for (size_t t = 0; t < n; ++t)
    if (npred[t] == 0) release(t);
  size_t done = 0;
  while (done < n) {
    for (int s = 0; s < nslots; ++s)
      while (busy[(size_t)s] < width && !ready[(size_t)s].empty()) {
        const size_t t = ready[(size_t)s].top();
        ready[(size_t)s].pop();
        start[t] = now;
        busy[(size_t)s]++;
        events.push(Ev(now + cost(plan.tasks[t]), t));
      }
    if (events.empty()) break;  // cannot happen for a DAG
    const Ev ev = events.top();
    events.pop();
    now = ev.first;
    const size_t t = ev.second;
    ++done;
    if (!is_copy(plan.tasks[t].kind)) busy[(size_t)plan.tasks[t].slot]--;
    for (int64_t e = soff[t]; e < soff[t + 1]; ++e) {
      const size_t u = (size_t)succ[(size_t)e];
      if (--npred[u] == 0) release(u);
    }
  }
  std::vector<size_t> ord(n);
  for (size_t t = 0; t < n; ++t) ord[t] = t;
  std::stable_sort(ord.begin() + (ptrdiff_t)first, ord.end(), [&](size_t a, size_t b) { return start[a] < start[b]; });
  std::vector<Task> tasks(n);
  TaskGraph g(ndata);
  for (size_t r = 0; r < n; ++r) {
    tasks[r] = plan.tasks[ord[r]];
    g.submit(accs[ord[r]].data(), (int)accs[ord[r]].size());
  }
  plan.tasks.swap(tasks);
  plan.graph = std::move(g);
}

void build_plan(Plan& plan, int64_t T, const PlanOptions& opt) {
  plan.T = T;
  plan.opt = opt;
  if (plan.opt.crit_streams < 1) plan.opt.crit_streams = 1;
  if (plan.opt.bulk_streams < 1) plan.opt.bulk_streams = 1;
  if (plan.opt.copy_streams < 1) plan.opt.copy_streams = 1;
  plan.tasks.clear();
  plan.ntransfers = 0;
  plan.npushed = 0;
  plan.nmerged = 0;
  plan.nloads = 0;
  plan.nstores = 0;
  plan.replicas_per_slot.assign((size_t)opt.nslots, 0);
  const int64_t NT = T * (T + 1) / 2;
  if (opt.frames > 0 && opt.frames < 3) plan.opt.frames = 3;  // a GEMM holds 3 tiles (callers validate F >= 3)
  if (plan.opt.frames > 0 && opt.nslots == 1 && opt.with_load && opt.with_store) {
    // out-of-core: datum ids = frames, then the caller's host tiles
    plan.graph = TaskGraph(plan.opt.frames + NT + 1);
    const int base = plan.opt.stream_pool ? (plan.opt.stream_pool == 1 ? 1 : 0)
                     : plan.opt.serial ? 1 : plan.opt.crit_streams + plan.opt.bulk_streams;
    const int store = plan.opt.stream_pool ? base : base + (plan.opt.copy_streams > 1 ? 1 : 0);
    OocBuilder b(plan, T, plan.opt.frames);
    b.run(plan.opt.crit_streams, plan.opt.bulk_streams, base, store, plan.opt.serial || plan.opt.stream_pool != 0,
          plan.opt.priority,
          // auto: 2D-blocked for re-ordered plans (n = 32768, nb = 1024: F = 33..396 all
          // ahead of the tall order); in program order only while less than half the
          // tiles fit (F = 33 / 66 / 132 +58% / +42% / +2%, F = 264 -1.6%)
          plan.opt.ooc_order >= 0 ? plan.opt.ooc_order
                                  : ((opt.order_mode == 2 && opt.ooc_reorder) || 2 * plan.opt.frames < NT ? 1 : 0));
    if (opt.order_mode == 2 && opt.ooc_reorder)
      reorder_list(plan, b.accs, plan.opt.frames + NT + 1, opt.sched_width > 0 ? opt.sched_width : 2, 0);
  } else {
    plan.opt.frames = 0;
    // dense datum ids: home tiles + at most one replica per (tile, slot)
    plan.graph = TaskGraph(NT + NT * opt.nslots + 1);
    Builder b(plan, T);
    if (opt.dev_order == 1 && !opt.with_load && !opt.with_store && opt.lookahead) {
      OocBuilder ob(plan, T, NT);  // 2D-blocked left-looking order, block budget from all tiles
      ob.make_sequence_2d();
      b.run_seq(ob.seq);
    } else {
      b.run();
    }
    if (opt.order_mode == 2)
      reorder_list(plan, b.accs, NT + NT * opt.nslots + 1, opt.sched_width > 0 ? opt.sched_width : 2, opt.order_tail);
    else if (opt.order_asap) reorder_asap(plan, b.accs, NT + NT * opt.nslots + 1);
  }
  // longest chain of compute tasks (COPY/LOAD/STORE weigh 0)
  std::vector<int64_t> depth(plan.tasks.size(), 0);
  int64_t best = 0;
  for (size_t t = 0; t < plan.tasks.size(); ++t) {
    int64_t d = 0;
    for (const int64_t* q = plan.graph.preds_begin((int64_t)t); q != plan.graph.preds_end((int64_t)t); ++q)
      d = std::max(d, depth[(size_t)*q]);
    const int32_t kd = plan.tasks[t].kind;
    depth[t] = d + ((kd <= K_GEMM) ? 1 : 0);
    best = std::max(best, depth[t]);
  }
  plan.critical_path = best;
}

}  // namespace stf
