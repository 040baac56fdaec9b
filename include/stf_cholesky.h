/*
 * stf_cholesky.h -- C ABI of the B200-native STF tiled FP64 Cholesky library
 * (libstf_cholesky.so).  No C++ or torch types cross this boundary.
 *
 * What the library computes.  For a symmetric positive definite n x n matrix A
 * (FP64, lower triangle referenced), the lower-triangular L with positive
 * diagonal such that A = L * L^T ("Cholesky decomposition", PAPER.md:384 and
 * :393, §VII-C).  It is computed as the right-looking tiled algorithm of ref.
 * [17]: the matrix is cut into nb x nb tiles, "one logical data
 * object per tile", and the program-order sequence
 *     for k: POTRF(k); for i>k: TRSM(i,k); for i>k: { SYRK(i,k); for k<j<i: GEMM(i,j,k) }
 * is turned into a task DAG purely from each task's read / read-write access
 * to tiles -- the Sequential Task Flow rule of PAPER.md:144 (§II-B): a task
 * depends on the previous tasks that modify its data and, if it modifies a
 * datum, on all previous readers of it.  The DAG runs asynchronously on 1..8
 * GPUs of one node, driven by ONE host process, with tiles
 * distributed 2D block-cyclically and finished tiles pushed to the GPUs that
 * read them (the MSI replicas of PAPER.md:210-216).  stf_potrf returns after
 * all work (and any write-back) has completed.
 *
 * Errors (LAPACK style).  Every function returns 0 on success.
 *   -1 n < 0;  -2 nb < 1, nb odd, or n % nb != 0;  -3 uplo not 'L'/'l'/'U'/'u'
 *   (or 'U' with a TILED descriptor);  -4 bad descriptor;  -5 bad ngpus
 *   -100 not initialised;  -101 CUDA error;  -103 device out of memory;
 *   -104 already initialised;  -105 bad option name / value.
 *   > 0 (stf_potrf only): the leading minor of that order is not positive
 *   definite (first failing global column, 1-based); A is then unspecified.
 * stf_last_error() returns a thread-local, NUL-terminated description of the
 * last non-zero return on the calling thread ("" if none).  The pointer stays
 * valid until the next library call on that thread.
 *
 * Threading: calls are serialised by an internal mutex; stf_potrf is not
 * re-entrant.  Stream ordering: a factorisation starts after all work the caller
 * enqueued before the call on the legacy default stream and on the calling
 * thread's per-thread default stream of every participating device (the library
 * records events there and its launch stream waits on them); work on other caller
 * streams must be synchronised by the caller.  It returns after all of its own
 * device work has completed.  Ownership: the caller owns A (and every tile) in all modes and
 * must not touch it during a call; the library owns its streams, events,
 * graphs, replicas and workspaces from stf_cholesky_init to stf_finalize.
 */
#ifndef STF_CHOLESKY_H
#define STF_CHOLESKY_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Matrix descriptor kinds. */
enum {
  /* Tiles already resident on their owners: tiles[i + j*T] (i >= j, T = n/nb)
   * is a device pointer to the nb x nb column-major tile A_ij (ld = nb) on GPU
   * slot (i % p) * q + (j % q); entries with i < j are ignored (may be NULL).
   * The headline benchmark layout (cuSolverMg-like pre-distributed input). */
  STF_DESC_TILED_2DBC = 0,
  /* ptr = device pointer (on CUDA device `device`) to an n x n column-major
   * matrix with leading dimension ld >= max(1, n).  Converted into library
   * tiles by copy tasks, factored, written back by copy tasks. */
  STF_DESC_DEVICE_COLMAJOR = 1,
  /* ptr = host pointer to an n x n column-major matrix (ld >= max(1, n));
   * page-locked memory (cudaHostAlloc / cudaHostRegister) is strongly
   * recommended: host<->device copies are tasks overlapped with the
   * factorisation and are only asynchronous from pinned memory. */
  STF_DESC_HOST_COLMAJOR = 2
};

typedef struct stf_matrix_desc {
  int32_t kind;         /* STF_DESC_* */
  int32_t device;       /* DEVICE_COLMAJOR: CUDA ordinal holding ptr */
  int64_t ld;           /* COLMAJOR: leading dimension (elements) */
  double *ptr;          /* COLMAJOR: the matrix; caller-owned */
  int32_t p, q;         /* TILED_2DBC: process grid, p * q == ngpus */
  double *const *tiles; /* TILED_2DBC: host array of T*T device pointers; caller-owned */
} stf_matrix_desc;

/* Initialise the library on `ngpus` GPU slots.  device_ids (length ngpus) maps
 * slot s -> CUDA ordinal; NULL means 0..ngpus-1.  An ordinal may repeat: slots
 * sharing a device are "virtual GPUs" with their own streams and replicas, so
 * the multi-GPU distribution and transfer logic runs (and is tested) on one
 * physical B200 (SURVEY.md §4.2 "virtual multi-GPU").  Enables peer access
 * between distinct devices, creates per-slot stream pools.
 * Returns 0, -5 (bad ngpus/ordinal), -101, or -104 if already initialised. */
int stf_cholesky_init(int ngpus, const int *device_ids);

/* Factorise A = L L^T (uplo 'L') or A = U^T U (uplo 'U', COLMAJOR kinds only;
 * U = L^T).  n >= 0, nb >= 2 even, n % nb == 0.  ngpus (1..initialised slots)
 * selects the slots 0..ngpus-1; for TILED_2DBC p*q must equal ngpus; for
 * COLMAJOR kinds the grid is p x q with p <= q, p maximal (1x1, 1x2, 2x2, 2x4)
 * unless STF_GRID / stf_set_option("grid_p") overrides.  Synchronous: on return
 * the lower (upper) triangle of A holds L (U); the strictly upper (lower)
 * triangle is neither read nor written.  n == 0 returns 0 at once. */
int stf_potrf(int64_t n, int64_t nb, char uplo, stf_matrix_desc *A_desc, int ngpus);

/* Destroy every library resource (graphs, streams, events, replicas, plans). */
int stf_finalize(void);

const char *stf_last_error(void);

/* ---------------------------------------------------------------- options
 * Execution options.  Each is read once from the environment at init (the
 * variable in the second column) and settable here; every option except
 * "threads" and "grid_p" is part of the memo key of a plan, so a plan or graph
 * built under one value is never reused under another.  Out-of-range values
 * (from either source) are rejected with -105.
 *   "dataflow" STF_DATAFLOW POTRF tile kernel: 1 single-launch dataflow (default), 0 recursive
 *   "trsm"     STF_TRSM     TRSM tile kernel: 3 (default) = resident panel for the critical
 *                           TRSM(k+1,k) when nb <= 1024 and nb % 64 == 0, row panel otherwise;
 *                           2 row panel, 1 dataflow, 0 recursive
 *   "trsm_split" STF_TRSM_SPLIT P in [1,16]: non-critical row-panel TRSMs run right-looking
 *                           over P column blocks (panel kernel + GEMM updates; default 4)
 *   "trsm_res_tail" STF_TRSM_RES_TAIL C >= 0: with trsm 3, every TRSM(i,k) of a panel step
 *                           whose trailing order n - k nb <= C uses the resident panel
 *                           (-1 default: 4096 at nb >= 1024, n = 8192 +7%; 8192 below, nb = 512
 *                           +6%; profiles/r02/pdl_and_tail.txt, split_potrf.txt)
 *   "trsm_res_split" STF_TRSM_RES_SPLIT 2 (default) or 4: a resident-panel TRSM runs as that many
 *                           column parts, right-looking, with a GEMM after each (more CTAs on the
 *                           critical path); 1: one launch
 *   "gemm_merge" STF_GEMM_MERGE D >= 0 (default 2): the tile updates GEMM(i,j,k) of a group of
 *                           G consecutive panels k = gG .. gG+G-1 ("gemm_group" G = 2..4; default
 *                           -1: 4 when n/nb >= 48, else 2) become ONE task at step gG+G-1 when the tile is at least D columns
 *                           right of that panel (one k sweep of G nb: one C load/store and
 *                           pipeline ramp instead of G; the same operations per element, same
 *                           bits); 0 = off.  Not with lookahead = 0.
 *   "trsm_rows" STF_TRSM_ROWS 32, 64 or 128 (default): rows per CTA of the row-panel TRSM
 *   "graph"    STF_GRAPH    1: capture the whole task DAG of a call into one CUDA graph,
 *                           memoised per (n, nb, grid, tiles, options) (default); 0: eager
 *                           lowering on streams + events.  A capture the driver rejects falls
 *                           back to eager (stf_plan_stats.graph_fallback = 1)
 *   "streams"  STF_STREAMS  bulk compute streams per GPU slot (default 32; pool sized at init)
 *   "stream_pool" STF_STREAM_POOL 0 (default): 6 high-priority + "streams" bulk + 2 copy streams
 *                           per slot; 1: one compute stream + one copy stream per slot; 2: one
 *                           stream per slot for everything (ablations of PAPER.md:401, :407)
 *   "serial"   STF_SERIAL   1: every compute task on one stream in program order (race check)
 *   "priority" STF_PRIO     1: critical-path tasks on high-priority streams (default 1)
 *   "prio_mode" STF_PRIO_MODE  priority level assignment variant (0 default; 1..3 ablations)
 *   "grid_p"   STF_GRID     rows P of the P x Q grid for COLMAJOR kinds (0 = auto)
 *   "push"     STF_PUSH     data plane of the finished-tile broadcast (NEXT-3):
 *                           0 (default) COPY tasks on the producer's copy streams (copy engine);
 *                           1 fused push: the POTRF(k) / TRSM(i,k) epilogues store L_kk / L_ik
 *                           straight into every consumer's replica (peer stores over NVLink);
 *                           2 the same through one NVSwitch multicast object (multimem.st: one
 *                           store reaches every device) when the call spans >= 2 distinct
 *                           devices that support multicast, in single-process mode; else as 1
 *                           (stf_plan_stats.data_plane reports what ran)
 *   "threads"  STF_THREADS  eager backend: host submission threads, slots split round-robin
 *                           (default 8, capped at ngpus; the graph backend captures on one thread)
 *   "lookahead" STF_LOOKAHEAD 1: pure STF DAG (default); 0: a fence task closes every
 *                           panel step (no look-ahead; ablation of PAPER.md:399).  Rejected
 *                           (-105) for out-of-core plans and in multi-process mode
 *   "order_mode" STF_ORDER_MODE submission order: -1 auto (default: list scheduling for
 *                           nb >= 512, else program order), 0 program order, 2 list scheduling
 *   "order_tail" STF_ORDER_TAIL with list scheduling, re-order only the last C panel steps
 *                           (-1 auto: 8 for device tiles with T > 16, else all; 0 all)
 *   "order_asap" STF_ORDER_ASAP 1: earliest-start submission order (with order_mode 0)
 *   "sched_width" STF_SCHED_WIDTH list-scheduling model width (0 auto from nb and the SM count)
 *   "dev_order" STF_DEV_ORDER 1: device-resident plans in the 2D-blocked left-looking order
 *   "mem_cap_tiles" STF_MEM_CAP_TILES  0 (default) or >= 3: a HOST_COLMAJOR call on one GPU
 *                           keeps at most this many nb x nb tiles on the device (out-of-core,
 *                           NEXT-4): tiles are loaded on demand and dirty
 *                           tiles written back on eviction (Belady order).  A cap >= T(T+1)/2
 *                           tiles means no cap.  Rejected (-105) for HOST_COLMAJOR calls on
 *                           more than one GPU; ignored for device-resident kinds
 *   "ooc_order" STF_OOC_ORDER  program order of an out-of-core plan: 1 2D-blocked, 0 tall
 *                           super-columns, -1 (default) auto.  Every order gives bit-identical L
 *   "ooc_reorder" STF_OOC_REORDER 1 (default): out-of-core plans re-submitted in list order
 *   "ooc_budget_pct" STF_OOC_BUDGET_PCT block budget of the 2D order in % of the frames
 *                           (-1 auto: 90 once 3/4 of the tiles fit, else 60)
 *   "host_stream" STF_HOST_STREAM  1 (default): an uncapped HOST_COLMAJOR call on one GPU with
 *                           nb >= 512 and n/nb >= 16 (list order, lookahead, default stream
 *                           pool) is planned by the out-of-core builder with one frame per
 *                           tile (2D-blocked left-looking order, no eviction); 0: the
 *                           right-looking plan with its LOAD/STORE tasks.  Same bits
 *   "host_stream_budget_pct" STF_HOST_STREAM_BUDGET_PCT block budget of that plan (default 90)
 *   "host_eager" STF_HOST_EAGER 1: HOST_COLMAJOR calls on pinned memory lowered eagerly
 *   "pdl"      STF_PDL      1 (default): the panel chain POTRF(k) -> TRSM(k+1,k) -> SYRK(k+1,k)
 *                           overlaps through programmatic dependent launch when the three
 *                           share a slot and stream (graph backend, dataflow POTRF,
 *                           trsm = 3, nb % 64 == 0, nb <= 1024): the TRSM reads L_kk block by
 *                           block as the POTRF publishes it, the SYRK reads L_{k+1,k} column
 *                           block by column block as the TRSM's CTAs finish them (device
 *                           flags, acquire/release).  The TRSM(k+1,k) is then one
 *                           resident-panel launch (trsm_res_split does not apply to it) in
 *                           every grid, so the bits do not depend on where it runs; they
 *                           equal pdl = 0 with trsm_res_split = 1 (tested)
 *   "potrf_split" STF_POTRF_SPLIT 1 (default): a POTRF tile is two launches -- the critical-chain
 *                           CTA with a few block-task CTAs, then 2-per-SM block-task CTAs it
 *                           releases (programmatic launch; the first completes the tile alone
 *                           when launches are serialised); 0: one launch.  Same bits
 *   "potrf_ctas" STF_POTRF_CTAS CTAs of a POTRF tile launch (0 default: 3 per 64-block column,
 *                           16..96); the critical chain needs at least one block-task CTA
 *   "pdl_lead" STF_PDL_LEAD 64-block steps before its end at which a chain kernel lets its
 *                           dependent launch (-1 default: nb/128, at least 2; >= nb/64: at its
 *                           start)
 *   "debug_skip" STF_DEBUG_SKIP bit mask (or names potrf,trsm,syrk,gemm,copy,trsm_as_gemm,
 *                           trsm_as_half_gemm) of task kinds NOT launched: timing what-ifs only,
 *                           results invalid
 *   "debug_trace" STF_DEBUG_TRACE 1: timing events around every task (one slot), see
 *                           stf_debug_last_trace in stf_harness.h
 *   "nvtx"     STF_NVTX     1: an NVTX range per task submission ("GEMM(i,j,k)@slot", eager
 *                           backend) and one around each call's graph launch (profiler timelines)
 * Returns 0 or -105. */
int stf_set_option(const char *name, int64_t value);
int stf_get_option(const char *name, int64_t *value);

/* ---------------------------------------------------------------- introspection
 * Counts of the last stf_potrf call's plan (or of a DAG built without running,
 * see stf_dag_build).  Integer host work, compared bit-exactly with the oracle. */
typedef struct stf_plan_stats {
  int64_t tasks;          /* compute tasks (POTRF + TRSM + SYRK + GEMM) */
  int64_t transfers;      /* inter-slot tile transfers (COPY tasks + fused pushes) */
  int64_t edges;          /* DAG edges between all tasks (compute + transfer) */
  int64_t transfer_bytes; /* bytes moved between slots */
  int64_t critical_path;  /* longest chain of compute tasks (3T-2 when P=Q=1) */
  int64_t graph_nodes;    /* nodes of the captured CUDA graph (0 if eager) */
  int64_t kernel_launches;/* kernels launched by one factorisation */
  double build_ms;        /* host time to build the plan (0 on a memo hit) */
  double device_ms;       /* device time of the last call: CUDA events recorded on the
                             library's launch stream immediately before the graph launch
                             (eager: before the fork) and after the join */
  int64_t graph_reuse;    /* 0 new plan, 1 exact memo hit, 2 plan of the same shape re-bound
                             to new caller storage (graph refreshed by cudaGraphExecUpdate) */
  int64_t dag_tasks;      /* all DAG vertices: compute + COPY + LOAD/STORE + FENCE tasks */
  int64_t host_loads;     /* LOAD tasks: tiles copied from the caller's matrix (COLMAJOR kinds) */
  int64_t host_stores;    /* STORE tasks: tiles written back to the caller's matrix */
  int64_t frames;         /* device tile frames of an out-of-core plan ("mem_cap_tiles"), else 0 */
  int64_t pushed;         /* replicas written by fused epilogue pushes (part of transfers) */
  int64_t replicas_max;   /* largest number of replica tiles held by one slot */
  int64_t data_plane;     /* 0 COPY tasks (copy engine), 1 fused epilogue push (peer stores),
                             2 fused push through an NVSwitch multicast object */
  int64_t graph_fallback; /* 1: the graph capture was rejected and the eager backend ran */
  int64_t graph;          /* 1: the call ran as one CUDA graph launch, 0: eager streams */
  int64_t devices;        /* distinct CUDA devices spanned by the call's slots */
  int64_t slots;          /* GPU slots of the call (ngpus) */
  int64_t peer_transfers; /* transfers whose source and destination are distinct devices */
  int64_t merged_gemms;   /* GEMM tasks that carry two consecutive tile updates ("gemm_merge") */
  int64_t pdl_edges;      /* programmatic graph edges of the panel chain (option "pdl"): a TRSM(k+1,k)
                             or SYRK(k+1,k) that may launch before its producer ends */
} stf_plan_stats;

int stf_last_stats(stf_plan_stats *out);

/* Build (without running) the STF DAG of a T x T tile Cholesky on a p x q grid
 * and copy up to `cap` edges (src, dst pairs of task indices in submission
 * order) into edges[2*cap].  kinds[cap_tasks] receives per-task codes
 * (0 POTRF, 1 TRSM, 2 SYRK, 3 GEMM, 4 COPY, 5 LOAD, 6 STORE, 7 FENCE) and ijk[3*cap_tasks]
 * the (i, j, k) indices (for COPY: tile i, j and destination slot k).  Any output pointer
 * may be NULL.  Fills *stats.  Uses the current options ("order_mode" / "order_tail" auto
 * mean program order; "mem_cap_tiles" with p = q = 1: the out-of-core plan of a
 * HOST_COLMAJOR call).  Returns 0, -1, -4 or -105.  Needs no GPU. */
int stf_dag_build(int64_t T, int p, int q, int64_t cap, int64_t *edges, int64_t cap_tasks, int32_t *kinds,
                  int64_t *ijk, stf_plan_stats *stats);

/* The plan stf_potrf(n, nb, 'L', desc of `kind`, ngpus) would execute with the
 * current options on a p x q grid of GPUs with `sms` SMs each (0: 148), built on
 * the host only (same code path as the call: submission order, host_stream /
 * out-of-core builders, stream assignment), exported like stf_dag_build.
 * Returns 0, -2, -4 or -105.  Needs no GPU. */
int stf_dag_build_call(int64_t n, int64_t nb, int kind, int ngpus, int p, int q, int sms, int64_t cap, int64_t *edges,
                       int64_t cap_tasks, int32_t *kinds, int64_t *ijk, stf_plan_stats *stats);

/* Buffers of the tasks of the last stf_dag_build(_call) on this thread: io[3*t] and
 * io[3*t+1] = buffer ids read (-1 unused), io[3*t+2] = buffer written (-1 for
 * STORE/FENCE).  Buffers: home tiles 0..T(T+1)/2-1 (tile (i,j) -> i(i+1)/2 + j)
 * then replicas; in an out-of-core plan the device frames 0..frames-1 (LOAD
 * writes a frame from the caller's tile (i, j), STORE reads one).  Returns the
 * number of buffers.  Needs no GPU. */
int stf_dag_tasks_io(int64_t cap_tasks, int64_t *io);

/* Further operand pairs of merged GEMM tasks ("gemm_merge") of the last
 * stf_dag_build(_call) on this thread: io2[6*t + 2(u-1)], io2[6*t + 2(u-1) + 1] =
 * the buffers of L_i,k+u and L_j,k+u (u = 1..3) of a task GEMM(i,j,k) that also
 * applies updates k+1, .. (-1 where unused).  Returns the number of merged tasks.
 * Needs no GPU. */
int64_t stf_dag_tasks_io2(int64_t cap_tasks, int64_t *io2);

/* Replica buffers written by the tasks of the last stf_dag_build(_call) on this
 * thread besides their output (fused push, "push" = 1): mir[8*t] = count (<= 7),
 * mir[8*t+1 ..] the buffer ids (-1 unused).  Returns the total number of pushed
 * replica writes.  Needs no GPU. */
int64_t stf_dag_tasks_mirrors(int64_t cap_tasks, int64_t *mir);

/* Generic STF rule on an arbitrary access list (the Algorithm 1 example):
 * ntasks tasks, task t has nacc[t] accesses listed consecutively in data[] and
 * modes[] (1 = read, 2 = write, 3 = read-write).  Writes up to cap edges.
 * Returns the number of edges (>= 0) or a negative error.  Needs no GPU. */
int64_t stf_infer_edges(int64_t ntasks, const int32_t *nacc, const int64_t *data, const int32_t *modes, int64_t cap,
                        int64_t *edges);

/* Harness entry points (input generation, direct tile kernels, kernel timing,
 * debug timelines) are declared in stf_harness.h; the same library exports them. */

/* ---------------------------------------------------------------- multi-process mode
 * One process per GPU (e.g. torch.distributed / torchrun): process `rank` owns
 * slot `rank` of a p x q grid (p*q == world) on CUDA device `device`.  Every
 * process builds the same plan (the STF DAG is deterministic) and runs only its
 * own slot's tasks.  A finished tile is pushed into the consumer process's
 * replica over NVLink (copy-engine copy into CUDA-IPC-mapped memory, or the
 * TRSM epilogue's peer stores with "push"), followed by a 32-bit flag write
 * into the consumer's flag array (cuStreamWriteValue32); the consumer's stream
 * waits on that flag (cuStreamWaitValue32) -- device-side hand-off, no host
 * round trip, no SMs.
 *   1. stf_mp_init(rank, world, device)
 *   2. stf_mp_prepare(n, nb, desc, blob): desc = TILED_2DBC whose tiles table
 *      holds this process's own tiles (others ignored); writes this process's
 *      stf_mp_blob_size() bytes of IPC handles into blob
 *   3. exchange the blobs (all-gather, rank order) and call stf_mp_import(blobs)
 *   4. per factorisation: barrier across processes, stf_mp_potrf() (returns the
 *      LAPACK info of this process's columns; the caller takes the minimum > 0
 *      over processes), barrier.
 * stf_finalize releases everything.  Errors as above. */
int stf_mp_init(int rank, int world, int device);
int64_t stf_mp_blob_size(void);
int stf_mp_prepare(int64_t n, int64_t nb, const stf_matrix_desc *A_desc, void *blob);
int stf_mp_import(const void *blobs);
int stf_mp_potrf(void);

#ifdef __cplusplus
}
#endif
#endif /* STF_CHOLESKY_H */
