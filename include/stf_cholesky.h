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
 * re-entrant.  Ownership: the caller owns A (and every tile) in all modes and
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
 * Execution options (defaults from the environment at init):
 *   "dataflow" STF_DATAFLOW POTRF tile kernel: 1 single-launch dataflow (default), 0 recursive
 *   "trsm"     STF_TRSM     TRSM tile kernel: 3 (default) = resident panel for the critical
 *                           TRSM(k+1,k) when nb <= 1024 and nb % 64 == 0, row panel otherwise;
 *                           2 row panel, 1 dataflow, 0 recursive
 *   "trsm_split" STF_TRSM_SPLIT P in [1,16]: non-critical row-panel TRSMs run right-looking
 *                           over P column blocks (panel kernel + GEMM updates; default 4);
 *                           1: one panel launch
 *   "trsm_res_tail" STF_TRSM_RES_TAIL C >= 0: with trsm 3, every TRSM(i,k) of a panel step
 *                           whose trailing order n - k nb <= C uses the resident panel (there
 *                           the factorisation is latency-bound; default 8192)
 *   "trsm_rows" STF_TRSM_ROWS 32, 64 or 128 (default): rows per CTA of the non-critical
 *                           row-panel TRSM launches (128: two substitution chains per SM
 *                           sub-partition, full 64-column blocks only, else 64; same bits)
 *   "graph"    STF_GRAPH    1: capture the whole task DAG of a call into one CUDA
 *                           graph, memoised per (n, nb, grid, tiles) (default);
 *                           0: eager lowering on streams + events
 *   "streams"  STF_STREAMS  bulk compute streams per GPU slot (default 32; the pool is sized at init)
 *   "serial"   STF_SERIAL   1: every task on one stream in program order (race check)
 *   "priority" STF_PRIO     1: critical-path tasks on high-priority streams (default 1)
 *   "grid_p"   STF_GRID     rows P of the P x Q grid for COLMAJOR kinds (0 = auto)
 *   "push"     STF_PUSH     1: TRSM(i,k) writes L_ik into its consumers' replicas from its own
 *                           epilogue (fused push over NVLink, NEXT-3); 0: COPY tasks (default)
 *   "threads"  STF_THREADS  eager backend: host submission threads, slots split round-robin
 *                           (default 8, capped at ngpus; the graph backend captures on one thread)
 *   "lookahead" STF_LOOKAHEAD 1: pure STF DAG (default); 0: a fence task closes every
 *                           panel step (no look-ahead; ablation of PAPER.md:399)
 *   "mem_cap_tiles" STF_MEM_CAP_TILES  0 (default) or >= 3: a HOST_COLMAJOR call on one GPU
 *                           keeps at most this many nb x nb tiles on the device (out-of-core,
 *                           NEXT-4): tiles are loaded on demand and dirty
 *                           tiles written back on eviction (Belady order, left-looking
 *                           super-columns).  A cap >= T(T+1)/2 tiles means no cap.  Rejected
 *                           (-105) for HOST_COLMAJOR calls on more than one GPU; ignored for
 *                           device-resident kinds, whose matrix is on the device already.
 *   "ooc_order" STF_OOC_ORDER  program order of an out-of-core plan: 1 2D-blocked (column
 *                           blocks swept in row chunks: fewer panel re-reads when a trailing
 *                           column alone fills the frames); 0 tall super-columns; -1 (default)
 *                           1 when the plan is re-submitted in list-scheduling order (nb >=
 *                           512), else 1 while the cap is below half the tiles, else 0.  Every
 *                           order gives bit-identical L.
 *   "host_stream" STF_HOST_STREAM  1 (default): an uncapped HOST_COLMAJOR call on one GPU with
 *                           nb >= 512 and n/nb >= 16 is planned by the out-of-core builder with one frame per
 *                           tile (2D-blocked left-looking order, no eviction); 0: the
 *                           right-looking plan with its LOAD/STORE tasks.  Same bits.
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
} stf_plan_stats;

int stf_last_stats(stf_plan_stats *out);

/* Build (without running) the STF DAG of a T x T tile Cholesky on a p x q grid
 * and copy up to `cap` edges (src, dst pairs of task indices in submission
 * order) into edges[2*cap].  kinds[cap_tasks] receives per-task codes
 * (0 POTRF, 1 TRSM, 2 SYRK, 3 GEMM, 4 COPY, 5 LOAD, 6 STORE, 7 FENCE) and ijk[3*cap_tasks]
 * the (i, j, k) indices (for COPY: tile i, j and destination slot k).  Any output pointer
 * may be NULL.  Fills *stats.  Uses the current "push", "lookahead" and "mem_cap_tiles"
 * options (the latter, for p = q = 1: the out-of-core plan of a HOST_COLMAJOR call).
 * Needs no GPU. */
int stf_dag_build(int64_t T, int p, int q, int64_t cap, int64_t *edges, int64_t cap_tasks, int32_t *kinds,
                  int64_t *ijk, stf_plan_stats *stats);

/* Buffers of the tasks of the last stf_dag_build on this thread: io[3*t] and
 * io[3*t+1] = buffer ids read (-1 unused), io[3*t+2] = buffer written (-1 for
 * STORE/FENCE).  Buffers: home tiles 0..T(T+1)/2-1 (tile (i,j) -> i(i+1)/2 + j)
 * then replicas; in an out-of-core plan the device frames 0..frames-1 (LOAD
 * writes a frame from the caller's tile (i, j), STORE reads one).  Returns the
 * number of buffers.  Needs no GPU. */
int stf_dag_tasks_io(int64_t cap_tasks, int64_t *io);

/* Generic STF rule on an arbitrary access list (the Algorithm 1 example):
 * ntasks tasks, task t has nacc[t] accesses listed consecutively in data[] and
 * modes[] (1 = read, 2 = write, 3 = read-write).  Writes up to cap edges.
 * Returns the number of edges (>= 0) or a negative error.  Needs no GPU. */
int64_t stf_infer_edges(int64_t ntasks, const int32_t *nacc, const int64_t *data, const int32_t *modes, int64_t cap,
                        int64_t *edges);

/* ---------------------------------------------------------------- harness helpers
 * Fill the seeded SPD metric matrix (SURVEY.md §8(d) generator; same bits as
 * synth/spd.py) into a TILED_2DBC descriptor (lower tiles) on the devices.
 * Synchronous.  Not part of the factorisation. */
int stf_fill_spd_tiles(int64_t n, int64_t nb, const stf_matrix_desc *A_desc, int ngpus, uint64_t seed);

/* Same generator into an arbitrary column-major device block: rows r0.., cols c0..
 * of the order-n matrix into dst (ld), on the current CUDA device, stream 0. */
int stf_fill_spd_block(double *dst, int64_t ld, int64_t n, int64_t r0, int64_t c0, int64_t rows, int64_t cols,
                       uint64_t seed);

/* Direct tile-kernel entry points (device pointers, current device, default
 * stream, synchronous) used by the kernel-level parity tests and the roofline
 * measurement:  C -= A B^T (lower: SYRK);  B <- B L^-T;  A <- chol(A). */
int stf_kernel_gemm_nt(int64_t M, int64_t N, int64_t K, const double *A, int64_t lda, const double *B, int64_t ldb,
                       double *C, int64_t ldc, int lower);
int stf_kernel_trsm(int64_t M, int64_t n, const double *L, int64_t ldl, double *B, int64_t ldb);
int stf_kernel_potrf(int64_t n, double *A, int64_t lda, int64_t *info);

/* Kernel timing for the roofline: `reps` launches of one tile kernel on a
 * library-owned stream of the current device, each bracketed by CUDA events
 * recorded on that same stream; *avg_ms = mean launch duration.  Inputs are
 * generated on the device (SPD generator) and regenerated (untimed) before
 * each POTRF launch.  kind: 0 GEMM C[MxN] -= A[MxK] B[NxK]^T, 1 SYRK (N = M),
 * 2 TRSM B[MxN] <- B L^-T (K ignored), 3 POTRF of an M x M tile.
 * Returns 0 / -4 / -101 / -103.  Not part of the factorisation. */
int stf_bench_kernel(int kind, int64_t M, int64_t N, int64_t K, int reps, double *avg_ms);

/* Debug timeline of the dataflow POTRF tile kernel (one launch on the current
 * device, A: n x n column-major device matrix, ctas <= 0: default grid).
 * trace[0 .. 6T) holds %globaltimer stamps (ns) of the critical-path CTA per
 * 64-block step kb (P start, P published, S inputs ready, S published, U inputs
 * ready, U done), T = ceil(n/64); trace[6T + 3t ..] the claim / inputs-ready /
 * done stamps of bulk ticket t (0 if unused).  Returns the number of entries
 * written (<= cap) or a negative error.  Not part of the factorisation. */
/* Debug timeline of the last stf_potrf on one GPU slot, recorded when the
 * environment had STF_DEBUG_TRACE=1 at plan build (timing events recorded
 * before and after every task on its stream; no SM work).  Writes up to
 * cap_tasks records of 7 int64 (kind as in stf_dag_build, i, j, k, stream index,
 * ns since the first task's start, at start and at end; -1 if unavailable) in
 * program order; returns the number of tasks of the call (0 if not traced). */
int64_t stf_debug_last_trace(int64_t *out, int64_t cap_tasks);

int64_t stf_debug_potrf_trace(int64_t n, double *A, int64_t lda, int ctas, int64_t *trace, int64_t cap);

/* Debug timeline of the resident-panel TRSM kernel (B[M x n] <- B L^-T, device
 * pointers, current device; requires 64 <= n <= 1024, n % 64 == 0).  With
 * T = n/64, trace[5 kb + e] holds the %globaltimer stamps (ns) of CTA 0 for
 * column block kb: e = 0 MMA step start, 1 MMA waits for the previous block's
 * solution, 2 it is available, 3 updated block handed to the solver, 4 solver
 * starts; trace[5T + kb] the solver's end.  Returns the number of entries
 * written (<= cap) or a negative error.  Not part of the factorisation. */
int64_t stf_debug_trsm_trace(int64_t M, int64_t n, const double *L, int64_t ldl, double *B, int64_t ldb,
                             int64_t *trace, int64_t cap);

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
