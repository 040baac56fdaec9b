#!/usr/bin/env python
"""Benchmark: FP64 Cholesky GFLOP/s (n^3/3) of the STF tiled factorisation.

Contract (driver): `python bench.py --gpus N --steps K --warmup W` prints ONE
JSON line on rank 0.  Under torchrun (N > 1) the default is the library's
multi-process mode (--mode mp, include/stf_cholesky.h stf_mp_*): one process per
GPU, rank r owns slot r of the block-cyclic grid, holds only its own tiles and
runs only its own tasks (one CUDA graph per process); tiles reach consumer
processes through CUDA-IPC replicas with device-side flag hand-off.  Each rank
times its own graph with CUDA events; the step time is the max over ranks.
--mode single keeps the paper's single-process multi-GPU call (PAPER.md:447,
north_star's `stf_potrf(..., ngpus)`): rank 0 drives all N GPUs and the other
ranks contribute 0 device time to the max-over-ranks.

One step = one synchronous stf_potrf of the whole matrix (every §8(a) row: DAG,
placement, replica pushes, POTRF/TRSM/SYRK/GEMM kernels, completion) on
device-resident 2D-block-cyclic tiles (TILED_2DBC).  The
workload is north_star's target matrix, n = 65536, nb = 1024 (BASELINE
configs[3]; 17.4 GB of lower tiles, fits one B200), at every N.  The matrix is
regenerated on the device before every step (untimed); it is far larger than
the 126 MB L2.  After the timed steps one more call factors the P2 matrix
A = L0 L0^T on the same plan and every tile is compared with L0
bit for bit on the box (`check`).
`value` = n^3/3 * steps / sum(device time), device time measured with CUDA
events on the library's launch stream around the graph launch.

`--impl reference` times the CPU oracle (the slow plain Cholesky, as it stands)
on a bounded sample of the same workload: the leading n' x n' principal block of
the same matrix (its factor is the leading block of L), n' sized so the whole
run ends within a few minutes.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "FP64 Cholesky GFLOP/s (n³/3) at 1/2/4/8 B200; fraction of FP64 tensor peak"
UNIT = "GFLOP/s"
# FP64 DMMA peak measured on this pool's B200 (tools/calib_fp64.cu -> profiles/calib_fp64_r01.json):
# 64 FMA/clk/SM x 148 SMs x 1965 MHz, clocks held at max under FP64 load.
FP64_PEAK_TFLOPS = 37.09
FP64_PEAK_SRC = "measured DMMA peak, profiles/calib_fp64_r01.json (MEASURED_PEAKS.json has no FP64 entry)"

GRIDS = {1: (1, 1), 2: (1, 2), 4: (2, 2), 8: (2, 4)}


def grid_for(n):
    if n in GRIDS:
        return GRIDS[n]
    p = max(d for d in range(1, int(math.isqrt(n)) + 1) if n % d == 0)
    return p, n // p


# ------------------------------------------------------------------ clocks
class ClockSampler:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "--query-gpu=" + self.FIELDS, "--format=csv,noheader,nounits",
                                       "-lms", "200"], stdout=self.f, stderr=subprocess.DEVNULL)
        except OSError:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        self.p.wait()
        self.f.flush()
        rows = []
        for ln in open(self.f.name):
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 9:
                continue
            try:
                rows.append((int(parts[0]), float(parts[1]), float(parts[2]), float(parts[3]), parts[5:9]))
            except ValueError:
                continue
        os.unlink(self.f.name)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        pmax = max(r[3] for r in rows)
        load = [r for r in rows if r[3] >= 0.5 * pmax] or rows
        sm = sorted(r[1] for r in load)
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in load for k in range(4) if r[4][k].lower().startswith("active")})
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": max(r[2] for r in rows), "reasons": reasons,
                "samples_under_load": len(load), "power_w_max": pmax}


# ------------------------------------------------------------------ oracle (cpu_baseline / reference arm)
def oracle_sample(n, seed, target_s, cap_n=None):
    """Time the oracle on the leading n' x n' block of the order-n metric matrix,
    n' chosen from a small calibration run so one sample takes ~target_s."""
    import oracle
    import synth

    cal = 1536
    A = synth.spd_block(seed, n, 0, 0, cal, cal)
    oracle.potrf(A)  # builds/loads liboracle.so
    t0 = time.perf_counter()
    oracle.potrf(A)
    tc = time.perf_counter() - t0
    m = int(cal * (target_s / max(tc, 1e-3)) ** (1.0 / 3.0))
    m = min(max(cal, m), cap_n or n, 16384)
    m -= m % 64
    A = synth.spd_block(seed, n, 0, 0, m, m)
    t0 = time.perf_counter()
    _, info = oracle.potrf(A)
    dt = time.perf_counter() - t0
    assert info == 0
    return m, dt, oracle.max_threads()


def max_over_ranks(x: float, dist_on: bool) -> float:
    """Max of a per-rank float over all ranks (NCCL on GPU boxes, gloo on CPU)."""
    if not dist_on:
        return x
    import torch
    import torch.distributed as dist

    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([x], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def workload_name(n, nb):
    cfg = {(65536, 1024): "configs[3]", (32768, 1024): "configs[2]", (131072, 2048): "configs[4]",
           (8192, 512): "configs[1]", (1024, 256): "configs[0]"}.get((n, nb), "custom")
    return "n=%d nb=%d FP64 SPD (seeded, diagonally dominant), %s" % (n, nb, cfg)


def p2_check(tiles, n, nb, owned=None):
    """Load the P2 dyadic matrix A = L0 L0^T (harness-side torch
    fp64 matmuls build it exactly in any order) into the tiles this process holds.
    `tiles` maps (i, j) -> the row-major (nb, nb) tensor holding tile (i, j)
    transposed.  Returns L0 per device for p2_compare after the factorisation."""
    import torch
    from synth.spd import dyadic_unit_lower_block_torch

    by_dev = {}
    for ij, t in tiles.items():
        by_dev.setdefault(t.device, []).append(ij)
    L0s = {}
    for dev in by_dev:
        free, _ = torch.cuda.mem_get_info(dev)
        if n * n * 8 > free // 2:
            # the full L0 does not fit next to the tiles (n = 131072: 128 GiB): accumulate
            # A_ij = sum_k L0_ik L0_jk^T panel by panel and let p2_compare regenerate the
            # reference blocks
            p2_fill_by_panels(tiles, by_dev[dev], n, nb, dev)
            L0s[dev] = None
            torch.cuda.synchronize(dev)
            continue
        L0 = torch.empty((n, n), dtype=torch.float64, device=dev)
        for r in range(0, n, 4096):
            L0[r:r + 4096] = dyadic_unit_lower_block_torch(101, n, r, 0, min(4096, n - r), n, device=dev)
        L0s[dev] = L0
        for (i, j) in by_dev[dev]:
            K = (j + 1) * nb
            tiles[(i, j)].copy_((L0[i * nb:(i + 1) * nb, :K] @ L0[j * nb:(j + 1) * nb, :K].T).T)
        torch.cuda.synchronize(dev)
    return L0s


def p2_fill_by_panels(tiles, mine, n, nb, dev):
    """Tiles (i, j) in `mine` <- (L0 L0^T)_ij accumulated over the column panels k of L0
    (P2: exact in FP64 in any summation order); only one n x nb panel of L0 is held."""
    from synth.spd import dyadic_unit_lower_block_torch

    mine = set(mine)
    for ij in mine:
        tiles[ij].zero_()
    for k in range(n // nb):
        P = dyadic_unit_lower_block_torch(101, n, k * nb, k * nb, n - k * nb, nb, device=dev)
        for (i, j) in mine:
            if j >= k:
                tiles[(i, j)] += (P[(i - k) * nb:(i - k + 1) * nb] @ P[(j - k) * nb:(j - k + 1) * nb].T).T
        del P


def p2_compare(tiles, L0s, nb, n):
    import torch

    from synth.spd import dyadic_unit_lower_block_torch

    bad = 0
    for (i, j), t in tiles.items():
        got = t.T
        L0 = L0s[t.device]
        ref = (L0[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb] if L0 is not None else
               dyadic_unit_lower_block_torch(101, n, i * nb, j * nb, nb, nb, device=t.device))
        if i == j:
            got, ref = torch.tril(got), torch.tril(ref)
        bad += not torch.equal(got, ref)
    return len(tiles), bad


def reference_arm(args, rank, world):
    if rank != 0:
        return 0
    n, nb = args.n, args.nb
    per_step = args.ref_seconds or max(2.0, min(20.0, 150.0 / max(1, args.steps + args.warmup)))
    m, _, cores = oracle_sample(n, 1, per_step, cap_n=args.ref_cap)
    import oracle
    import synth

    A = synth.spd_block(1, n, 0, 0, m, m)
    for _ in range(args.warmup):
        oracle.potrf(A)
    ts = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        _, info = oracle.potrf(A)
        ts.append(time.perf_counter() - t0)
        assert info == 0
    tot = sum(ts)
    value = m ** 3 / 3 * len(ts) / tot / 1e9
    sample = ("leading %dx%d principal block of the seed-1 n=%d metric matrix per step "
              "(its factor is the leading block of L); plain unblocked Cholesky-Crout, OpenMP" % (m, m, n))
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(1000 * tot / len(ts), 3),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": workload_name(n, nb),
                   "n": n, "nb": nb, "grid": "%dx%d" % grid_for(args.gpus), "sample_n": m, "l2": "n/a (CPU)"},
        "cpu_baseline": {"value": round(value, 4), "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
        "e2e": {"value": round(value, 4), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ our arm
def run_ours(args, rank, world):
    import torch
    import torch.distributed as dist

    dist_on = world > 1
    if dist_on:
        # NCCL needs one GPU per rank; virtual slots (all ranks on cuda:0) use gloo
        nccl = torch.cuda.is_available() and not args.virtual
        dist.init_process_group("nccl" if nccl else "gloo")
        if torch.cuda.is_available():
            torch.cuda.set_device(0 if args.virtual else int(os.environ.get("LOCAL_RANK", "0")))
    N = args.gpus
    n, nb = args.n, args.nb
    P, Q = grid_for(N) if not args.grid else tuple(int(x) for x in args.grid.lower().split("x"))
    assert P * Q == N, "--grid must have P*Q == --gpus"
    mode = args.mode or ("mp" if dist_on else "single")
    if mode == "mp":
        assert dist_on and world == N, "--mode mp needs torchrun with one rank per GPU"
        return run_mp(args, rank, world, P, Q)
    result = None
    total_ms = 0.0
    if rank == 0:
        import paper_conf_sc_augonnetasg24_b200 as stf

        devices = list(range(N)) if args.virtual == 0 else [0] * N
        stf.init(N, devices)
        M = stf.TiledMatrix(n, nb, P, Q, devices=devices)
        first_ms = None
        for w in range(args.warmup):
            M.fill_spd(1)
            t0 = time.perf_counter()
            assert M.potrf() == 0 or os.environ.get("STF_DEBUG_SKIP")
            if w == 0:
                first_ms = 1000 * (time.perf_counter() - t0)
        for d in set(devices):
            torch.cuda.synchronize(d)
    if dist_on:
        dist.barrier()
    clocks = ClockSampler()
    steps_ms = []
    walls = []
    stats = None
    if rank == 0:
        clocks.start()
        for _ in range(args.steps):
            M.fill_spd(1)  # untimed regeneration (input is overwritten by L)
            for d in set(devices):
                torch.cuda.synchronize(d)
            t0 = time.perf_counter()
            torch.cuda.nvtx.range_push("bench_step")  # lets ncu capture only timed steps (tools/launchlist.sh)
            info = M.potrf()  # synchronous
            torch.cuda.nvtx.range_pop()
            walls.append(1e3 * (time.perf_counter() - t0))
            assert info == 0 or os.environ.get("STF_DEBUG_SKIP"), info
            stats = stf.last_stats()
            steps_ms.append(stats["device_ms"])
        for d in set(devices):
            torch.cuda.synchronize(d)
        clk = clocks.stop()
        total_ms = sum(steps_ms)
        check = None
        if not args.no_check:
            L0s = p2_check(M.tiles, n, nb)
            info = M.potrf()
            ntile, bad = p2_compare(M.tiles, L0s, nb, n)
            del L0s
            check = {"input": "P2 dyadic A = L0 L0^T (m=25, seed 101), same plan, after the timed steps",
                     "info": info, "tiles_checked": ntile, "tiles_mismatched": bad, "bit_exact": bad == 0 and info == 0}
            torch.cuda.empty_cache()
    if dist_on:
        total_ms = max_over_ranks(total_ms, True)
        dist.barrier()
    if rank != 0:
        if dist_on:
            dist.destroy_process_group()
        return 0

    del M
    torch.cuda.empty_cache()
    report(args, stf, N, P, Q, total_ms, steps_ms, stats, clk, first_ms, "single", args.steps * stats["kernel_launches"],
           check, walls)
    stf.finalize()
    if dist_on:
        dist.destroy_process_group()
    return 0


def run_mp(args, rank, world, P, Q):
    """--mode mp: one process per GPU (stf_mp_*), max over ranks of each rank's device time."""
    import torch
    import torch.distributed as dist
    import paper_conf_sc_augonnetasg24_b200 as stf

    N, n, nb = world, args.n, args.nb
    dev = 0 if args.virtual else int(os.environ.get("LOCAL_RANK", rank))
    torch.cuda.set_device(dev)
    stf.mp_init(rank, world, dev)
    A = stf.MpTiledMatrix(n, nb, P, Q, rank, dev)
    blob = A.prepare()
    blobs = [None] * world
    dist.all_gather_object(blobs, blob)
    A.import_blobs(blobs)

    walls = []

    def step():
        A.fill_spd(1)  # untimed regeneration of this rank's tiles
        torch.cuda.synchronize(dev)
        dist.barrier()
        t0 = time.perf_counter()
        info = A.potrf()  # synchronous
        assert info == 0 or os.environ.get("STF_DEBUG_SKIP"), info
        ms = stf.last_stats()["device_ms"]
        dist.barrier()
        walls.append(1e3 * (time.perf_counter() - t0))  # barrier to barrier (cross-check of the device time)
        return ms

    t0 = time.perf_counter()
    step()
    first_ms = 1000 * (time.perf_counter() - t0)
    for _ in range(args.warmup - 1):
        step()
    clocks = ClockSampler()
    if rank == 0:
        clocks.start()
    walls.clear()
    mine = [step() for _ in range(args.steps)]
    wall_ms = [max_over_ranks(x, True) for x in walls]
    clk = clocks.stop() if rank == 0 else None
    stats = stf.last_stats()
    check = None
    if not args.no_check:
        L0s = p2_check(A.tiles, n, nb)
        dist.barrier()
        info = A.potrf()
        dist.barrier()
        ntile, bad = p2_compare(A.tiles, L0s, nb, n)
        del L0s
        torch.cuda.empty_cache()
        got = [None] * world
        dist.all_gather_object(got, (info, ntile, bad))
        bad_all = sum(g[2] for g in got)
        check = {"input": "P2 dyadic A = L0 L0^T (m=25, seed 101), same plan, after the timed steps",
                 "info": max(g[0] for g in got), "tiles_checked": sum(g[1] for g in got), "tiles_mismatched": bad_all,
                 "bit_exact": bad_all == 0 and all(g[0] == 0 for g in got)}
    steps_ms = [max_over_ranks(x, True) for x in mine]  # per step: the slowest rank
    total_ms = sum(steps_ms)
    launches = torch.tensor([float(stats["kernel_launches"])], dtype=torch.float64,
                            device="cuda" if dist.get_backend() == "nccl" else "cpu")
    dist.all_reduce(launches)
    nodes = [None] * world
    dist.all_gather_object(nodes, stats["graph_nodes"])
    stf.finalize()
    dist.barrier()
    if rank == 0:
        # e2e and kernels-alone numbers through the single-process API on all N GPUs
        devices = list(range(N)) if args.virtual == 0 else [0] * N
        stf.init(N, devices)
        stats = dict(stats, graph_nodes=sum(nodes), kernel_launches=int(launches.item()))
        del A
        torch.cuda.empty_cache()
        report(args, stf, N, P, Q, total_ms, steps_ms, stats, clk, first_ms, "mp", args.steps * int(launches.item()),
               check, wall_ms)
        stf.finalize()
    dist.barrier()
    dist.destroy_process_group()
    return 0


def report(args, stf, N, P, Q, total_ms, steps_ms, stats, clk, first_ms, mode, gpu_launches, check=None, wall_ms=None):
    import torch

    n, nb = args.n, args.nb
    flops = n ** 3 / 3.0
    value = flops * args.steps / (total_ms * 1e-3) / 1e9
    ms_per_step = total_ms / args.steps

    # ---- e2e: same metric through the C ABI with HOST buffers (pinned), copies inside the timed region
    e2e = None
    if not args.no_e2e:
        e2e = e2e_run(stf, n, nb, N, args)

    # ---- roofline: the factorisation is one graph launch on the library's launch stream
    achieved_tf = value / 1e3
    ndev = 1 if args.virtual else N  # virtual slots share one GPU's tensor cores
    roof = {"bound": "tensor", "achieved": round(achieved_tf, 3), "peak": FP64_PEAK_TFLOPS * ndev, "unit": "TFLOP/s",
            "frac": round(achieved_tf / (FP64_PEAK_TFLOPS * ndev), 4), "traffic": None,
            "kernel": "whole-DAG CUDA graph launch (n^3/3 flop per launch, %d kernels inside)" % stats["kernel_launches"],
            "peak_src": FP64_PEAK_SRC}
    # dominant kernel (GEMM tile update) timed alone on its own stream at this nb and at full occupancy
    from paper_conf_sc_augonnetasg24_b200 import _abi
    import ctypes

    kern = {}
    for name, kind, M_, N_, K_ in (("gemm_tile", 0, nb, nb, nb), ("gemm_full", 0, 8 * nb, 8 * nb, nb),
                                   ("syrk_tile", 1, nb, nb, nb), ("trsm_tile", 2, nb, nb, 0),
                                   ("potrf_tile", 3, nb, nb, nb)):
        ms = ctypes.c_double()
        torch.cuda.set_device(0)
        rc = _abi.stf_bench_kernel(kind, M_, N_, K_, 10, ctypes.byref(ms))
        if rc == 0:
            fl = {0: 2.0 * M_ * N_ * K_, 1: 1.0 * M_ * M_ * K_, 2: 1.0 * M_ * N_ * N_, 3: M_ ** 3 / 3.0}[kind]
            kern[name] = {"ms": round(ms.value, 4), "tflops": round(fl / (ms.value * 1e-3) / 1e12, 3),
                          "frac": round(fl / (ms.value * 1e-3) / 1e12 / FP64_PEAK_TFLOPS, 4),
                          "shape": [M_, N_, K_ if kind in (0, 1) else None]}
    roof["kernels_alone"] = kern
    # dominant kernel: the GEMM tile update (GEMM+SYRK are (T-1)(T-2)/T^2 + (T-1)/T^2 of the flops)
    T = n // nb
    tr = load_traffic(nb)
    dom = {"name": "gemm_nt_dmma (GEMM/SYRK tile update C -= A B^T)",
           "flop_share": round(((T - 1) * (T - 2) + (T - 1)) / T ** 2, 4),
           "launches_per_step": T * (T - 1) * (T - 2) // 6 + T * (T - 1) // 2,
           "alone_tile": kern.get("gemm_tile"), "alone_full_occupancy": kern.get("gemm_full"),
           "traffic_bytes_per_tile_launch": tr, "algorithmic_bytes_per_tile_launch": 4 * nb * nb * 8}
    roof["dominant_kernel"] = dom
    gt = load_graph_traffic(n, nb) if ndev == 1 else None
    if gt:
        roof["traffic"] = gt["traffic_bytes"]
        roof["traffic_src"] = gt["src"]
    roof["traffic_note"] = ("traffic = DRAM bytes of one whole-DAG graph launch (ncu --graph-profiling graph, "
                            "committed under profiles/, null when none was captured at this n, nb); algorithmic "
                            "minimum %.2f GB (lower tiles read and written once); per-kernel DRAM traffic of the GEMM "
                            "tile in dominant_kernel (nb=1024 capture only)" % (2 * 8 * nb * nb * T * (T + 1) / 2 / 1e9))

    cpu = None
    if N == 1 and not args.no_cpu:
        m, dt, cores = oracle_sample(n, 1, args.cpu_seconds)
        cpu = {"value": round(m ** 3 / 3 / dt / 1e9, 4), "unit": UNIT, "cores": cores, "kind": "oracle",
               "sample": "leading %dx%d principal block of the same seed-1 n=%d matrix (its factor is the "
                         "leading block of L), %.1f s" % (m, m, n, dt)}

    line = {
        "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": N, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms_per_step, 3), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": workload_name(n, nb),
                   "n": n, "nb": nb, "grid": "%dx%d" % (P, Q), "descriptor": "TILED_2DBC (device-resident tiles)",
                   "l2": "inputs larger than L2 (%.1f GB of tiles) and regenerated before every step" %
                         (n // nb * (n // nb + 1) / 2 * nb * nb * 8 / 1e9),
                   "graph": bool(stats["graph"]), "graph_fallback": bool(stats["graph_fallback"]),
                   "streams": stf.get_option("streams"),
                   "panel_chain": ("programmatic launch, lead %d blocks (pdl)" % (stf.get_option("pdl_lead") if
                                                                                 stf.get_option("pdl_lead") >= 0 else
                                                                                 max(2, nb // 128))
                                   if stf.get_option("pdl") else "full-completion edges"),
                   "virtual_slots": bool(args.virtual),
                   "processes": ("one per GPU (stf_mp_*, CUDA-IPC replicas, device-side flags)" if mode == "mp"
                                 else "one process drives all %d GPU(s) (stf_potrf)" % N)},
        "gpu_launches": int(gpu_launches),
        "clocks": clk,
        "roofline": roof,
        "cpu_baseline": cpu,
        "e2e": e2e,
        "plan": {k: stats[k] for k in ("tasks", "dag_tasks", "edges", "critical_path", "graph_nodes", "kernel_launches",
                                       "transfers", "transfer_bytes", "pushed", "replicas_max", "data_plane",
                                       "devices", "slots", "peer_transfers", "merged_gemms", "pdl_edges", "build_ms")},
        "check": check,
        "first_call_ms": round(first_ms, 1) if first_ms else None,
        "step_ms": [round(x, 3) for x in steps_ms],
        "step_wall_ms": [round(x, 3) for x in wall_ms] if wall_ms else None,
    }
    print(json.dumps(line), flush=True)


def e2e_run(stf, n, nb, N, args):
    """stf_potrf on a pinned HOST column-major matrix: lower tiles H2D, factor,
    lower tiles D2H, all tasks of one timed call.  Regeneration is untimed."""
    import torch

    T = n // nb
    A_host = torch.empty((n, n), dtype=torch.float64, pin_memory=True)  # row-major storage = col-major A^T = A
    dev = torch.empty((n, n), dtype=torch.float64, device="cuda:0")
    from paper_conf_sc_augonnetasg24_b200 import _abi

    def regen():
        rc = _abi.stf_fill_spd_block(dev.data_ptr(), n, n, 0, 0, n, n, 1)
        assert rc == 0
        A_host.copy_(dev)
        torch.cuda.synchronize()

    times = []
    for it in range(args.e2e_steps + 1):
        regen()
        t0 = time.perf_counter()
        info = stf.potrf_colmajor(A_host.data_ptr(), n, n, nb, "L", None, N)
        wall = time.perf_counter() - t0
        assert info == 0
        if it > 0:
            times.append((stf.last_stats()["device_ms"], wall * 1e3))
    del dev
    tile_bytes = T * (T + 1) // 2 * nb * nb * 8
    dev_ms = sum(t[0] for t in times) / len(times)
    wall_ms = sum(t[1] for t in times) / len(times)
    return {"value": round(n ** 3 / 3 / (dev_ms * 1e-3) / 1e9, 3), "unit": UNIT,
            "h2d_bytes_per_step": tile_bytes, "d2h_bytes_per_step": tile_bytes,
            "ms_per_step": round(dev_ms, 3), "host_wall_ms_per_step": round(wall_ms, 3),
            "api": "stf_potrf(STF_DESC_HOST_COLMAJOR, pinned), lower tiles copied in and written back as tasks",
            "steps": len(times)}


def load_graph_traffic(n, nb):
    """DRAM bytes of one whole-DAG graph launch at (n, nb), from the newest committed ncu summary."""
    import glob

    best = None
    for p in sorted(glob.glob(os.path.join(ROOT, "profiles", "r*", "graph_traffic_n%d_nb%d*.json" % (n, nb)))):
        try:
            d = json.load(open(p))
            best = {"traffic_bytes": d["traffic_bytes"], "src": os.path.relpath(p, ROOT)}
        except (OSError, ValueError, KeyError):
            pass
    return best


def load_traffic(nb):
    """dram bytes per GEMM launch from the committed ncu --set full summary, if
    present and captured at this tile size (nb=1024)."""
    p = os.path.join(ROOT, "profiles", "gemm_traffic.json")
    try:
        d = json.load(open(p))
        return d.get("traffic_bytes_per_launch") if "nb=%d)" % nb in d.get("kernel", "") else None
    except (OSError, ValueError):
        return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--n", "--order", dest="n", type=int, default=65536)
    ap.add_argument("--nb", "--tile", dest="nb", type=int, default=1024)
    ap.add_argument("--virtual-slots", dest="virtual", type=int, default=0, help="map all slots onto cuda:0")
    ap.add_argument("--grid", default="", help="PxQ process grid (default: P <= Q, P maximal)")
    ap.add_argument("--mode", default=None, choices=["single", "mp"],
                    help="N>1: mp = one process per GPU (default under torchrun), single = rank 0 drives all GPUs")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-check", action="store_true", help="skip the post-timing P2 bit-exactness check")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--ref-cap", type=int, default=0, help="cap on the reference sample order (0 = none)")
    ap.add_argument("--ref-seconds", type=float, default=0.0, help="oracle seconds per reference step (0 = auto)")
    args = ap.parse_args()
    assert args.warmup >= 1
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if args.impl == "reference":
        return reference_arm(args, rank, world)
    return run_ours(args, rank, world)


if __name__ == "__main__":
    sys.exit(main())
