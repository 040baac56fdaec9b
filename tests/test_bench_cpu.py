"""bench.py plumbing that runs without a GPU: the reference arm (the CPU oracle
timed on a bounded sample), its JSON line, and the multi-process path (torchrun
world size 2 over gloo on 127.0.0.1; only rank 0 prints)."""
import json
import os
import socket
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


REF_ARGS = ["--impl", "reference", "--steps", "2", "--warmup", "1", "--ref-seconds", "0.2", "--ref-cap", "1536"]


def _json_lines(out):
    return [json.loads(l) for l in out.splitlines() if l.strip().startswith("{")]


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, "bench.py"] + REF_ARGS, cwd=ROOT, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr
    lines = _json_lines(r.stdout)
    assert len(lines) == 1
    d = lines[0]
    assert d["impl"] == "reference" and d["unit"] == "GFLOP/s" and d["higher_is_better"] is True
    assert d["value"] > 0 and d["steps"] == 2 and d["warmup"] == 1
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
    assert d["config"]["n"] == 65536 and d["config"]["nb"] == 1024
    assert "configs[3]" in d["config"]["workload"]


def test_reference_arm_under_torchrun_two_ranks():
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), "bench.py", "--gpus", "2"] + REF_ARGS
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = _json_lines(r.stdout)
    assert len(lines) == 1 and lines[0]["n_gpus"] == 2


_WORKER = r"""
import os, sys
sys.path.insert(0, sys.argv[1])
import torch.distributed as dist
import bench
dist.init_process_group("gloo")
r = dist.get_rank()
m = bench.max_over_ranks(10.0 * (r + 1), True)
print("RANK%d MAX %.1f" % (r, m), flush=True)
dist.destroy_process_group()
"""


def test_max_over_ranks_gloo(tmp_path):
    w = tmp_path / "w.py"
    w.write_text(_WORKER)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), str(w), ROOT]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    assert "RANK0 MAX 20.0" in r.stdout and "RANK1 MAX 20.0" in r.stdout


def test_p2_fill_by_panels_matches_the_full_product():
    """bench.py's memory-light P2 input (used when the full L0 does not fit, n = 131072)
    equals the tiles of L0 L0^T formed at once, bit for bit (P2 is exact in any order)."""
    import importlib.util

    import numpy as np
    import torch

    import synth

    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    bench = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(bench)
    n, nb = 256, 64
    T = n // nb
    tiles = {(i, j): torch.empty((nb, nb), dtype=torch.float64) for i in range(T) for j in range(i + 1)}
    bench.p2_fill_by_panels(tiles, list(tiles), n, nb, "cpu")
    A, _ = synth.dyadic_spd(101, n)
    for (i, j), t in tiles.items():
        ref = A[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb]
        assert np.array_equal(t.numpy().T, ref), (i, j)
