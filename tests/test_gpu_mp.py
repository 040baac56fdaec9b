"""Multi-process mode (one process per GPU, include/stf_cholesky.h stf_mp_*):
p*q processes each own one slot of the block-cyclic grid, hold only their own
tiles and run only their own tasks; finished tiles reach consumer processes as
CUDA-IPC replicas with device-side flag hand-off.  The box
has one GPU, so all ranks share cuda:0 -- the IPC/flag protocol is the same as
across NVLink peers.  Checked: bit equality with the single-process run of the
same plan (virtual slots), info, and two back-to-back runs of one plan."""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(n, nb, p, q, push=0, reps=2, port=29611, graph=1, p2=0):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=%d" % (p * q),
           "--master-addr", "127.0.0.1", "--master-port", str(port),
           os.path.join(ROOT, "tests", "mp_worker.py"), str(n), str(nb), str(p), str(q), str(push), str(reps), str(graph), str(p2)]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert out.returncode == 0, out.stdout[-3000:] + out.stderr[-3000:]
    line = [l for l in out.stdout.splitlines() if l.startswith("MP_RESULT")]
    assert line and "mismatched=0" in line[0], out.stdout[-2000:]
    return line[0]


@pytest.mark.gpu
@pytest.mark.parametrize("p,q,push,graph,port", [(1, 2, 0, 1, 29611), (2, 2, 0, 1, 29621), (2, 2, 1, 1, 29631),
                                                 (2, 1, 1, 1, 29641), (2, 2, 0, 0, 29661), (1, 2, 1, 0, 29671)])
def test_multiprocess_bit_equal_to_single_process(p, q, push, graph, port):
    line = _run(1536, 128, p, q, push=push, port=port, graph=graph, reps=3)
    print(line)
    if graph:  # the whole local DAG, flag waits/writes included, is one CUDA graph per process
        nodes = eval(line.split("graph_nodes=")[1].split(" ms=")[0])
        assert all(g > 0 for g in nodes), line


@pytest.mark.gpu
@pytest.mark.parametrize("p,q,push,port", [(2, 2, 0, 29681), (2, 2, 1, 29691), (1, 2, 1, 29701)])
def test_multiprocess_p2_exact(p, q, push, port):
    """Against the closed form: every rank's tiles equal L0 bit for bit (P2)."""
    line = _run(1536, 128, p, q, push=push, port=port, reps=2, p2=1)
    assert "p2=1" in line


@pytest.mark.gpu
def test_multiprocess_large_tile():
    print(_run(2048, 512, 2, 2, push=1, reps=2, port=29651))


@pytest.mark.gpu
@pytest.mark.parametrize("mode", ["mp", "single"])
def test_bench_two_ranks_virtual_slots(mode):
    """bench.py under torchrun with 2 ranks (both on cuda:0): the N > 1 line carries
    the plan statistics and the on-box P2 check (every tile bit-exact)."""
    import json

    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr", "127.0.0.1", "--master-port", "29721" if mode == "mp" else "29731",
           os.path.join(ROOT, "bench.py"), "--gpus", "2", "--virtual-slots", "1", "--mode", mode,
           "--order", "4096", "--tile", "512", "--steps", "2", "--warmup", "1", "--no-e2e", "--no-cpu"]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert out.returncode == 0, out.stdout[-3000:] + out.stderr[-3000:]
    lines = [json.loads(l) for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    d = lines[0]
    assert d["n_gpus"] == 2 and d["config"]["grid"] == "1x2" and d["value"] > 0
    assert d["check"]["bit_exact"] and d["check"]["tiles_checked"] == 36
    assert d["plan"]["slots"] == 2 and d["plan"]["transfers"] > 0
    assert d["step_wall_ms"] and len(d["step_ms"]) == 2
