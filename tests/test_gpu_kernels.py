"""Kernel-level parity of the sm_100a tile kernels (through the C ABI's direct
kernel entry points) against the oracle's tile-task definitions.

Tolerances are rigorous forward-error bounds of the operation, not fitted
numbers:  GEMM/SYRK: |dC| <= 2 (K+2) eps (|C| + |A| |B|^T) elementwise;
TRSM/POTRF: residual / backward-error bounds (see each test)."""
import ctypes

import numpy as np
import pytest

import oracle
from gpu_util import EPS, from_dev, to_dev

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def abi():
    from paper_conf_sc_augonnetasg24_b200 import _abi
    return _abi


@pytest.fixture(params=[(1, 3, 64), (1, 2, 64), (1, 2, 128), (1, 1, 64), (0, 0, 64)],
                ids=["dataflow+resident", "dataflow+rowpanel", "dataflow+rowpanel128", "dataflow", "recursive"])
def variant(request, abi):
    """(POTRF, TRSM, rows) implementations: POTRF dataflow (1) / recursive (0);
    TRSM resident panel (3, product default; row panel where unsupported) /
    row panel (2, 64 or 128 rows per CTA) / dataflow (1) / recursive (0)."""
    abi.stf_set_option(b"dataflow", request.param[0])
    abi.stf_set_option(b"trsm", request.param[1])
    abi.stf_set_option(b"trsm_rows", request.param[2])
    yield request.param
    abi.stf_set_option(b"dataflow", 1)
    abi.stf_set_option(b"trsm", 3)
    abi.stf_set_option(b"trsm_rows", 128)


def _even(x):
    return x + (x & 1)


def _gemm_case(abi, M, N, K, lower, lda=None, ldb=None, ldc=None, seed=0):
    # TMA needs 16-byte global strides: leading dimensions of A and B are even
    lda = lda or (_even(M) if M & 1 else None)
    ldb = ldb or (_even(N) if N & 1 else None)
    rng = np.random.default_rng(seed)
    A = rng.standard_normal((M, K))
    B = A if lower else rng.standard_normal((N, K))
    C = rng.standard_normal((M, N))
    dA, dC = to_dev(A, lda), to_dev(C, ldc)
    dB = dA if lower else to_dev(B, ldb)
    rc = abi.stf_kernel_gemm_nt(M, N, K, dA.data_ptr(), lda or M, dB.data_ptr(), (lda or M) if lower else (ldb or N),
                                dC.data_ptr(), ldc or M, int(lower))
    assert rc == 0, abi.stf_last_error()
    got = from_dev(dC, M)
    ref = oracle.tile_syrk(C, A) if lower else oracle.tile_gemm(C, A, B)
    bound = 2 * (K + 2) * EPS * (np.abs(C) + np.abs(A) @ np.abs(B).T)
    if lower:
        iu = np.triu_indices(M, 1)
        assert np.array_equal(got[iu], C[iu]), "strictly upper part of C was modified"
        il = np.tril_indices(M)
        assert np.all(np.abs(got[il] - ref[il]) <= bound[il])
    else:
        assert np.all(np.abs(got - ref) <= bound)
    # padding rows beyond M in the ld must be untouched
    if ldc and ldc > M:
        pad = dC.cpu().numpy()[:, M:]
        assert np.all(pad == 0)


@pytest.mark.parametrize("M,N,K", [(128, 128, 16), (256, 384, 100), (1024, 1024, 1024), (77, 130, 33),
                                   (1, 1, 1), (129, 257, 17), (64, 64, 1024)])
def test_gemm_nt(abi, M, N, K):
    _gemm_case(abi, M, N, K, False)


def test_gemm_nt_odd_leading_dim_is_rejected(abi):
    import torch

    t = torch.zeros((8, 8), dtype=torch.float64, device="cuda")
    rc = abi.stf_kernel_gemm_nt(7, 7, 7, t.data_ptr(), 7, t.data_ptr(), 8, t.data_ptr(), 8, 0)
    assert rc == -101 and b"misaligned" in abi.stf_last_error()


def test_gemm_nt_leading_dims(abi):
    _gemm_case(abi, 100, 60, 40, False, lda=104, ldb=64, ldc=110)


@pytest.mark.parametrize("N,K", [(128, 64), (256, 256), (1024, 1024), (200, 70), (64, 300)])
def test_syrk_lower(abi, N, K):
    _gemm_case(abi, N, N, K, True)


@pytest.mark.parametrize("M,n", [(64, 64), (100, 70), (1024, 1024), (300, 200), (1, 1), (512, 129), (2048, 2048),
                                 (130, 1000), (1000, 1024), (17, 64), (1, 128), (33, 192), (250, 512), (1024, 960)])
def test_trsm(abi, variant, M, n):
    rng = np.random.default_rng(M + n)
    Lfull = np.tril(rng.standard_normal((n, n))) * 0.1 + np.diag(1.0 + rng.random(n))
    B = rng.standard_normal((M, n))
    U = np.triu(rng.standard_normal((n, n)), 1)  # garbage above the diagonal must be ignored
    ldl, ldb = _even(n), _even(M)
    dL, dB = to_dev(Lfull + U, ldl), to_dev(B, ldb)
    assert abi.stf_kernel_trsm(M, n, dL.data_ptr(), ldl, dB.data_ptr(), ldb) == 0, abi.stf_last_error()
    X = from_dev(dB, M)
    ref = oracle.tile_trsm(B, Lfull + U)
    # componentwise residual bound of a substitution: |X L^T - B| <= c n eps |X| |L|^T
    res = np.abs(X @ Lfull.T - B)
    assert np.all(res <= 4 * (n + 2) * EPS * (np.abs(X) @ np.abs(Lfull).T + np.abs(B)))
    assert np.linalg.norm(X - ref) <= 1e-12 * np.linalg.norm(ref)


@pytest.mark.parametrize("n", [1, 2, 17, 64, 65, 100, 256, 1024, 2048])
def test_potrf_tile(abi, variant, n):
    import synth

    A = synth.spd_matrix(20 + n, n)
    lda = _even(n)
    dA = to_dev(A, lda)
    info = ctypes.c_int64(-7)
    assert abi.stf_kernel_potrf(n, dA.data_ptr(), lda, ctypes.byref(info)) == 0, abi.stf_last_error()
    assert info.value == 0
    got = from_dev(dA, n)
    iu = np.triu_indices(n, 1)
    assert np.array_equal(got[iu], A[iu]), "strictly upper part modified"
    L = np.tril(got)
    Lo, _ = oracle.potrf(A)
    assert np.linalg.norm(L - Lo) <= 1e-13 * np.linalg.norm(Lo)


@pytest.mark.parametrize("n,j", [(64, 0), (64, 63), (200, 64), (200, 199), (1024, 511)])
def test_potrf_tile_info(abi, variant, n, j):
    import synth

    A = synth.spd_matrix(3, n)
    A[j, j] = -1.0
    dA = to_dev(A)
    info = ctypes.c_int64(0)
    assert abi.stf_kernel_potrf(n, dA.data_ptr(), n, ctypes.byref(info)) == 0
    assert info.value == j + 1


def test_generator_bits_match_synth(abi):
    import torch
    import synth

    n = 1000
    for (r0, c0, rows, cols) in [(0, 0, 64, 64), (936, 0, 64, 100), (500, 500, 37, 21)]:
        t = torch.zeros((cols, rows), dtype=torch.float64, device="cuda")
        assert abi.stf_fill_spd_block(t.data_ptr(), rows, n, r0, c0, rows, cols, 7) == 0
        got = t.cpu().numpy().T
        ref = synth.spd_block(7, n, r0, c0, rows, cols)
        assert np.array_equal(got.view(np.uint64), np.ascontiguousarray(ref).view(np.uint64))


def test_potrf_tile_completes_with_serialised_launches():
    """The two-launch POTRF tile (option potrf_split) must complete when its launches
    run one after the other (CUDA_LAUNCH_BLOCKING=1, as under profilers and
    sanitizers): the first launch carries block-task CTAs of its own.  Run in a
    subprocess with a timeout, so a hang fails the test instead of the suite."""
    import os
    import subprocess
    import sys

    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = (
        "import ctypes, sys; sys.path.insert(0, %r); import numpy as np; import oracle, synth\n"
        "from gpu_util import to_dev, from_dev\n"
        "from paper_conf_sc_augonnetasg24_b200 import _abi\n"
        "n = 1024; A = synth.spd_matrix(31, n); dA = to_dev(A, n); info = ctypes.c_int64(-7)\n"
        "assert _abi.stf_kernel_potrf(n, dA.data_ptr(), n, ctypes.byref(info)) == 0\n"
        "L = np.tril(from_dev(dA, n)); Lo, _ = oracle.potrf(A)\n"
        "print(info.value, np.linalg.norm(L - Lo) / np.linalg.norm(Lo))\n" % root)
    env = dict(os.environ, CUDA_LAUNCH_BLOCKING="1", STF_POTRF_SPLIT="1",
               PYTHONPATH=os.pathsep.join([root, os.path.join(root, "tests")]))
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=env, timeout=300)
    assert r.returncode == 0, r.stderr[-800:]
    info, rel = r.stdout.split()
    assert int(info) == 0 and float(rel) <= 1e-13
