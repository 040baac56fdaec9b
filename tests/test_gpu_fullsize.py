"""Parity at exactly the configurations bench.py reports (BASELINE configs[2] and
configs[3], n = 32768 / 65536, nb = 1024), in the launch configuration the bench
times (one stf_potrf call on device-resident TILED_2DBC tiles) and through the
e2e path (HOST_COLMAJOR, pinned, the host_stream plan at T = 32).

* P2 (north_star's closed form): A = L0 L0^T with the dyadic
  unit-lower L0 (m = 25) is exact in FP64 under any summation order, so A is
  built on the GPU with torch fp64 matmuls (harness only, independent of the
  library) and EVERY tile of the factor must equal L0 bit for bit.
* Metric inputs (seed 1): the full backward error ||A - L L^T||_F /
  (||A||_F n eps) <= 10 tile by tile with torch matmuls, plus a Freivalds probe
  ||A x - L (L^T x)||_2 / (||A||_F ||x||_2 n eps) <= 10.
"""
import gc

import numpy as np
import pytest

from synth.spd import dyadic_unit_lower_block_torch

pytestmark = pytest.mark.gpu
EPS = np.finfo(np.float64).eps


@pytest.fixture(scope="module")
def stf():
    import paper_conf_sc_augonnetasg24_b200 as s
    s.init(1, [0])
    yield s
    s.finalize()


def _dyadic(n, seed=101):
    """L0 (n x n, lower, on cuda:0) and a function giving tile (i, j) of A = L0 L0^T."""
    import torch

    rows = 4096
    L0 = torch.empty((n, n), dtype=torch.float64, device="cuda")
    for r in range(0, n, rows):
        L0[r:r + rows] = dyadic_unit_lower_block_torch(seed, n, r, 0, rows, n)

    def a_tile(i, j, nb):  # A_ij = sum_{k <= j} L0_ik L0_jk^T  (exact in any order)
        K = (j + 1) * nb
        return L0[i * nb:(i + 1) * nb, :K] @ L0[j * nb:(j + 1) * nb, :K].T

    return L0, a_tile


def _check_tiles_equal(get_tile, L0, n, nb):
    import torch

    T = n // nb
    bad = []
    for j in range(T):
        for i in range(j, T):
            got = get_tile(i, j)
            ref = L0[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb]
            if i == j:  # the diagonal tile's strictly upper part is not referenced
                got, ref = torch.tril(got), torch.tril(ref)
            if not torch.equal(got, ref):
                bad.append((i, j))
    return bad


@pytest.mark.parametrize("n,nb", [(32768, 1024), (65536, 1024)])
def test_p2_bit_exact_full_size_device_tiles(stf, n, nb):
    """configs[2] / configs[3] on one GPU, the bench's launch configuration."""
    import torch

    L0, a_tile = _dyadic(n)
    M = stf.TiledMatrix(n, nb, 1, 1, devices=[0])
    for (i, j), t in M.tiles.items():
        t.copy_(a_tile(i, j, nb).T)  # row-major storage of the transpose = column-major tile
    torch.cuda.synchronize()
    assert M.potrf() == 0
    st = stf.last_stats()
    T = n // nb
    assert st["graph"] == 1 and st["graph_fallback"] == 0
    assert st["tasks"] <= T + T * (T - 1) + T * (T - 1) * (T - 2) // 6  # merged GEMMs carry several updates
    bad = _check_tiles_equal(lambda i, j: M.tiles[(i, j)].T, L0, n, nb)
    assert not bad, bad[:10]
    del M, L0
    gc.collect()
    torch.cuda.empty_cache()


def test_p2_bit_exact_full_size_host_e2e(stf):
    """The e2e path bench.py reports: HOST_COLMAJOR on pinned memory, host_stream
    plan (one frame per tile, 2D-blocked left-looking order, list re-submission)."""
    import torch

    n, nb = 32768, 1024
    T = n // nb
    L0, a_tile = _dyadic(n)
    H = torch.empty((n, n), dtype=torch.float64, pin_memory=True)  # row-major H = column-major H^T
    sentinel = 1234.5
    for j in range(T):
        for i in range(j, T):
            H[j * nb:(j + 1) * nb, i * nb:(i + 1) * nb] = a_tile(i, j, nb).T.cpu()
    # strictly upper part of the column-major matrix (element (0, c) is H[c, 0]): must come back untouched
    H[1:nb, 0] = sentinel
    assert stf.potrf_colmajor(H.data_ptr(), n, n, nb, "L", None, 1) == 0
    st = stf.last_stats()
    assert st["frames"] == T * (T + 1) // 2 and st["host_loads"] == T * (T + 1) // 2  # host_stream plan
    assert torch.all(H[1:nb, 0] == sentinel)
    bad = _check_tiles_equal(lambda i, j: H[j * nb:(j + 1) * nb, i * nb:(i + 1) * nb].T.cuda(), L0, n, nb)
    assert not bad, bad[:10]
    del H, L0
    gc.collect()
    torch.cuda.empty_cache()


def test_metric_input_full_backward_error_and_freivalds(stf):
    """configs[2] on metric inputs (seed 1): full backward error over every tile
    and a Freivalds probe, both against north_star's bound of 10."""
    import torch
    from paper_conf_sc_augonnetasg24_b200 import _abi

    n, nb = 32768, 1024
    T = n // nb
    M = stf.TiledMatrix(n, nb, 1, 1, devices=[0])
    M.fill_spd(1)
    assert M.potrf() == 0
    L = torch.zeros((n, n), dtype=torch.float64, device="cuda")
    for (i, j), t in M.tiles.items():
        L[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb] = t.T
    L = torch.tril(L)
    del M
    A = torch.empty((n, n), dtype=torch.float64, device="cuda")  # column-major A^T = A (symmetric)
    assert _abi.stf_fill_spd_block(A.data_ptr(), n, n, 0, 0, n, n, 1) == 0
    normA = float(torch.linalg.norm(A))
    ss = 0.0
    for j in range(T):
        for i in range(j, T):
            K = (j + 1) * nb
            R = A[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb] - L[i * nb:(i + 1) * nb, :K] @ L[j * nb:(j + 1) * nb, :K].T
            ss += (1.0 if i == j else 2.0) * float((R * R).sum())
    backward = ss ** 0.5 / (normA * n * EPS)
    assert backward <= 10, backward
    g = torch.Generator(device="cuda").manual_seed(5)
    x = torch.randn(n, dtype=torch.float64, device="cuda", generator=g)
    fr = float(torch.linalg.norm(A @ x - L @ (L.T @ x))) / (normA * float(torch.linalg.norm(x)) * n * EPS)
    assert fr <= 10, fr
    print("n=%d backward=%.3e freivalds=%.3e" % (n, backward, fr))
    del A, L
    gc.collect()
    torch.cuda.empty_cache()
