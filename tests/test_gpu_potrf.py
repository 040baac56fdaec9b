"""Parity of the full STF Cholesky path (stf_potrf through the C ABI) against
the CPU oracle, plus the exact pins of SURVEY.md §8(c) through the GPU
pipeline, determinism across schedules / grids, COLMAJOR descriptors and info.

Gate (north_star): ||L_gpu - L_ref||_F / ||L_ref||_F <= 1e-10 and backward
error ||A - L L^T||_F / (||A||_F n eps) <= 10."""
import numpy as np
import pytest

import oracle
import synth
from gpu_util import backward_ratio, relF

pytestmark = pytest.mark.gpu

NSLOTS = 8  # slots 0..7 all on cuda:0 ("virtual GPUs")


@pytest.fixture(scope="module")
def stf():
    import paper_conf_sc_augonnetasg24_b200 as s
    s.init(NSLOTS, [0] * NSLOTS)
    yield s
    s.finalize()


@pytest.mark.parametrize("trsm,split", [(1, 1), (2, 1), (2, 2), (2, 4), (2, 8), (3, 4)])
def test_parity_trsm_variants(stf, trsm, split):
    _options(stf, trsm=trsm, trsm_split=split)
    M, info = _factor_spd(stf, 1536, 512, seed=2)
    _options(stf, trsm=3, trsm_split=4)
    assert info == 0
    Lo, _ = oracle.potrf(synth.spd_matrix(2, 1536))
    assert relF(M.to_dense().numpy(), Lo) <= 1e-10


@pytest.mark.parametrize("rows", [32, 128])
def test_trsm_panel_rows_same_bits(stf, rows):  # 128 is the default
    """The row-panel TRSM at 32 / 128 rows per CTA (128: half-depth stages, two
    solver warps per SM sub-partition) keeps every sum in the same order as the
    64-row form, so the whole factorisation is bit-identical."""
    for n, nb, split in [(2048, 512, 4), (3072, 1024, 4), (1536, 512, 2)]:
        ref = _bits(stf, n, nb, trsm=2, trsm_split=split, trsm_rows=64)
        got = _bits(stf, n, nb, trsm=2, trsm_split=split, trsm_rows=rows)
        assert np.array_equal(ref, got), (n, nb, split)
        Lo, _ = oracle.potrf(synth.spd_matrix(3, n))
        assert relF(got, Lo) <= 1e-10


def test_parity_recursive_panel_kernels(stf):
    """The recursive (GEMM-based) POTRF/TRSM variant through the whole path."""
    _options(stf, dataflow=0, trsm=0)
    M, info = _factor_spd(stf, 2048, 512, seed=1)
    _options(stf, dataflow=1, trsm=3)
    assert info == 0
    Lo, _ = oracle.potrf(synth.spd_matrix(1, 2048))
    assert relF(M.to_dense().numpy(), Lo) <= 1e-10


def _options(stf, **kw):
    for k, v in kw.items():
        stf.set_option(k, v)


@pytest.fixture(autouse=True)
def _reset_options(request):
    yield
    if "stf" in request.fixturenames:
        s = request.getfixturevalue("stf")
        _options(s, graph=1, serial=0, priority=1, streams=32, grid_p=0, dataflow=1, trsm=3, threads=8, lookahead=1, trsm_split=4, push=0,
                 trsm_rows=128, stream_pool=0, prio_mode=0, order_mode=-1, dev_order=0, order_asap=0, host_eager=0,
                 pdl=1, pdl_lead=-1, trsm_res_split=2)


def _factor_spd(stf, n, nb, p=1, q=1, seed=1):
    M = stf.TiledMatrix(n, nb, p, q, devices=[0] * (p * q))
    M.fill_spd(seed)
    info = M.potrf()
    return M, info


# ---------------------------------------------------------------- parity vs oracle
@pytest.mark.parametrize("n,nb", [(1024, 256), (576, 192), (480, 96), (200, 100), (2048, 512), (256, 256)])
def test_parity_metric_inputs(stf, n, nb):
    M, info = _factor_spd(stf, n, nb, seed=1)
    assert info == 0
    L = M.to_dense().numpy()
    A = synth.spd_matrix(1, n)
    Lo, oinfo = oracle.potrf(A)
    assert oinfo == 0
    assert relF(L, Lo) <= 1e-10
    assert backward_ratio(A, L) <= 10


@pytest.mark.parametrize("n,nb", [(2, 2), (4, 2), (6, 2), (64, 2), (50, 10), (90, 18), (130, 26), (300, 150)])
def test_parity_tiny_and_ragged_tiles(stf, n, nb):
    """Degenerate tile sizes: 2x2 tiles (T up to 32), tiles not a multiple of the
    16-row TMA box / 64-column dataflow block / 128-row CTA tile."""
    M, info = _factor_spd(stf, n, nb, seed=5)
    assert info == 0
    L = M.to_dense().numpy()
    A = synth.spd_matrix(5, n)
    Lo, _ = oracle.potrf(A)
    assert relF(L, Lo) <= 1e-10
    assert backward_ratio(A, L) <= 10


@pytest.mark.parametrize("n,nb,p,q", [(64, 2, 2, 4), (90, 18, 2, 2)])
def test_tiny_tiles_on_virtual_grids_bit_equal(stf, n, nb, p, q):
    ref = _bits(stf, n, nb, 1, 1, seed=6)
    assert np.array_equal(ref, _bits(stf, n, nb, p, q, seed=6))
    _options(stf, push=1)
    got = _bits(stf, n, nb, p, q, seed=6)
    _options(stf, push=0)
    assert np.array_equal(ref, got)
    for push in (0, 1):  # and against the closed form
        L, L0, _ = _p2(stf, n, nb, p, q, push=push)
        assert np.array_equal(L, L0)


@pytest.fixture(scope="module")
def oracle_8192():
    A = synth.spd_matrix(1, 8192)
    L, info = oracle.potrf(A)
    assert info == 0
    return A, L


@pytest.mark.parametrize("nb", [256, 512, 1024, 2048])  # 2048: CFG4's tile (BASELINE configs[4])
def test_parity_cfg1_nb_sweep(stf, oracle_8192, nb):
    A, Lo = oracle_8192
    M, info = _factor_spd(stf, 8192, nb, seed=1)
    assert info == 0
    L = M.to_dense().numpy()
    assert relF(L, Lo) <= 1e-10
    assert backward_ratio(A, L) <= 10


# ---------------------------------------------------------------- exact pins through the GPU path
def _factor_dense(stf, A, nb, p=1, q=1):
    import torch

    n = A.shape[0]
    M = stf.TiledMatrix(n, nb, p, q, devices=[0] * (p * q))
    M.load_dense(torch.from_numpy(np.ascontiguousarray(A)))
    info = M.potrf()
    return M.to_dense().numpy(), info


@pytest.mark.parametrize("n,nb", [(512, 128), (1024, 256), (384, 96)])
def test_p1_min_matrix_bit_exact(stf, n, nb):
    L, info = _factor_dense(stf, synth.min_matrix(n), nb)
    assert info == 0 and np.array_equal(L, np.tril(np.ones((n, n))))


@pytest.mark.parametrize("n,nb,p,q", [(1024, 256, 1, 1), (2048, 256, 2, 2), (1024, 128, 1, 2)])
def test_p2_dyadic_bit_exact(stf, n, nb, p, q):
    A, L0 = synth.dyadic_spd(101, n)
    L, info = _factor_dense(stf, A, nb, p, q)
    assert info == 0 and np.array_equal(L, L0)


def test_p3_diagonal_bit_exact(stf):
    A = synth.diag_matrix(5, 768)
    L, info = _factor_dense(stf, A, 256)
    assert info == 0 and np.array_equal(L, np.diag(np.sqrt(np.diag(A))))


@pytest.mark.parametrize("rho,tol", [(0.5, 1e-13), (0.9, 1e-12)])
def test_p6_kms(stf, rho, tol):
    n = 1024
    L, info = _factor_dense(stf, synth.kms_matrix(n, rho), 256)
    assert info == 0
    i = np.arange(n)
    Lref = np.where(i[:, None] >= i[None, :], rho ** (i[:, None] - i[None, :]).clip(0).astype(float), 0.0)
    Lref[1:, 1:] *= np.sqrt(1 - rho * rho)
    assert relF(L, Lref) <= tol


@pytest.mark.parametrize("j", [0, 255, 256, 1023])
def test_p10_info_at_tile_boundaries(stf, j):
    A = synth.spd_matrix(1, 1024)
    A[j, j] = -1.0
    _, info = _factor_dense(stf, A, 256)
    assert info == j + 1


def test_info_on_other_grid_slot(stf):
    A = synth.spd_matrix(1, 1024)
    A[700, 700] = -1.0  # tile (2,2) -> slot 0 on 2x2... and column 700 on slot (2%2)*2+2%2
    _, info = _factor_dense(stf, A, 256, 2, 2)
    assert info == 701


# ---------------------------------------------------------------- determinism / race checks (P9)
def _bits(stf, n, nb, p=1, q=1, seed=3, **opts):
    _options(stf, **opts)
    M, info = _factor_spd(stf, n, nb, p, q, seed)
    assert info == 0
    out = M.to_dense().numpy().copy()
    _options(stf, graph=1, serial=0, priority=1, streams=32, threads=8)
    return out


def _p2(stf, n, nb, p=1, q=1, **opts):
    """Factor the P2 dyadic matrix A = L0 L0^T (exact in any summation order) with
    the given options; every variant must return L0 bit for bit."""
    A, L0 = synth.dyadic_spd(101, n)
    _options(stf, **opts)
    try:
        L, info = _factor_dense(stf, A, nb, p, q)
        st = stf.last_stats()
    finally:
        _options(stf, graph=1, serial=0, priority=1, streams=32, threads=8, lookahead=1, push=0, stream_pool=0,
                 prio_mode=0, order_mode=-1, dev_order=0, order_asap=0)
    assert info == 0
    return L, L0, st


@pytest.mark.parametrize("variant", [
    {}, {"serial": 1}, {"graph": 0}, {"priority": 0, "streams": 3}, {"lookahead": 0},
    {"stream_pool": 1}, {"stream_pool": 2}, {"stream_pool": 1, "lookahead": 0}, {"prio_mode": 2},
    {"order_mode": 0}, {"order_mode": 2}, {"order_mode": 0, "order_asap": 1}, {"dev_order": 1}],
    ids=lambda v: ",".join("%s=%s" % kv for kv in v.items()) or "default")
def test_schedule_variants_p2_exact(stf, variant):
    """Every schedule / ablation variant (NEXT-1: stream pools, single stream, 1
    compute + 1 copy stream, per-step fences, priorities, submission orders,
    eager vs graph) against the closed form: L == L0 exactly."""
    L, L0, st = _p2(stf, 2048, 256, **variant)
    assert np.array_equal(L, L0)
    assert st["graph"] == (0 if variant.get("graph") == 0 else 1) and st["graph_fallback"] == 0


@pytest.mark.parametrize("p,q", [(1, 2), (2, 1), (2, 2), (2, 4), (1, 8)])
@pytest.mark.parametrize("variant", [{}, {"graph": 0, "threads": 1}, {"graph": 0}, {"push": 1}, {"push": 2},
                                     {"push": 1, "graph": 0}, {"lookahead": 0}],
                         ids=["graph", "eager1", "eager_threads", "push", "push_mc", "push_eager", "fence"])
def test_virtual_grids_p2_exact(stf, p, q, variant):
    """Distributed plans (2D block-cyclic and the 1D column block-cyclic 1x8 grid
    of cuSolverMg) with COPY tasks or fused pushes, eager or graph,
    with or without per-step fences: L == L0 exactly."""
    L, L0, st = _p2(stf, 2048, 256, p, q, **variant)
    assert np.array_equal(L, L0)
    assert st["slots"] == p * q and st["transfers"] > 0
    assert st["graph_fallback"] == 0 and st["graph"] == (0 if variant.get("graph") == 0 else 1)
    # push=2 (multicast) needs distinct devices: on virtual slots it keeps the peer stores of push=1
    assert st["data_plane"] == (1 if variant.get("push") else 0)
    assert (st["pushed"] > 0) == bool(variant.get("push"))


def test_same_shape_new_tiles_rebinds_graph(stf):
    """NEXT-2: a second matrix of the same shape re-uses the plan; the graph is
    re-captured and applied with cudaGraphExecUpdate; results stay exact."""
    A, L0 = synth.dyadic_spd(101, 1024)
    import torch

    M1 = stf.TiledMatrix(1024, 256)
    M1.fill_spd(3)
    assert M1.potrf() == 0
    assert stf.last_stats()["graph_reuse"] == 0
    M2 = stf.TiledMatrix(1024, 256)
    M2.load_dense(torch.from_numpy(np.ascontiguousarray(A)))
    assert M2.potrf() == 0
    st = stf.last_stats()
    assert st["graph_reuse"] == 2
    assert np.array_equal(M2.to_dense().numpy(), L0)
    M2.load_dense(torch.from_numpy(np.ascontiguousarray(A)))
    assert M2.potrf() == 0
    assert stf.last_stats()["graph_reuse"] == 1
    assert np.array_equal(M2.to_dense().numpy(), L0)


def test_repeated_calls_reuse_graph(stf):
    M = stf.TiledMatrix(1024, 256)
    M.fill_spd(2)
    assert M.potrf() == 0
    s1 = stf.last_stats()
    M.fill_spd(2)
    assert M.potrf() == 0
    s2 = stf.last_stats()
    assert s1["build_ms"] > 0 and s2["build_ms"] == 0
    assert s2["graph_nodes"] > 0 and s2["kernel_launches"] > 0
    assert s2["tasks"] == 20 and s2["edges"] == 30


# ---------------------------------------------------------------- COLMAJOR descriptors
@pytest.mark.parametrize("where", ["device", "host_pinned", "host_pageable"])
@pytest.mark.parametrize("order", ["F", "C"])
@pytest.mark.parametrize("ngpus", [1, 4])
def test_colmajor_descriptors(stf, where, order, ngpus):
    import torch

    n, nb = 768, 128
    A = synth.spd_matrix(4, n)
    A[np.triu_indices(n, 1)] = 12345.0  # the other triangle: must come back untouched
    if order == "F":
        base = np.asfortranarray(A)
    else:
        base = np.ascontiguousarray(A)
    if where == "device":
        t = torch.from_numpy(np.ascontiguousarray(base.T if order == "F" else base)).cuda()
        if order == "F":
            t = t.t()  # column-major view of A
    else:
        t = torch.from_numpy(np.ascontiguousarray(base.T if order == "F" else base))
        if where == "host_pinned":
            t = t.pin_memory()
        if order == "F":
            t = t.t()
    info = stf.potrf(t, nb, ngpus=ngpus)
    assert info == 0
    got = t.cpu().numpy()
    Lo, _ = oracle.potrf(synth.spd_matrix(4, n))
    assert relF(np.tril(got), Lo) <= 1e-10
    assert np.all(got[np.triu_indices(n, 1)] == 12345.0)


@pytest.mark.parametrize("ngpus", [1, 2])
def test_host_colmajor_submission_orders_same_bits(stf, ngpus):
    """HOST_COLMAJOR calls with nb >= 512 are re-submitted in list-scheduling
    order; that order, the earliest-start order and the eager lowering
    all keep the DAG, so the same bits as the device-resident tiles."""
    import torch

    n, nb = 4096, 1024
    ref = _bits(stf, n, nb, 1, ngpus, seed=7)
    A = synth.spd_matrix(7, n)
    for opts in ({}, {"order_mode": 0, "order_asap": 1}, {"host_eager": 1}):
        _options(stf, **opts)  # options are part of the memo key: each builds its own plan
        t = torch.from_numpy(np.ascontiguousarray(A)).pin_memory().t()  # column-major view
        assert stf.potrf(t, nb, ngpus=ngpus) == 0
        st = stf.last_stats()
        _options(stf, order_mode=-1, order_asap=0, host_eager=0)
        assert st["host_loads"] == 10 and (st["graph_nodes"] == 0) == ("host_eager" in opts)
        assert st["graph"] == (0 if "host_eager" in opts else 1)
        assert np.array_equal(np.tril(t.numpy()), np.tril(ref)), opts


def test_n_zero(stf):
    import torch

    t = torch.zeros((1, 1), dtype=torch.float64, device="cuda")
    assert stf.potrf_colmajor(t.data_ptr(), 0, 1, 2, "L", 0) == 0


# ---------------------------------------------------------------- full-size sampled parity
@pytest.mark.parametrize("n,nb,m", [(32768, 1024, 4096)])
def test_bench_config_leading_block_and_residual(stf, n, nb, m):
    """At the bench's full size: the leading m x m block of L is the Cholesky
    factor of A[:m,:m] (oracle computes it), and sampled rows of L L^T match A."""
    import torch

    M, info = _factor_spd(stf, n, nb, seed=1)
    assert info == 0
    T = n // nb
    mb = m // nb
    Llead = np.zeros((m, m))
    for (i, j), t in M.tiles.items():
        if i < mb and j < mb:
            Llead[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb] = t.T.cpu().numpy()
    Llead = np.tril(Llead)
    Lo, _ = oracle.potrf(synth.spd_block(1, n, 0, 0, m, m))
    assert relF(Llead, Lo) <= 1e-10
    # sampled rows: (L L^T)[r, :] = sum_k L[r, k] L[:, k]  vs  A[r, :]   (torch fp64 on GPU, harness only)
    rng = np.random.default_rng(0)
    rows = sorted(rng.choice(n, size=8, replace=False).tolist())
    Ld = torch.zeros((n, n), dtype=torch.float64, device="cuda")
    for (i, j), t in M.tiles.items():
        Ld[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb] = t.T
    Ld = torch.tril(Ld)
    for r in rows:
        got = (Ld[r:r + 1, :] @ Ld.T).cpu().numpy()[0]
        Arow = synth.spd_block(1, n, r, 0, 1, n)[0]
        err = np.linalg.norm(got - Arow) / (np.linalg.norm(Arow) * n * np.finfo(float).eps)
        assert err <= 10
    del Ld
    assert T == n // nb


def test_orders_after_callers_default_stream_work(stf):
    """Ordering contract (include/stf_cholesky.h): a call starts after the work
    the caller enqueued before it on the default stream -- here a long matmul
    followed by the device-to-device copies that fill the tiles, with no host
    synchronisation in between."""
    import torch

    n, nb = 1024, 256
    A, L0 = synth.dyadic_spd(101, n)
    Ad = torch.from_numpy(np.ascontiguousarray(A)).cuda()
    M = stf.TiledMatrix(n, nb)
    for t in M.tiles.values():
        t.zero_()
    big = torch.randn((6144, 6144), dtype=torch.float64, device="cuda")
    torch.cuda.synchronize()
    for _ in range(3):
        big = big @ big / 6144.0  # ~40 ms of default-stream work ahead of the tile copies
    for (i, j), t in M.tiles.items():
        t.copy_(Ad[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb].T)
    assert M.potrf() == 0
    assert np.array_equal(M.to_dense().numpy(), L0)


# ---------------------------------------------------------------- panel chain overlap (pdl)
@pytest.mark.parametrize("n,nb", [(2048, 256), (4096, 1024), (3072, 512)])
def test_chain_overlap_same_bits_and_oracle(stf, n, nb):
    """pdl = 1 (TRSM(k+1,k) launched while POTRF(k) runs, SYRK(k+1,k) while the TRSM
    runs, device flags between them) computes exactly what the same kernels compute
    without the overlap (pdl = 0 with the one-launch critical TRSM, trsm_res_split =
    1), whatever the trigger lead, on every grid (the overlap only exists where the
    chain shares a slot), and matches the oracle."""
    ref = _bits(stf, n, nb, seed=9, pdl=0, trsm_res_split=1)
    for lead in (0, 4, 8, 64):
        assert np.array_equal(ref, _bits(stf, n, nb, seed=9, pdl=1, pdl_lead=lead)), lead
    for p, q in ((1, 2), (2, 2), (2, 1)):
        assert np.array_equal(ref, _bits(stf, n, nb, p, q, seed=9, pdl=1)), (p, q)
    A = synth.spd_matrix(9, n)
    Lo, _ = oracle.potrf(A)
    assert relF(ref, Lo) <= 1e-10
    assert backward_ratio(A, ref) <= 10


@pytest.mark.parametrize("lead", [0, 3, 8, 16])
def test_chain_overlap_p2_exact(stf, lead):
    """The overlapped chain against the closed form at nb = 1024 (T = 4) and nb = 512."""
    for nb in (1024, 512):
        L, L0, st = _p2(stf, 4096, nb, pdl=1, pdl_lead=lead)
        assert np.array_equal(L, L0), nb
        assert st["graph"] == 1 and st["graph_fallback"] == 0


def test_chain_overlap_edges_reported(stf):
    """The plan statistics count the programmatic edges of the panel chain: two per
    panel step (TRSM(k+1,k), SYRK(k+1,k)) with the graph backend, none without pdl
    or with the eager backend."""
    n, nb = 4096, 1024
    T = n // nb
    for opts, want in (({"pdl": 1}, 2 * (T - 1)), ({"pdl": 0}, 0), ({"pdl": 1, "graph": 0}, 0)):
        _options(stf, **opts)
        M, info = _factor_spd(stf, n, nb, seed=2)
        assert info == 0
        assert stf.last_stats()["pdl_edges"] == want, opts
    _options(stf, pdl=1, graph=1)


def test_chain_step_bench_overlap_is_faster(stf):
    """stf_bench_kernel kind 4 (POTRF -> TRSM -> SYRK on 1024 tiles, one graph): the
    programmatic overlap shortens the chain step (measured 507 -> 374 us)."""
    import ctypes
    from paper_conf_sc_augonnetasg24_b200 import _abi
    t = {}
    for pdl in (0, 1):
        _options(stf, pdl=pdl, pdl_lead=8)
        ms = ctypes.c_double()
        assert _abi.stf_bench_kernel(4, 1024, 1024, 1024, 5, ctypes.byref(ms)) == 0, _abi.stf_last_error()
        t[pdl] = ms.value
    assert t[1] < 0.9 * t[0], t
