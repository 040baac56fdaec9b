"""Out-of-core factorisation (NEXT-4): a HOST_COLMAJOR call
with "mem_cap_tiles" = F keeps at most F nb x nb tiles on the device, loading
tiles on demand and writing dirty ones back on eviction.  Same kernels, same
per-tile update order as the in-core call, so the factor must be bit-identical
to it; and within the parity tolerance of the oracle."""
import numpy as np
import pytest

import oracle
import synth
from gpu_util import relF

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def stf():
    import paper_conf_sc_augonnetasg24_b200 as s
    s.init(2, [0, 0])
    yield s
    s.set_option("mem_cap_tiles", 0)
    s.finalize()


def _host(A, order, pinned=True):
    """torch CPU tensor holding A column-major (order F) or row-major (C)."""
    import torch

    t = torch.from_numpy(np.ascontiguousarray(A.T if order == "F" else A).copy())
    if pinned:
        t = t.pin_memory()
    return t.t() if order == "F" else t


def _factor(stf, A, nb, cap, order="F", pinned=True):
    stf.set_option("mem_cap_tiles", cap)
    try:
        t = _host(A, order, pinned)
        info = stf.potrf(t, nb)
        st = stf.last_stats()
    finally:
        stf.set_option("mem_cap_tiles", 0)
    return t.numpy().copy(), info, st


@pytest.mark.parametrize("cap", [3, 5, 12, 24])
@pytest.mark.parametrize("order", ["F", "C"])
def test_out_of_core_bit_equal_to_in_core(stf, cap, order):
    n, nb = 2048, 256
    T = n // nb
    NT = T * (T + 1) // 2
    A = synth.spd_matrix(5, n)
    A[np.triu_indices(n, 1)] = 777.0  # the unreferenced triangle must come back untouched
    ref, info0, st0 = _factor(stf, A, nb, 0, order)
    got, info, st = _factor(stf, A, nb, cap, order)
    assert info0 == 0 and info == 0
    assert st0["frames"] == 0 and st["frames"] == cap
    assert st["host_stores"] >= NT and st["host_loads"] >= NT
    assert np.array_equal(np.tril(got), np.tril(ref))
    assert np.all(got[np.triu_indices(n, 1)] == 777.0)
    Lo, _ = oracle.potrf(synth.spd_matrix(5, n))
    assert relF(np.tril(got), Lo) <= 1e-10


def test_out_of_core_pageable_host_memory(stf):
    n, nb = 1536, 256
    A = synth.spd_matrix(6, n)
    ref, _, _ = _factor(stf, A, nb, 0, "F", pinned=False)
    got, info, st = _factor(stf, A, nb, 7, "F", pinned=False)
    assert info == 0 and st["frames"] == 7 and st["graph_nodes"] == 0  # pageable: eager lowering
    assert np.array_equal(np.tril(got), np.tril(ref))


@pytest.mark.parametrize("j", [0, 255, 256, 1000, 2047])
def test_out_of_core_info(stf, j):
    n, nb = 2048, 256
    A = synth.spd_matrix(3, n)
    A[j, j] = -1.0
    _, info, _ = _factor(stf, A, nb, 6)
    assert info == j + 1


def test_out_of_core_larger_tiles_and_repeat(stf):
    """T = 16 with 20 frames (15% of the tiles); twice in a row (memoised plan)."""
    n, nb = 8192, 512
    A = synth.spd_matrix(8, n)
    stf.set_option("host_stream", 0)  # reference: the right-looking in-core plan
    try:
        ref, _, _ = _factor(stf, A, nb, 0)
    finally:
        stf.set_option("host_stream", 1)
    for rep in range(2):
        got, info, st = _factor(stf, A, nb, 20)
        assert info == 0 and st["frames"] == 20
        assert st["graph_reuse"] == (1 if rep else 0)
        assert np.array_equal(np.tril(got), np.tril(ref))


def test_out_of_core_rejected_on_several_gpus(stf):
    A = synth.spd_matrix(1, 512)
    stf.set_option("mem_cap_tiles", 4)
    try:
        t = _host(A, "F")
        with pytest.raises(stf.StfError) as e:
            stf.potrf(t, 128, ngpus=2)
        assert e.value.code == -105
    finally:
        stf.set_option("mem_cap_tiles", 0)


@pytest.mark.parametrize("ooc_order", [0, 1])
def test_out_of_core_orders_bit_equal(stf, ooc_order):
    """Both program orders of the out-of-core plan (tall super-columns, 2D-blocked
    row chunks) give the in-core call's bits; the 2D order loads fewer tiles."""
    n, nb, cap = 4096, 256, 20
    A = synth.spd_matrix(9, n)
    ref, _, _ = _factor(stf, A, nb, 0)
    stf.set_option("ooc_order", ooc_order)
    try:
        got, info, st = _factor(stf, A, nb, cap)
    finally:
        stf.set_option("ooc_order", -1)
    assert info == 0 and st["frames"] == cap
    assert np.array_equal(np.tril(got), np.tril(ref))
    stf.set_option("ooc_order", 1 - ooc_order)
    try:
        _, _, st_other = _factor(stf, A, nb, cap)
    finally:
        stf.set_option("ooc_order", -1)
    two_d, tall = (st, st_other) if ooc_order == 1 else (st_other, st)
    assert two_d["host_loads"] < tall["host_loads"]


@pytest.mark.parametrize("n,nb,order", [(8192, 512, "F"), (8192, 512, "C"), (4096, 256, "F"), (8192, 1024, "F")])
def test_host_stream_plan_bit_equal_to_right_looking_plan(stf, n, nb, order):
    """An uncapped HOST_COLMAJOR call at nb >= 512 and T >= 16 runs the
    out-of-core builder with one frame per tile ("host_stream", default); it must
    give the bits of the right-looking plan with LOAD/STORE tasks (host_stream 0)
    and load and write back every tile exactly once.  Below those sizes the
    right-looking plan runs either way."""
    T = n // nb
    NT = T * (T + 1) // 2
    A = synth.spd_matrix(12, n)
    A[np.triu_indices(n, 1)] = 777.0
    stf.set_option("host_stream", 0)
    try:
        ref, info0, st0 = _factor(stf, A, nb, 0, order)
    finally:
        stf.set_option("host_stream", 1)
    got, info, st = _factor(stf, A, nb, 0, order)
    assert info0 == 0 and info == 0
    streamed = nb >= 512 and T >= 16
    assert st0["frames"] == 0 and st["frames"] == (NT if streamed else 0)
    assert st["host_loads"] == NT and st["host_stores"] == NT
    assert np.array_equal(np.tril(got), np.tril(ref))
    assert np.all(got[np.triu_indices(n, 1)] == 777.0)
