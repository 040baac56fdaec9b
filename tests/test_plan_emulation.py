"""Execute the library's plans (the exact task list, buffers and DAG edges that
stf_potrf lowers) on the CPU with the oracle's tile operations, in RANDOM
topological orders of the DAG.  An edge the plan is missing -- a replica read
before its COPY, a frame reloaded while a reader still needs the old tile, a
reload before the write-back -- lets some order read a wrong tile, and the
result leaves oracle.tiled_potrf's bits.  Since every tile still receives its
updates k = 0, 1, ... in order, the result must equal oracle.tiled_potrf
bit for bit.  Integer/ordering work: exact comparison.  No GPU needed.

Covers the 2D block-cyclic plans with replicas (§8 rows a3/a5/a7), the
fence ablation (NEXT-1) and the out-of-core plans over F device frames with
LOAD/STORE tasks (NEXT-4)."""
import numpy as np
import pytest

import oracle
import paper_conf_sc_augonnetasg24_b200 as stf
import synth

NB = 4  # tile order for the emulation (values are irrelevant to the schedule)


def _plan(T, p, q, frames=0, lookahead=1, ooc_order=1, push=0, merge=0, group=2):
    """Plan of stf_dag_build with these options (gemm_merge restored to its default 2 after)."""
    stf.set_option("mem_cap_tiles", frames)
    stf.set_option("lookahead", lookahead)
    stf.set_option("ooc_order", ooc_order)
    stf.set_option("push", push)
    stf.set_option("gemm_merge", merge)
    stf.set_option("gemm_group", group)
    try:
        edges, kinds, ijk, st = stf.dag(T, p, q)
        io, nbuf = stf.dag_io(len(kinds))
        _extras(len(kinds))
    finally:
        stf.set_option("mem_cap_tiles", 0)
        stf.set_option("lookahead", 1)
        stf.set_option("ooc_order", -1)
        stf.set_option("push", 0)
        stf.set_option("gemm_merge", 2)
        stf.set_option("gemm_group", -1)
    return edges, kinds, ijk, io, nbuf, st


_MIRRORS = []  # replica writes (fused push) of the tasks of the last _plan()
_IO2 = []      # second operand pair of merged GEMM tasks of the last _plan()


def _extras(ntasks):
    _MIRRORS.clear()
    _MIRRORS.extend(stf.dag_mirrors(ntasks))
    _IO2.clear()
    _IO2.extend(stf.dag_io2(ntasks))


def _emulate(T, A, kinds, ijk, io, nbuf, edges, order_seed, host_resident):
    """Run the tasks in a random topological order (Kahn, random ready pick)."""
    nb = NB
    # column-major tiles written in place, as oracle.tiled_potrf does (numpy's
    # matmul rounding depends on operand layout)
    H = {(i, j): np.asfortranarray(A[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb]) for i in range(T) for j in range(i + 1)}
    buf = [np.zeros((nb, nb), order="F") for _ in range(nbuf)]
    if not host_resident:  # TILED_2DBC: home buffers hold the caller's tiles
        for (i, j), t in H.items():
            buf[i * (i + 1) // 2 + j][:, :] = t
    n = len(kinds)
    succ = [[] for _ in range(n)]
    indeg = [0] * n
    for s, d in edges:
        succ[s].append(d)
        indeg[d] += 1
    rng = np.random.default_rng(max(order_seed, 0))
    ready = [t for t in range(n) if indeg[t] == 0]
    done = 0
    while ready:
        t = ready.pop(int(rng.integers(len(ready))) if order_seed >= 0 else 0)
        (r0, r1), w = io[t]
        kd = kinds[t]
        i, j, k = ijk[t]
        if kd == "POTRF":
            L, info = oracle.potrf(buf[w])
            assert info == 0
            buf[w][:, :] = L
        elif kd == "TRSM":
            buf[w][:, :] = oracle.tile_trsm(buf[w], buf[r0])
        elif kd == "SYRK":
            buf[w][:, :] = oracle.tile_syrk(buf[w], buf[r0])
        elif kd == "GEMM":
            buf[w][:, :] = oracle.tile_gemm(buf[w], buf[r0], buf[r1])
            for a2, b2 in (_IO2[t] if _IO2 else []):  # merged task: updates k+1, .. right after update k
                buf[w][:, :] = oracle.tile_gemm(buf[w], buf[a2], buf[b2])
        elif kd == "COPY":
            buf[w][:, :] = buf[r0]
        elif kd == "LOAD":
            buf[w][:, :] = H[(i, j)]
        elif kd == "STORE":
            H[(i, j)][:, :] = buf[r0]
        else:
            assert kd == "FENCE"
        if _MIRRORS and kd in ("POTRF", "TRSM"):  # fused push: the epilogue also writes these replicas
            for m in _MIRRORS[t]:
                buf[m][:, :] = buf[w]
        done += 1
        for d in succ[t]:
            indeg[d] -= 1
            if indeg[d] == 0:
                ready.append(d)
        if order_seed < 0:
            ready.sort()
    assert done == n, "the plan's DAG has a cycle"
    out = np.zeros((T * nb, T * nb))
    for (i, j) in H:
        tile = H[(i, j)] if host_resident else buf[i * (i + 1) // 2 + j]
        out[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb] = tile
    return np.tril(out)


def _reference(T, A):
    L, info = oracle.tiled_potrf(A, NB)
    assert info == 0
    return np.tril(L)


@pytest.mark.parametrize("push", [0, 1])
@pytest.mark.parametrize("T,p,q,lookahead", [(5, 1, 1, 1), (6, 1, 2, 1), (6, 2, 2, 1), (7, 2, 4, 1), (6, 2, 2, 0),
                                             (9, 1, 8, 1), (9, 1, 8, 0)])
def test_distributed_plan_any_topological_order(T, p, q, lookahead, push):
    """2D block-cyclic grids and the 1D column block-cyclic 1 x 8 grid (cuSolverMg's
    layout), with and without per-step fences, COPY tasks or fused pushes."""
    A = synth.spd_matrix(7, T * NB)
    edges, kinds, ijk, io, nbuf, st = _plan(T, p, q, lookahead=lookahead, push=push)
    if push and p * q > 1:
        assert "COPY" not in kinds and st["pushed"] == st["transfers"] > 0
    ref = _reference(T, A)
    for seed in (-1, 1, 2, 3):
        got = _emulate(T, A, kinds, ijk, io, nbuf, edges, seed, host_resident=False)
        assert np.array_equal(got, ref), (seed, np.abs(got - ref).max())


@pytest.mark.parametrize("list_order", [False, True])
@pytest.mark.parametrize("ooc_order", [0, 1, -1])
@pytest.mark.parametrize("T,frames", [(4, 3), (4, 5), (6, 3), (6, 4), (6, 7), (6, 12), (8, 6), (8, 20), (9, 10),
                                      (12, 9), (12, 30)])
def test_out_of_core_plan_any_topological_order(T, frames, ooc_order, list_order):
    """list_order: the plan re-submitted in simulated list-scheduling order
    (order_mode 2, what the runtime does at nb >= 512)."""
    A = synth.spd_matrix(11, T * NB)
    stf.set_option("order_mode", 2 if list_order else -1)
    try:
        edges, kinds, ijk, io, nbuf, st = _plan(T, 1, 1, frames=frames, ooc_order=ooc_order)
    finally:
        stf.set_option("order_mode", -1)
    NT = T * (T + 1) // 2
    assert st["frames"] == frames and nbuf == frames
    assert "COPY" not in kinds
    # every buffer a task touches is a frame; each tile is loaded and written back at least once
    for (r0, r1), w in io:
        assert all(-1 <= b < frames for b in (r0, r1, w))
    assert st["host_loads"] >= NT and st["host_stores"] >= NT
    assert kinds.count("LOAD") == st["host_loads"] and kinds.count("STORE") == st["host_stores"]
    ref = _reference(T, A)
    for seed in (-1, 1, 2, 3, 4):
        got = _emulate(T, A, kinds, ijk, io, nbuf, edges, seed, host_resident=True)
        assert np.array_equal(got, ref), (seed, np.abs(got - ref).max())


def test_out_of_core_compute_order_matches_stf_closure():
    """Frames add orderings (WAR on reuse), never drop one: every pair the
    single-GPU STF closure orders is still ordered among the compute tasks."""
    T, frames = 6, 5
    edges, kinds, ijk, io, nbuf, st = _plan(T, 1, 1, frames=frames)
    comp = [t for t, k in enumerate(kinds) if k in ("POTRF", "TRSM", "SYRK", "GEMM")]
    R = oracle.transitive_closure(len(kinds), set(edges))
    ot = oracle.cholesky_tasks(T)
    Ro = oracle.transitive_closure(len(ot), oracle.stf_edges([acc for _, _, acc in ot]))
    # map our compute tasks (left-looking order) onto the oracle's task list by (kind, i, j, k)
    name = {}
    for idx, (kd, (i, j, k), _) in enumerate(ot):
        name[(kd, i, j, k)] = idx
    ours = []
    for t in comp:
        kd = kinds[t]
        i, j, k = ijk[t]
        # library names: TRSM(i,k) = (i,k,k), SYRK(i,k) = (i,i,k) -- same as the oracle's
        ours.append(name[(kd, i, j, k)])
    assert sorted(ours) == list(range(len(ot)))
    sub = R[np.ix_(comp, comp)]
    for a, ta in enumerate(ours):
        for b, tb in enumerate(ours):
            if Ro[ta, tb]:
                assert sub[a, b], (kinds[comp[a]], ijk[comp[a]], kinds[comp[b]], ijk[comp[b]])


def test_out_of_core_traffic_left_looking():
    """With room for wide super-columns the plan re-reads far fewer tiles than a
    right-looking sweep: loads stay within a small multiple of the tile count."""
    T = 16
    NT = T * (T + 1) // 2
    _, _, _, _, _, st_small = _plan(T, 1, 1, frames=24)
    _, _, _, _, _, st_big = _plan(T, 1, 1, frames=NT // 2)
    assert st_big["host_loads"] < st_small["host_loads"]
    assert st_big["host_stores"] == NT  # every tile written back exactly once
    assert st_big["host_loads"] <= 3 * NT
    _, _, _, _, _, st_none = _plan(T, 1, 1, frames=NT)  # cap >= matrix: no out-of-core plan
    assert st_none["frames"] == 0 and st_none["host_loads"] == 0


def test_out_of_core_2d_order_cuts_panel_reloads():
    """The 2D-blocked order (row chunks under each column block) re-reads fewer
    panel tiles than tall super-columns once a trailing column alone fills the
    frames (T = 32: the bench's n = 32768, nb = 1024), and never loads a tile
    less than once or writes one back more than once per eviction."""
    T = 32
    NT = T * (T + 1) // 2
    for frames, gain in ((33, 0.75), (66, 0.75), (132, 0.95)):
        st0 = _plan(T, 1, 1, frames=frames, ooc_order=0)[5]
        st1 = _plan(T, 1, 1, frames=frames, ooc_order=1)[5]
        assert NT <= st1["host_loads"] <= gain * st0["host_loads"], (frames, st0["host_loads"], st1["host_loads"])
        assert st1["host_stores"] == NT


def _call_plan(n, nb, kind, p=1, q=1):
    edges, kinds, ijk, st = stf.dag_call(n, nb, kind, p, q)
    io, nbuf = stf.dag_io(len(kinds))
    _extras(len(kinds))
    return edges, kinds, ijk, io, nbuf, st


@pytest.mark.parametrize("n,nb,kind,p,q", [
    (32768, 1024, stf.STF_DESC_HOST_COLMAJOR, 1, 1),   # bench e2e: host_stream plan, T = 32
    (16384, 512, stf.STF_DESC_HOST_COLMAJOR, 1, 1),    # host_stream plan, T = 32, nb = 512
    (16384, 1024, stf.STF_DESC_HOST_COLMAJOR, 1, 1),   # host_stream plan, T = 16 (smallest T it serves)
    (8192, 1024, stf.STF_DESC_HOST_COLMAJOR, 1, 1),    # T = 8: right-looking plan with LOAD/STORE tasks
    (32768, 1024, stf.STF_DESC_TILED_2DBC, 1, 1),      # bench: device tiles, list order over the last 8 steps
    (32768, 1024, stf.STF_DESC_TILED_2DBC, 2, 4),      # the 8-GPU grid of the bench's scaling run
    (16384, 1024, stf.STF_DESC_HOST_COLMAJOR, 2, 2),   # HOST_COLMAJOR on 4 GPUs
])
def test_call_plans_any_topological_order(n, nb, kind, p, q):
    """The exact plans stf_potrf executes for the configurations bench.py and
    the e2e measurement report (stf_dag_build_call: same code path as the call,
    including the host_stream builder and the list-scheduling re-submission),
    executed with the oracle's tile operations on 4 x 4 tiles in random
    topological orders: oracle.tiled_potrf's bits in every order."""
    T = n // nb
    edges, kinds, ijk, io, nbuf, st = _call_plan(n, nb, kind, p, q)
    NT = T * (T + 1) // 2
    # merged GEMM tasks (gemm_merge, device-resident plans) carry several tile updates each
    assert st["tasks"] + sum(len(x) for x in _IO2) == T + T * (T - 1) + T * (T - 1) * (T - 2) // 6
    host = kind == stf.STF_DESC_HOST_COLMAJOR
    if host and p * q == 1 and T >= 16:
        assert st["frames"] == NT  # host_stream: one frame per tile, nothing evicted
    if host:
        assert st["host_loads"] == NT and st["host_stores"] == NT
    A = synth.spd_matrix(13, T * NB)
    ref = _reference(T, A)
    for seed in (-1, 1, 2):
        got = _emulate(T, A, kinds, ijk, io, nbuf, edges, seed, host_resident=host)
        assert np.array_equal(got, ref), (seed, np.abs(got - ref).max())


def test_call_plan_fence_and_stream_pool_ablations():
    """lookahead=0 (fence per step) and the reduced stream pools keep the
    right-looking builder for host calls (they implement those variants), and
    stay exact in any order."""
    n, nb, T = 16384, 1024, 16
    A = synth.spd_matrix(14, T * NB)
    ref = _reference(T, A)
    for name, val in (("lookahead", 0), ("stream_pool", 1), ("stream_pool", 2)):
        stf.set_option(name, val)
        try:
            edges, kinds, ijk, io, nbuf, st = _call_plan(n, nb, stf.STF_DESC_HOST_COLMAJOR)
        finally:
            stf.set_option(name, 1 if name == "lookahead" else 0)
        assert st["frames"] == 0, name
        assert ("FENCE" in kinds) == (name == "lookahead")
        got = _emulate(T, A, kinds, ijk, io, nbuf, edges, 5, host_resident=True)
        assert np.array_equal(got, ref), name


def test_out_of_core_rejects_fence_ablation():
    stf.set_option("mem_cap_tiles", 10)
    stf.set_option("lookahead", 0)
    try:
        with pytest.raises(stf.StfError):
            stf.dag(8, 1, 1)
        with pytest.raises(stf.StfError):
            stf.dag_call(8192, 1024, stf.STF_DESC_HOST_COLMAJOR)
    finally:
        stf.set_option("mem_cap_tiles", 0)
        stf.set_option("lookahead", 1)


@pytest.mark.parametrize("T,p,q,merge,push,group", [(8, 1, 1, 1, 0, 2), (9, 1, 1, 3, 0, 2), (12, 2, 2, 2, 0, 2),
                                                   (12, 2, 4, 3, 1, 2), (10, 1, 8, 1, 0, 2), (16, 1, 1, 3, 0, 2),
                                                   (16, 1, 1, 1, 0, 3), (17, 2, 2, 2, 1, 4), (13, 1, 1, 1, 0, 4)])
def test_merged_gemm_plans_any_topological_order(T, p, q, merge, push, group):
    """gemm_merge: GEMM(i,j,k) and GEMM(i,j,k+1) of far tiles as one task (two
    consecutive updates in one k sweep): the plan stays a correct STF DAG -- the
    oracle's bits in random orders -- with fewer GEMM tasks."""
    A = synth.spd_matrix(17, T * NB)
    e0, k0, _, _, _, st0 = _plan(T, p, q, push=push)
    edges, kinds, ijk, io, nbuf, st = _plan(T, p, q, push=push, merge=merge, group=group)
    assert st["merged_gemms"] > 0 and st0["merged_gemms"] == 0
    extra = sum(len(x) for x in _IO2)  # updates carried by merged tasks beyond their first
    assert kinds.count("GEMM") + extra == k0.count("GEMM")
    assert st["tasks"] + extra == st0["tasks"]
    ref = _reference(T, A)
    for seed in (-1, 1, 2):
        got = _emulate(T, A, kinds, ijk, io, nbuf, edges, seed, host_resident=False)
        assert np.array_equal(got, ref), (seed, np.abs(got - ref).max())


def test_merged_gemm_call_plan_bench_config():
    """The bench's plan (n = 65536, nb = 1024, T = 64) with the default merge
    distance, executed in a random topological order on 4 x 4 tiles."""
    n, nb, T = 65536, 1024, 64
    edges, kinds, ijk, io, nbuf, st = _call_plan(n, nb, stf.STF_DESC_TILED_2DBC)
    assert st["merged_gemms"] > 0
    A = synth.spd_matrix(18, T * NB)
    got = _emulate(T, A, kinds, ijk, io, nbuf, edges, 3, host_resident=False)
    assert np.array_equal(got, _reference(T, A))
