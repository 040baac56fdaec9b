"""The host STF scheduler (C++, through the C ABI) against the oracle's literal
STF rule and the task list of ref. [17]: integer work, compared
exactly.  No GPU needed."""
import numpy as np
import pytest

import oracle
import paper_conf_sc_augonnetasg24_b200 as stf

KIND = {"POTRF": "POTRF", "TRSM": "TRSM", "SYRK": "SYRK", "GEMM": "GEMM"}



@pytest.fixture(autouse=True)
def _paper_granularity():
    """These tests check the paper's DAG: one task per tile update (no merged GEMMs)."""
    stf.set_option("gemm_merge", 0)
    yield
    stf.set_option("gemm_merge", 2)

def test_alg1_worked_example_cpp_core():
    # PAPER.md:31-40 (Algorithm 1) -> Fig. 1: {O1->O2, O1->O3, O2->O4, O3->O4}
    X, Y, Z = 0, 1, 2
    tasks = [[(X, "rw")], [(Y, "rw"), (X, "r")], [(Z, "rw"), (X, "r")], [(Z, "rw"), (Y, "r")]]
    assert stf.infer_edges(tasks) == {(0, 1), (0, 2), (1, 3), (2, 3)}


@pytest.mark.parametrize("seed", range(6))
def test_random_access_lists_same_reachability_as_literal_rule(seed):
    rng = np.random.default_rng(seed)
    ntasks, ndata = 40, 6
    tasks = []
    for _ in range(ntasks):
        ds = rng.choice(ndata, size=rng.integers(1, 4), replace=False)
        tasks.append([(int(d), ["r", "w", "rw"][rng.integers(0, 3)]) for d in ds])
    ours = stf.infer_edges(tasks)
    lit = oracle.stf_edges([[(d, "r" if m == "r" else "rw") for d, m in acc] for acc in tasks])
    assert ours <= lit  # never an edge without a conflict
    R1 = oracle.transitive_closure(ntasks, ours)
    R2 = oracle.transitive_closure(ntasks, lit)
    assert np.array_equal(R1, R2)  # every conflicting pair ordered


@pytest.mark.parametrize("T", [1, 2, 3, 4, 5, 8])
def test_cholesky_dag_single_gpu_matches_oracle(T):
    edges, kinds, ijk, st = stf.dag(T, 1, 1)
    ot = oracle.cholesky_tasks(T)
    assert len(kinds) == len(ot) == st["tasks"]
    assert st["transfers"] == 0
    for (kd, (i, j, k)), (okd, (oi, oj, ok), _) in zip(zip(kinds, ijk), ot):
        assert kd == okd
        # the library names tasks by the tile it writes: TRSM(i,k)=(i,k,k), SYRK(i,k)=(i,i,k)
        assert (i, j, k) == (oi, oj, ok)
    lit = oracle.stf_edges([acc for _, _, acc in ot])
    ours = set(edges)
    assert ours <= lit
    assert np.array_equal(oracle.transitive_closure(len(ot), ours), oracle.transitive_closure(len(ot), lit))
    G = T * (T - 1) * (T - 2) // 6
    expect = (T - 1) + 2 * (T * (T - 1) - (T - 1)) + (3 * G - (T - 1) * (T - 2) // 2 if T >= 2 else 0)
    assert st["edges"] == len(ours) == expect
    assert st["critical_path"] == max(1, 3 * T - 2) if T else True


@pytest.mark.parametrize("T,p,q", [(4, 1, 2), (5, 2, 2), (8, 2, 4), (6, 3, 1)])
def test_cholesky_dag_with_transfers_orders_compute_like_oracle(T, p, q):
    """Through replica copies, reachability among compute tasks equals the
    single-GPU STF closure: distribution adds transfers, never reorders."""
    edges, kinds, ijk, st = stf.dag(T, p, q)
    comp = [t for t, k in enumerate(kinds) if k != "COPY"]
    idx = {t: c for c, t in enumerate(comp)}
    R = oracle.transitive_closure(len(kinds), set(edges))
    ot = oracle.cholesky_tasks(T)
    Ro = oracle.transitive_closure(len(ot), oracle.stf_edges([acc for _, _, acc in ot]))
    sub = R[np.ix_(comp, comp)]
    assert np.array_equal(sub, Ro)
    # every COPY moves a tile to a slot that is not its owner, and precedes a reader there
    owner = lambda i, j: (i % p) * q + (j % q)
    for t, k in enumerate(kinds):
        if k == "COPY":
            i, j, dst = ijk[t]
            assert owner(i, j) != dst
    assert idx  # non-empty


def _expected_transfers(T, p, q):
    """Consumers of each final tile L_ij: the owners of every tile that reads it,
    minus its own owner (SURVEY.md §8(e) enumeration)."""
    owner = lambda i, j: (i % p) * q + (j % q)
    total = 0
    for j in range(T):
        for i in range(j, T):
            readers = set()
            if i == j:  # L_kk read by TRSM(r, k), r > k
                readers |= {owner(r, j) for r in range(j + 1, T)}
            else:  # L_ik read by SYRK(i,k), GEMM(i,c,k) (k<c<i), GEMM(r,i,k) (r>i)
                readers.add(owner(i, i))
                readers |= {owner(i, c) for c in range(j + 1, i)}
                readers |= {owner(r, i) for r in range(i + 1, T)}
            readers.discard(owner(i, j))
            total += len(readers)
    return total


@pytest.mark.parametrize("T,p,q,known", [(32, 1, 2, 496), (32, 2, 2, 992), (32, 2, 4, 1892), (64, 2, 4, 7876)])
def test_transfer_counts_match_enumeration(T, p, q, known):
    _, _, _, st = stf.dag(T, p, q)
    assert st["transfers"] == _expected_transfers(T, p, q) == known


@pytest.mark.parametrize("T", [4, 8, 16, 32, 64])
def test_task_counts_closed_form(T):
    _, _, _, st = stf.dag(T, 1, 1)
    assert st["tasks"] == T + T * (T - 1) + T * (T - 1) * (T - 2) // 6
    assert st["critical_path"] == 3 * T - 2


@pytest.mark.parametrize("T,p,q,known", [(8, 2, 2, None), (32, 2, 4, 1892)])
def test_fused_push_replaces_panel_copies(T, p, q, known):
    """NEXT-3: with push on, TRSM(i,k) writes L_ik's replicas and POTRF(k) writes
    L_kk's from their epilogues: no COPY task is left, total transfers are
    unchanged (all of them pushes), and reachability among compute tasks still
    equals the single-GPU STF closure.  With the recursive POTRF (dataflow 0)
    L_kk still moves by COPY."""
    stf.set_option("push", 1)
    try:
        edges, kinds, ijk, st = stf.dag(T, p, q)
        stf.set_option("dataflow", 0)
        _, kinds0, ijk0, st0 = stf.dag(T, p, q)
    finally:
        stf.set_option("push", 0)
        stf.set_option("dataflow", 1)
    assert st["transfers"] == _expected_transfers(T, p, q) == st0["transfers"]
    if known:
        assert st["transfers"] == known
    assert "COPY" not in kinds and st["pushed"] == st["transfers"] and st["data_plane"] == 1
    stf.set_option("push", 2)  # multicast data plane: the same plan (pushes), lowered through one multicast object
    try:
        e2, k2, ijk2, st2 = stf.dag(T, p, q)
    finally:
        stf.set_option("push", 0)
    assert (e2, k2, ijk2) == (edges, kinds, ijk) and st2["data_plane"] == 2
    for t, k in enumerate(kinds0):
        if k == "COPY":
            i, j, _ = ijk0[t]
            assert i == j  # only diagonal (POTRF) tiles are still copied
    comp = [t for t, k in enumerate(kinds) if k != "COPY"]
    R = oracle.transitive_closure(len(kinds), set(edges))
    ot = oracle.cholesky_tasks(T)
    if T <= 8:
        Ro = oracle.transitive_closure(len(ot), oracle.stf_edges([acc for _, _, acc in ot]))
        assert np.array_equal(R[np.ix_(comp, comp)], Ro)


@pytest.mark.parametrize("T,p,q", [(6, 1, 1), (8, 2, 2), (8, 2, 4), (5, 1, 2), (16, 1, 1)])
@pytest.mark.parametrize("order", [("order_asap", 1), ("order_mode", 2), ("dev_order", 1)],
                         ids=["asap", "list", "left_looking"])
def test_submission_orders_same_dag(T, p, q, order, options):
    """The re-submission orders (plan.cpp reorder_asap / reorder_list, the latter
    the default for nb >= 512) are topological orders of the program-order DAG,
    and re-applying the STF rule in that order yields the same DAG (edges
    identical up to the task relabelling): only the stream-order chains change."""
    e0, k0, ijk0, st0 = stf.dag(T, p, q)
    options(*order)
    e1, k1, ijk1, st1 = stf.dag(T, p, q)
    keys0 = [(k, *x) for k, x in zip(k0, ijk0)]
    keys1 = [(k, *x) for k, x in zip(k1, ijk1)]
    assert len(set(keys0)) == len(keys0) and sorted(keys0) == sorted(keys1)
    pos = {key: t for t, key in enumerate(keys1)}
    perm = [pos[key] for key in keys0]
    assert all(a < b for a, b in e1)  # submission order is topological
    assert {(perm[a], perm[b]) for a, b in e0} == set(e1)
    assert st1["critical_path"] == st0["critical_path"] and st1["edges"] == st0["edges"]


def test_list_order_submits_the_panel_chain_early(options):
    """List-scheduling order (default for T <= 16 and COLMAJOR calls): POTRF(k+1)
    is submitted as soon as its chain allows, ahead of bulk updates of step k that
    are not its ancestors (in program order it comes after all of them)."""
    T = 8
    options("order_mode", 2)
    e, k, ijk, st = stf.dag(T, 1, 1)
    pos = {(kd, *x): t for t, (kd, x) in enumerate(zip(k, ijk))}
    for step in range(T - 2):
        assert pos[("POTRF", step + 1, step + 1, step + 1)] < pos[("GEMM", T - 1, T - 2, step)]
    options("order_mode", 0)
    e0, k0, ijk0, _ = stf.dag(T, 1, 1)
    pos0 = {(kd, *x): t for t, (kd, x) in enumerate(zip(k0, ijk0))}
    assert pos0[("POTRF", 1, 1, 1)] > pos0[("GEMM", T - 1, T - 2, 0)]


def test_dag_dot_export(tmp_path):
    """DOT export of the DAG (SURVEY §5 tracing): one node per task, one edge per
    STF dependency, COPY nodes for the replica transfers of a distributed plan."""
    edges, kinds, ijk, st = stf.dag(4, 1, 2)
    path = tmp_path / "chol.dot"
    stf.dag_dot(edges, kinds, ijk, str(path))
    txt = path.read_text()
    assert txt.startswith("digraph stf")
    assert txt.count("->") == st["edges"] == len(edges)
    assert txt.count("[label=") == st["dag_tasks"]
    assert "COPY(" in txt and 'POTRF(0,0,0)' in txt
