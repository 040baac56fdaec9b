"""Pins for the CPU oracle.

The oracle must be checked against something other than itself: closed forms,
exact rational arithmetic, LAPACK, invariants and the paper's worked example.
Each pin is chosen so a plausible slip in the oracle (dropped term, wrong sign,
wrong index, transposed operand) fails at least one of them.
"""
import math
import os
from decimal import Decimal, getcontext
from fractions import Fraction

import numpy as np
import pytest

import oracle
import synth

EPS = np.finfo(np.float64).eps
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def relF(X, Y):
    return np.linalg.norm(X - Y) / np.linalg.norm(Y)


def backward_ratio(A, L):
    """||A - L L^T||_F / (||A||_F * n * eps), lower triangle of A."""
    n = A.shape[0]
    Asym = np.tril(A) + np.tril(A, -1).T
    return np.linalg.norm(Asym - L @ L.T) / (np.linalg.norm(Asym) * n * EPS)


# ---------------------------------------------------------------- P1
@pytest.mark.parametrize("n", [1, 2, 7, 64, 256])
def test_p1_min_matrix_bit_exact(n):
    L, info = oracle.potrf(synth.min_matrix(n))
    assert info == 0
    assert np.array_equal(L, np.tril(np.ones((n, n))))


# ---------------------------------------------------------------- P2
@pytest.mark.parametrize("n,seed", [(16, 101), (256, 101), (512, 102)])
def test_p2_dyadic_unit_lower_bit_exact(n, seed):
    A, L0 = synth.dyadic_spd(seed, n)
    # the construction itself must be non-trivial (entries of both signs, many nonzeros)
    assert (L0[np.tril_indices(n, -1)] > 0).any() and (L0[np.tril_indices(n, -1)] < 0).any()
    L, info = oracle.potrf(A)
    assert info == 0
    assert np.array_equal(L, L0)


# ---------------------------------------------------------------- P3
@pytest.mark.parametrize("n", [1, 5, 100])
def test_p3_diagonal_bit_exact(n):
    A = synth.diag_matrix(7, n)
    L, info = oracle.potrf(A)
    assert info == 0
    assert np.array_equal(L, np.diag(np.sqrt(np.diag(A))))


# ---------------------------------------------------------------- P4
def _read_golden_p4():
    rows = [ln.split() for ln in open(os.path.join(GOLDEN, "p4_2x2.txt")) if ln.strip() and not ln.startswith("#")]
    n = int(rows[0][0])
    A = np.array([float(x) for x in rows[1]]).reshape(n, n)
    L = np.array([float(x) for x in rows[2]]).reshape(n, n)
    return A, L


def test_p4_2x2_golden():
    A, Lref = _read_golden_p4()
    L, info = oracle.potrf(A)
    assert info == 0
    assert np.array_equal(L, Lref)


@pytest.mark.parametrize("a,b,c", [(4.0, 2.0, 5.0), (2.0, -1.0, 3.0), (9.0, 0.5, 1.0)])
def test_p4_2x2_closed_form(a, b, c):
    L, info = oracle.potrf(np.array([[a, b], [b, c]]))
    assert info == 0
    l00 = math.sqrt(a)
    l10 = b / l00
    l11 = math.sqrt(c - l10 * l10)
    assert L[0, 0] == l00 and L[1, 0] == l10 and L[0, 1] == 0.0
    assert abs(L[1, 1] - l11) <= 2 * EPS * l11


def test_oracle_reads_lower_triangle_only():
    A = synth.spd_matrix(3, 33)
    B = np.array(A)
    B[np.triu_indices(33, 1)] = np.nan  # strictly upper must not be referenced
    L1, _ = oracle.potrf(A)
    L2, _ = oracle.potrf(B)
    assert np.array_equal(L1, L2)


# ---------------------------------------------------------------- P5
def _exact_cholesky(A_int):
    """Exact rational LDL^T, then L = l * sqrt(d) with 60-digit decimal sqrt."""
    n = len(A_int)
    l = [[Fraction(0)] * n for _ in range(n)]
    d = [Fraction(0)] * n
    for j in range(n):
        d[j] = Fraction(A_int[j][j]) - sum(l[j][k] ** 2 * d[k] for k in range(j))
        l[j][j] = Fraction(1)
        for i in range(j + 1, n):
            l[i][j] = (Fraction(A_int[i][j]) - sum(l[i][k] * l[j][k] * d[k] for k in range(j))) / d[j]
    getcontext().prec = 60
    L = np.zeros((n, n))
    for j in range(n):
        sd = Decimal(d[j].numerator) / Decimal(d[j].denominator)
        sd = sd.sqrt()
        for i in range(j, n):
            v = Decimal(l[i][j].numerator) / Decimal(l[i][j].denominator) * sd
            L[i, j] = float(v)
    return L


@pytest.mark.parametrize("n", [2, 3, 4, 5, 6, 7, 8])
def test_p5_bruteforce_exact_rational(n):
    rng = np.random.default_rng(1000 + n)
    for _ in range(5):
        B = rng.integers(-4, 5, size=(n, n))
        A_int = (B @ B.T + n * np.eye(n, dtype=np.int64)).astype(np.int64)
        Lref = _exact_cholesky(A_int.tolist())
        L, info = oracle.potrf(A_int.astype(np.float64))
        assert info == 0
        for i in range(n):
            scale = np.max(np.abs(Lref[i, : i + 1]))
            assert np.all(np.abs(L[i] - Lref[i]) <= 8 * n * EPS * scale), (i, L[i], Lref[i])


# ---------------------------------------------------------------- P6
@pytest.mark.parametrize("rho,tol", [(0.5, 1e-14), (0.9, 1e-13), (0.99, 1e-12)])
def test_p6_kms_closed_form(rho, tol):
    n = 512
    L, info = oracle.potrf(synth.kms_matrix(n, rho))
    assert info == 0
    i = np.arange(n)
    Lref = np.where(i[:, None] >= i[None, :], rho ** (i[:, None] - i[None, :]).clip(0).astype(float), 0.0)
    Lref[1:, 1:] *= math.sqrt(1 - rho * rho)
    assert relF(L, Lref) <= tol


# ---------------------------------------------------------------- P7
@pytest.mark.parametrize("n,seed", [(1, 2), (17, 3), (300, 4), (1024, 1)])
def test_p7_against_lapack(n, seed):
    A = synth.spd_matrix(seed, n)
    L, info = oracle.potrf(A)
    assert info == 0
    Lref = np.linalg.cholesky(A)
    assert relF(L, Lref) <= 1e-13


# ---------------------------------------------------------------- P8
@pytest.mark.parametrize("n", [64, 512])
def test_p8_invariants(n):
    A = synth.spd_matrix(5, n)
    L, info = oracle.potrf(A, nthreads=2)
    assert info == 0
    assert np.all(np.diag(L) > 0)
    assert np.all(L[np.triu_indices(n, 1)] == 0)
    assert backward_ratio(A, L) <= 10


def test_thread_count_does_not_change_bits():
    A = synth.spd_matrix(9, 300)
    L1, _ = oracle.potrf(A, nthreads=1)
    L4, _ = oracle.potrf(A, nthreads=4)
    assert np.array_equal(L1, L4)


# ---------------------------------------------------------------- P10
@pytest.mark.parametrize("j", [0, 63, 64, 255])
def test_p10_info_first_failing_column(j):
    n = 256
    A = synth.spd_matrix(1, n)
    A[j, j] = -1.0
    _, info = oracle.potrf(A)
    assert info == j + 1


def test_info_nan_pivot():
    A = synth.spd_matrix(1, 40)
    A[10, 3] = np.nan  # poisons column 3 from row 10 -> pivot of column 10 is NaN
    _, info = oracle.potrf(A)
    assert info == 11


def test_n_zero():
    L, info = oracle.potrf(np.zeros((0, 0)))
    assert info == 0 and L.shape == (0, 0)


# ---------------------------------------------------------------- P11 (STF rule + task list)
def _read_alg1():
    lines = [ln.strip() for ln in open(os.path.join(GOLDEN, "alg1_dag.txt")) if ln.strip() and not ln.startswith("#")]
    k = lines.index("edges")
    tasks = []
    for ln in lines[:k]:
        parts = ln.split()[1:]
        tasks.append([(p.split(":")[0], p.split(":")[1]) for p in parts])
    edges = {tuple(int(x) for x in ln.split()) for ln in lines[k + 1:]}
    return tasks, edges


def test_p11_alg1_worked_example():
    tasks, golden = _read_alg1()
    assert oracle.stf_edges(tasks) == golden


def test_stf_rule_read_after_read_is_free_and_war_is_ordered():
    # r, r, rw on one datum: the two readers are concurrent, the writer waits for both
    e = oracle.stf_edges([[("D", "r")], [("D", "r")], [("D", "rw")]])
    assert e == {(0, 2), (1, 2)}


def _reduction(n, edges):
    R = oracle.transitive_closure(n, edges)
    red = set()
    for s, t in edges:
        # (s,t) is redundant iff some successor u != t of s reaches t
        if not any(R[u, t] for (s2, u) in edges if s2 == s and u != t):
            red.add((s, t))
    return red


@pytest.mark.parametrize("T", [1, 2, 3, 4, 6, 8])
def test_p11_cholesky_task_and_edge_counts(T):
    tasks = oracle.cholesky_tasks(T)
    G = T * (T - 1) * (T - 2) // 6
    assert len(tasks) == T + T * (T - 1) + G
    edges = oracle.stf_edges([acc for _, _, acc in tasks])
    red = _reduction(len(tasks), edges)
    # closed form of the reduced DAG (SURVEY.md §8(a) "Incoming edges"):
    expect = (T - 1) + 2 * (T * (T - 1) - (T - 1)) + (3 * G - (T - 1) * (T - 2) // 2 if T >= 2 else 0)
    assert len(red) == expect
    if T == 4:
        assert len(red) == 30
    if T == 8:
        assert len(red) == 252
    # every surviving edge is read-after-write (no WAR/WAW survives the reduction)
    for s, t in red:
        ws = {d for d, m in tasks[s][2] if m == oracle.RW}
        rt = {d for d, m in tasks[t][2] if m == oracle.READ} | {d for d, m in tasks[t][2] if m == oracle.RW}
        assert ws & rt


@pytest.mark.parametrize("T", [4, 8])
def test_p11_critical_path(T):
    tasks = oracle.cholesky_tasks(T)
    edges = oracle.stf_edges([acc for _, _, acc in tasks])
    depth = [1] * len(tasks)
    for s, t in sorted(edges, key=lambda e: e[1]):
        depth[t] = max(depth[t], depth[s] + 1)
    assert max(depth) == 3 * T - 2


@pytest.mark.parametrize("n,nb", [(64, 16), (96, 32), (256, 64)])
def test_tiled_task_list_matches_unblocked(n, nb):
    A = synth.spd_matrix(11, n)
    Lt, info = oracle.tiled_potrf(A, nb)
    L, _ = oracle.potrf(A)
    assert info == 0
    assert relF(Lt, L) <= 1e-14


def test_tiled_task_list_dyadic_bit_exact():
    A, L0 = synth.dyadic_spd(101, 128)
    Lt, info = oracle.tiled_potrf(A, 32)
    assert info == 0 and np.array_equal(Lt, L0)
