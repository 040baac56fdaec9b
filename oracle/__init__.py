"""ORACLE -- TEST INFRASTRUCTURE ONLY.

Plain CPU implementations of what the hot path computes, written from the
paper, used to check the CUDA path.  Only ``tests/``, ``__graft_entry__.smoke()``
and ``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  It never imports ``paper_conf_sc_augonnetasg24_b200`` and the product
never imports it.

Functions and the passages they follow:

* :func:`potrf` -- the Cholesky factor L of A = L L^T (PAPER.md:384, :393,
  §VII-C; the plain definition); C code in ``oracle_potrf.c``.
  Pinned by tests/test_oracle.py (P1-P8, P10 of SURVEY.md §8(c)).
* :func:`cholesky_tasks` -- the right-looking tiled Cholesky task sequence in
  program order with each task's access modes (ref. [17] PAPER.md:495; "one
  logical data object per tile").  Pinned by task counts in
  closed form and by the reduction to LAPACK (tests/test_oracle.py).
* :func:`stf_edges` -- the STF dependency rule of PAPER.md:144 (§II-B), applied
  literally by brute force: every task depends on every earlier task that
  modifies one of its data, and, when it modifies a datum, on every earlier
  reader of it.  Pinned by the worked example of Algorithm 1 / Fig. 1
  (tests/golden/alg1_dag.txt).
* :func:`tile_gemm`, :func:`tile_syrk`, :func:`tile_trsm` -- the tile tasks
  of PAPER.md:393 written as their definitions (numpy matmul as a step).
* :func:`tiled_potrf` -- executes :func:`cholesky_tasks` in a topological
  order of :func:`stf_edges` with numpy tile operations (definition of each
  tile task), proving the task list + rule compute the same L as
  :func:`potrf` up to rounding.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Dict, List, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle_potrf.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle_potrf.c into oracle/liboracle.so (plain gcc, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O3", "-fopenmp", "-ffp-contract=off", "-fno-fast-math", "-shared",
               "-fPIC", "-o", _LIB, _SRC, "-lm"]
        subprocess.check_call(cmd)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.oracle_potrf.restype = ctypes.c_int64
        lib.oracle_potrf.argtypes = [ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64,
                                     ctypes.c_void_p, ctypes.c_int]
        lib.oracle_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def max_threads() -> int:
    return int(_load().oracle_max_threads())


def potrf(A: np.ndarray, nthreads: int = 0) -> Tuple[np.ndarray, int]:
    """Cholesky factor of the lower triangle of A.

    Returns (L, info): L is an n x n float64 array (lower triangular, strictly
    upper zero); info = 0 on success, else the 1-based first failing column
    (LAPACK convention).
    """
    A = np.asarray(A, dtype=np.float64)
    n = A.shape[0]
    assert A.shape == (n, n)
    Af = np.asfortranarray(A)
    L = np.empty((n, n), dtype=np.float64, order="C")  # row-major
    info = _load().oracle_potrf(n, Af.ctypes.data, max(1, n), L.ctypes.data, int(nthreads))
    return L, int(info)


# --------------------------------------------------------------------------
# Task sequence and the STF rule
# --------------------------------------------------------------------------
READ, RW = "r", "rw"


def cholesky_tasks(T: int) -> List[Tuple[str, Tuple[int, ...], Tuple[Tuple[Tuple[int, int], str], ...]]]:
    """Right-looking tiled Cholesky (ref. [17]) in program order.

    Each entry is (kind, (i, j, k) indices, ((tile, mode), ...)) where tile =
    (row, col) of the lower tile A_rc and mode is READ or RW:
        for k:  POTRF(k)           A_kk:rw
                for i>k: TRSM(i,k)  A_kk:r, A_ik:rw
                for i>k: SYRK(i,k)  A_ik:r, A_ii:rw
                         for k<j<i: GEMM(i,j,k)  A_ik:r, A_jk:r, A_ij:rw
    """
    out = []
    for k in range(T):
        out.append(("POTRF", (k, k, k), (((k, k), RW),)))
        for i in range(k + 1, T):
            out.append(("TRSM", (i, k, k), (((k, k), READ), ((i, k), RW))))
        for i in range(k + 1, T):
            out.append(("SYRK", (i, i, k), (((i, k), READ), ((i, i), RW))))
            for j in range(k + 1, i):
                out.append(("GEMM", (i, j, k), (((i, k), READ), ((j, k), READ), ((i, j), RW))))
    return out


def stf_edges(accesses: Sequence[Sequence[Tuple[object, str]]]) -> set:
    """Literal STF rule, brute force O(tasks^2).

    For task t and each datum d it accesses: an edge s -> t for every s < t that
    modifies d; if t modifies d, also an edge s -> t for every s < t that reads d.
    Returns the set of (s, t) pairs.
    """
    edges = set()
    for t, acc_t in enumerate(accesses):
        for d, mode_t in acc_t:
            for s in range(t):
                for d2, mode_s in accesses[s]:
                    if d2 != d:
                        continue
                    if mode_s != READ or mode_t != READ:
                        edges.add((s, t))
    return edges


def transitive_closure(n: int, edges) -> np.ndarray:
    """Boolean reachability matrix R[s, t] (s ->* t, s != t) of a DAG whose
    edges all go forward in program order."""
    R = np.zeros((n, n), dtype=bool)
    succ: Dict[int, List[int]] = {}
    for s, t in edges:
        succ.setdefault(s, []).append(t)
    for s in range(n - 1, -1, -1):
        for t in succ.get(s, []):
            R[s, t] = True
            R[s] |= R[t]
    return R


# --------------------------------------------------------------------------
# Tiled execution of the task list (numpy tile ops, one definition per task)
# --------------------------------------------------------------------------
def tile_gemm(C: np.ndarray, A: np.ndarray, B: np.ndarray) -> np.ndarray:
    """GEMM tile task: C - A B^T (numpy matmul as a library step)."""
    return C - A @ B.T


def tile_syrk(C: np.ndarray, A: np.ndarray) -> np.ndarray:
    """SYRK tile task: lower triangle of C - A A^T; strictly upper of C kept."""
    return np.tril(C - A @ A.T) + np.triu(C, 1)


def tile_trsm(B: np.ndarray, L: np.ndarray) -> np.ndarray:
    """TRSM tile task: X with X L^T = B, L lower (only its lower
    triangle is read); column-by-column forward substitution in plain numpy:
    x_c = (b_c - sum_{p<c} x_p L_cp) / L_cc."""
    L = np.tril(L)
    X = np.array(B, dtype=np.float64)
    for c in range(L.shape[0]):
        if c:
            X[:, c] -= X[:, :c] @ L[c, :c]
        X[:, c] /= L[c, c]
    return X


def tiled_potrf(A: np.ndarray, nb: int) -> Tuple[np.ndarray, int]:
    """Run cholesky_tasks(T) in program order (a valid topological order of the
    STF DAG) on nb x nb tiles with the textbook tile operations of PAPER.md:393:
        POTRF: A_kk <- chol(A_kk) via :func:`potrf` on the tile
        TRSM:  A_ik <- A_ik L_kk^-T     (forward substitution, tile_trsm)
        SYRK:  A_ii <- A_ii - L_ik L_ik^T
        GEMM:  A_ij <- A_ij - L_ik L_jk^T
    Used only to pin that the task list computes the same factor as potrf().
    """
    A = np.array(A, dtype=np.float64, order="F")
    n = A.shape[0]
    assert n % nb == 0
    T = n // nb

    def tile(i, j):
        return A[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb]

    for kind, (i, j, k), _ in cholesky_tasks(T):
        if kind == "POTRF":
            Lkk, info = potrf(tile(k, k))
            if info:
                return np.tril(A), k * nb + info
            tile(k, k)[:, :] = Lkk
        elif kind == "TRSM":
            tile(i, k)[:, :] = tile_trsm(tile(i, k), tile(k, k))
        elif kind == "SYRK":
            tile(i, i)[:, :] = tile_syrk(tile(i, i), tile(i, k))
        else:
            tile(i, j)[:, :] = tile_gemm(tile(i, j), tile(i, k), tile(j, k))
    return np.tril(A), 0
