"""B200-native STF tiled FP64 Cholesky (CUDASTF, Augonnet et al., SC'24).

Thin Python layer over libstf_cholesky.so (include/stf_cholesky.h).  torch is
used only to allocate device memory for the caller-owned tiles; every step of
the factorisation runs in the library's CUDA kernels.  Import fails loudly if
the library has not been built.
"""
from __future__ import annotations

import ctypes
from typing import List, Optional, Sequence

from . import _abi
from ._abi import (  # noqa: F401  (same names as the C ABI)
    STF_DESC_DEVICE_COLMAJOR,
    STF_DESC_HOST_COLMAJOR,
    STF_DESC_TILED_2DBC,
    StfError,
    check,
    stf_matrix_desc,
    stf_plan_stats,
)

LIB_PATH = _abi.LIB_PATH


def init(ngpus: int = 1, devices: Optional[Sequence[int]] = None) -> None:
    """stf_cholesky_init; devices may repeat an ordinal (virtual GPU slots)."""
    arr = None
    if devices is not None:
        assert len(devices) == ngpus
        arr = (ctypes.c_int * ngpus)(*devices)
    check(_abi.stf_cholesky_init(ngpus, arr), "stf_cholesky_init")


def finalize() -> None:
    check(_abi.stf_finalize(), "stf_finalize")


def set_option(name: str, value: int) -> None:
    check(_abi.stf_set_option(name.encode(), int(value)), "stf_set_option(%s)" % name)


def get_option(name: str) -> int:
    v = ctypes.c_int64()
    check(_abi.stf_get_option(name.encode(), ctypes.byref(v)), "stf_get_option(%s)" % name)
    return v.value


def last_stats() -> dict:
    s = stf_plan_stats()
    check(_abi.stf_last_stats(ctypes.byref(s)), "stf_last_stats")
    return s.as_dict()


def dag(T: int, p: int = 1, q: int = 1):
    """(edges, kinds, ijk, stats) of the plan DAG, built on the host only."""
    st = stf_plan_stats()
    check(_abi.stf_dag_build(T, p, q, 0, None, 0, None, None, ctypes.byref(st)), "stf_dag_build")
    ntasks = st.dag_tasks
    E = (ctypes.c_int64 * (2 * max(1, st.edges)))()
    K = (ctypes.c_int32 * max(1, ntasks))()
    IJK = (ctypes.c_int64 * (3 * max(1, ntasks)))()
    check(_abi.stf_dag_build(T, p, q, st.edges, E, ntasks, K, IJK, ctypes.byref(st)), "stf_dag_build")
    edges = [(E[2 * e], E[2 * e + 1]) for e in range(st.edges)]
    kinds = [_abi.KIND_NAMES[K[t]] for t in range(ntasks)]
    ijk = [(IJK[3 * t], IJK[3 * t + 1], IJK[3 * t + 2]) for t in range(ntasks)]
    return edges, kinds, ijk, st.as_dict()


def dag_call(n: int, nb: int, kind: int = STF_DESC_TILED_2DBC, p: int = 1, q: int = 1, sms: int = 148):
    """(edges, kinds, ijk, stats) of the plan stf_potrf(n, nb, 'L', <kind>, p*q)
    would execute with the current options (stf_dag_build_call), host only."""
    st = stf_plan_stats()
    args = (n, nb, kind, p * q, p, q, sms)
    check(_abi.stf_dag_build_call(*args, 0, None, 0, None, None, ctypes.byref(st)), "stf_dag_build_call")
    ntasks = st.dag_tasks
    E = (ctypes.c_int64 * (2 * max(1, st.edges)))()
    K = (ctypes.c_int32 * max(1, ntasks))()
    IJK = (ctypes.c_int64 * (3 * max(1, ntasks)))()
    check(_abi.stf_dag_build_call(*args, st.edges, E, ntasks, K, IJK, ctypes.byref(st)), "stf_dag_build_call")
    edges = [(E[2 * e], E[2 * e + 1]) for e in range(st.edges)]
    kinds = [_abi.KIND_NAMES[K[t]] for t in range(ntasks)]
    ijk = [(IJK[3 * t], IJK[3 * t + 1], IJK[3 * t + 2]) for t in range(ntasks)]
    return edges, kinds, ijk, st.as_dict()


def dag_dot(edges, kinds, ijk, path: str) -> None:
    """Write the DAG of dag()/dag_call() as a Graphviz DOT file (one node per task,
    labelled KIND(i,j,k); COPY nodes carry the destination slot as k)."""
    col = {"POTRF": "red", "TRSM": "orange", "SYRK": "blue", "GEMM": "gray", "COPY": "green", "LOAD": "cyan",
           "STORE": "cyan", "FENCE": "black"}
    with open(path, "w") as f:
        f.write("digraph stf {\n  node [shape=box, fontsize=9];\n")
        for t, (k, (i, j, kk)) in enumerate(zip(kinds, ijk)):
            f.write('  t%d [label="%s(%d,%d,%d)", color=%s];\n' % (t, k, i, j, kk, col.get(k, "black")))
        for a, b in edges:
            f.write("  t%d -> t%d;\n" % (a, b))
        f.write("}\n")


def dag_io(ntasks: int):
    """(buffers read, buffer written) of every task of the last dag() call, and
    the number of buffers (home tiles + replicas, or device frames out of core)."""
    IO = (ctypes.c_int64 * (3 * max(1, ntasks)))()
    nbuf = check(_abi.stf_dag_tasks_io(ntasks, IO), "stf_dag_tasks_io")
    return [((IO[3 * t], IO[3 * t + 1]), IO[3 * t + 2]) for t in range(ntasks)], nbuf


def dag_io2(ntasks: int):
    """Further operand pairs of merged GEMM tasks: per task a list of (L_i,k+u, L_j,k+u)
    buffer pairs, u = 1.. (empty for a single update)."""
    IO = (ctypes.c_int64 * (6 * max(1, ntasks)))()
    check(_abi.stf_dag_tasks_io2(ntasks, IO), "stf_dag_tasks_io2")
    return [[(IO[6 * t + 2 * u], IO[6 * t + 2 * u + 1]) for u in range(3) if IO[6 * t + 2 * u] >= 0]
            for t in range(ntasks)]


def dag_mirrors(ntasks: int):
    """Replica buffers each task of the last dag()/dag_call() also writes (fused push)."""
    MI = (ctypes.c_int64 * (8 * max(1, ntasks)))()
    check(_abi.stf_dag_tasks_mirrors(ntasks, MI), "stf_dag_tasks_mirrors")
    return [[MI[8 * t + 1 + m] for m in range(MI[8 * t])] for t in range(ntasks)]


def infer_edges(tasks: Sequence[Sequence[tuple]]) -> set:
    """Generic STF rule (C++ core) on [[(datum:int, mode:'r'|'w'|'rw'), ...], ...]."""
    mode_code = {"r": 1, "w": 2, "rw": 3}
    nacc, data, modes = [], [], []
    for acc in tasks:
        nacc.append(len(acc))
        for d, m in acc:
            data.append(int(d))
            modes.append(mode_code[m])
    nt = len(tasks)
    NA = (ctypes.c_int32 * max(1, nt))(*nacc)
    D = (ctypes.c_int64 * max(1, len(data)))(*data)
    M = (ctypes.c_int32 * max(1, len(modes)))(*modes)
    ne = check(_abi.stf_infer_edges(nt, NA, D, M, 0, None), "stf_infer_edges")
    E = (ctypes.c_int64 * (2 * max(1, ne)))()
    check(_abi.stf_infer_edges(nt, NA, D, M, ne, E), "stf_infer_edges")
    return {(E[2 * e], E[2 * e + 1]) for e in range(ne)}


class TiledMatrix:
    """Lower tiles of an n x n matrix distributed 2D block-cyclically over a
    p x q grid of slots: tile (i, j) lives on slot (i % p) * q + (j % q).

    Each slot's tiles are views into ONE torch allocation on that slot's
    device (torch = device memory only).  Tiles are column-major nb x nb
    (ld = nb): tile.view is a (nb, nb) row-major torch tensor holding the
    transpose, i.e. A_ij = tiles[(i, j)].T.
    """

    def __init__(self, n: int, nb: int, p: int = 1, q: int = 1, devices: Optional[Sequence[int]] = None):
        import torch

        assert n % nb == 0
        self.n, self.nb, self.p, self.q = n, nb, p, q
        self.T = T = n // nb
        ng = p * q
        self.devices = list(devices) if devices is not None else list(range(ng))
        assert len(self.devices) == ng
        counts = [0] * ng
        for j in range(T):
            for i in range(j, T):
                counts[self.owner(i, j)] += 1
        self.slabs = [torch.empty((max(1, c), nb, nb), dtype=torch.float64, device="cuda:%d" % self.devices[s])
                      for s, c in enumerate(counts)]
        used = [0] * ng
        self.tiles = {}
        for j in range(T):
            for i in range(j, T):
                s = self.owner(i, j)
                self.tiles[(i, j)] = self.slabs[s][used[s]]
                used[s] += 1
        self._table = (ctypes.c_void_p * (T * T))()
        for (i, j), t in self.tiles.items():
            self._table[i + j * T] = t.data_ptr()
        self.desc = stf_matrix_desc(STF_DESC_TILED_2DBC, 0, 0, None, p, q,
                                    ctypes.cast(self._table, ctypes.POINTER(ctypes.c_void_p)))

    def owner(self, i: int, j: int) -> int:
        return (i % self.p) * self.q + (j % self.q)

    @property
    def ngpus(self) -> int:
        return self.p * self.q

    def fill_spd(self, seed: int) -> None:
        """Metric SPD matrix (SURVEY §8(d) generator), generated on the owners."""
        check(_abi.stf_fill_spd_tiles(self.n, self.nb, ctypes.byref(self.desc), self.ngpus, seed),
              "stf_fill_spd_tiles")

    def load_dense(self, A) -> None:
        """Copy the lower tiles of a dense (n, n) torch/numpy matrix in."""
        import torch

        A = torch.as_tensor(A, dtype=torch.float64)
        nb = self.nb
        for (i, j), t in self.tiles.items():
            blk = A[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb]
            t.copy_(blk.T.to(t.device))  # row-major storage of the transpose == column-major blk

    def to_dense(self, lower_only: bool = True):
        """(n, n) CPU float64 torch tensor of the lower tiles (zeros above if lower_only)."""
        import torch

        nb = self.nb
        out = torch.zeros((self.n, self.n), dtype=torch.float64)
        for (i, j), t in self.tiles.items():
            out[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb] = t.T.cpu()
        return torch.tril(out) if lower_only else out

    def potrf(self) -> int:
        """stf_potrf on this descriptor; returns LAPACK info (>= 0)."""
        return check(_abi.stf_potrf(self.n, self.nb, b"L", ctypes.byref(self.desc), self.ngpus), "stf_potrf")


class MpTiledMatrix:
    """Multi-process mode (one process per GPU): this process's share of a
    p x q block-cyclic TILED_2DBC matrix -- only the tiles it owns, in one
    allocation on `device`.  Usage (see include/stf_cholesky.h):

        mp_init(rank, world, device)
        A = MpTiledMatrix(n, nb, p, q, rank, device); A.fill_spd(seed)
        blob = A.prepare(); A.import_blobs(all_gather(blob)); barrier()
        info = A.potrf(); barrier()

    The blob exchange and barriers are the caller's (torch.distributed).
    """

    def __init__(self, n: int, nb: int, p: int, q: int, rank: int, device: int):
        import torch

        assert n % nb == 0 and 0 <= rank < p * q
        self.n, self.nb, self.p, self.q, self.rank, self.device = n, nb, p, q, rank, device
        self.T = T = n // nb
        own = [(i, j) for j in range(T) for i in range(j, T) if self.owner(i, j) == rank]
        self.slab = torch.empty((max(1, len(own)), nb, nb), dtype=torch.float64, device="cuda:%d" % device)
        self.tiles = {ij: self.slab[k] for k, ij in enumerate(own)}
        self._table = (ctypes.c_void_p * (T * T))()
        for (i, j), t in self.tiles.items():
            self._table[i + j * T] = t.data_ptr()
        self.desc = stf_matrix_desc(STF_DESC_TILED_2DBC, device, 0, None, p, q,
                                    ctypes.cast(self._table, ctypes.POINTER(ctypes.c_void_p)))

    def owner(self, i: int, j: int) -> int:
        return (i % self.p) * self.q + (j % self.q)

    def fill_spd(self, seed: int) -> None:
        check(_abi.stf_fill_spd_tiles(self.n, self.nb, ctypes.byref(self.desc), self.p * self.q, seed),
              "stf_fill_spd_tiles")

    def prepare(self) -> bytes:
        """Build this process's plan and return its IPC blob (stf_mp_prepare)."""
        buf = ctypes.create_string_buffer(int(_abi.stf_mp_blob_size()))
        check(_abi.stf_mp_prepare(self.n, self.nb, ctypes.byref(self.desc), buf), "stf_mp_prepare")
        return buf.raw

    def import_blobs(self, blobs: Sequence[bytes]) -> None:
        """stf_mp_import with every process's blob, in rank order."""
        joined = b"".join(blobs)
        assert len(joined) == len(blobs) * int(_abi.stf_mp_blob_size())
        buf = ctypes.create_string_buffer(joined, len(joined))
        check(_abi.stf_mp_import(buf), "stf_mp_import")

    def potrf(self) -> int:
        """stf_mp_potrf: runs this process's tasks; LAPACK info of its columns."""
        return check(_abi.stf_mp_potrf(), "stf_mp_potrf")


def mp_init(rank: int, world: int, device: int) -> None:
    check(_abi.stf_mp_init(rank, world, device), "stf_mp_init")


def potrf_colmajor(ptr: int, n: int, ld: int, nb: int, uplo: str = "L", device: Optional[int] = None,
                   ngpus: int = 1) -> int:
    """stf_potrf on a caller column-major matrix (device ordinal -> DEVICE_COLMAJOR,
    None -> HOST_COLMAJOR)."""
    kind = STF_DESC_HOST_COLMAJOR if device is None else STF_DESC_DEVICE_COLMAJOR
    d = stf_matrix_desc(kind, device or 0, ld, ctypes.c_void_p(ptr), 0, 0, None)
    return check(_abi.stf_potrf(n, nb, uplo.encode(), ctypes.byref(d), ngpus), "stf_potrf")


def potrf(A, nb: int, ngpus: int = 1) -> int:
    """Factor a square FP64 matrix in place: lower triangle (row-major sense) <- L.

    A: torch tensor (CUDA -> DEVICE_COLMAJOR, CPU -> HOST_COLMAJOR) or numpy
    array.  A C-contiguous (row-major) matrix is a column-major A^T, so it is
    passed with uplo='U' (lower of A == upper of A^T); a Fortran-ordered one
    with uplo='L'.
    """
    import numpy as np

    try:
        import torch
    except ImportError:  # pragma: no cover
        torch = None
    if torch is not None and isinstance(A, torch.Tensor):
        assert A.dtype == torch.float64 and A.dim() == 2 and A.shape[0] == A.shape[1]
        n = A.shape[0]
        if A.stride() == (1, n):
            uplo = "L"
        elif A.is_contiguous():
            uplo = "U"
        else:
            raise ValueError("A must be row- or column-contiguous")
        dev = A.device.index if A.is_cuda else None
        return potrf_colmajor(A.data_ptr(), n, max(1, n), nb, uplo, dev, ngpus)
    A = np.asarray(A)
    assert A.dtype == np.float64 and A.ndim == 2 and A.shape[0] == A.shape[1]
    n = A.shape[0]
    if A.flags.f_contiguous:
        uplo = "L"
    elif A.flags.c_contiguous:
        uplo = "U"
    else:
        raise ValueError("A must be contiguous")
    return potrf_colmajor(A.ctypes.data, n, max(1, n), nb, uplo, None, ngpus)
