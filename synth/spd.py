"""Counter-based seeded SPD inputs and closed-form test matrices
(SURVEY.md §8(c) pins P1, P2, P3, P6).  No factorization arithmetic lives here.

All matrices are returned as float64 numpy arrays in column-major (Fortran)
order, the layout LAPACK and the C ABI's COLMAJOR descriptors use.
"""
from __future__ import annotations

import math

import numpy as np

METRIC_SEED = 1  # seed of the metric inputs

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_C0 = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)


def splitmix64(x):
    """SplitMix64 finaliser, vectorised over uint64 arrays (wraps mod 2^64)."""
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x = x + _C0
        z = (x ^ (x >> np.uint64(30))) * _C1
        z = (z ^ (z >> np.uint64(27))) * _C2
        return z ^ (z >> np.uint64(31))


def _uniform_pm1(seed: int, i: np.ndarray, j: np.ndarray) -> np.ndarray:
    """a(i, j) = 2u - 1 for the key (max(i,j), min(i,j)); exact in float64."""
    hi = np.maximum(i, j).astype(np.uint64)
    lo = np.minimum(i, j).astype(np.uint64)
    s = splitmix64(np.uint64(seed))
    h = splitmix64(((hi << np.uint64(32)) | lo) ^ s)
    u = (h >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)
    return 2.0 * u - 1.0


def spd_block(seed: int, n: int, r0: int, c0: int, rows: int, cols: int) -> np.ndarray:
    """Rows r0..r0+rows-1, columns c0..c0+cols-1 of the n x n metric matrix."""
    i = np.arange(r0, r0 + rows, dtype=np.int64)[:, None]
    j = np.arange(c0, c0 + cols, dtype=np.int64)[None, :]
    i, j = np.broadcast_arrays(i, j)
    a = _uniform_pm1(seed, i, j)
    diag = i == j
    a[diag] = a[diag] + float(n)
    return np.asfortranarray(a)


def spd_matrix(seed: int, n: int) -> np.ndarray:
    """Full symmetric n x n metric matrix (column-major)."""
    return spd_block(seed, n, 0, 0, n, n)


def min_matrix(n: int) -> np.ndarray:
    """P1: A_ij = min(i, j) (1-based); its Cholesky factor is tril(ones)."""
    i = np.arange(1, n + 1, dtype=np.float64)
    return np.asfortranarray(np.minimum(i[:, None], i[None, :]))


def diag_matrix(seed: int, n: int) -> np.ndarray:
    """P3: diagonal matrix with entries in [1, 3)."""
    idx = np.arange(n, dtype=np.int64)
    d = 2.0 + _uniform_pm1(seed, idx, idx)
    return np.asfortranarray(np.diag(d))


def kms_matrix(n: int, rho: float) -> np.ndarray:
    """P6: Kac-Murdock-Szego matrix A_ij = rho^|i-j|."""
    i = np.arange(n)
    return np.asfortranarray(rho ** np.abs(i[:, None] - i[None, :]).astype(np.float64))


def dyadic_unit_lower(seed: int, n: int, m: int = 25) -> np.ndarray:
    """P2: unit lower-triangular L0 whose strictly-lower entries are k * 2^-m with
    |k| < 2^p, p = m - ceil(log2 n)  (m = 25)."""
    p = m - max(1, math.ceil(math.log2(max(n, 2))))
    assert p >= 1, "n too large for this m"
    i = np.arange(n, dtype=np.int64)[:, None]
    j = np.arange(n, dtype=np.int64)[None, :]
    i, j = np.broadcast_arrays(i, j)
    s = splitmix64(np.uint64(seed))
    h = splitmix64(((i.astype(np.uint64) << np.uint64(32)) | j.astype(np.uint64)) ^ s)
    span = np.uint64((1 << (p + 1)) - 1)
    k = (h >> np.uint64(11)) % span
    kf = k.astype(np.float64) - float((1 << p) - 1)
    L0 = np.where(i > j, kf * (2.0 ** -m), 0.0)
    L0[np.arange(n), np.arange(n)] = 1.0
    return np.asfortranarray(L0)


def dyadic_spd(seed: int, n: int, m: int = 25):
    """(A, L0) with A = L0 @ L0.T, exact in float64 under any summation order."""
    L0 = dyadic_unit_lower(seed, n, m)
    A = np.asfortranarray(L0 @ L0.T)
    return A, L0


# ---------------------------------------------------------------- torch (device) form
def _t_splitmix64(x):
    """splitmix64 on int64 torch tensors (two's complement wraps like uint64;
    logical right shifts emulated with a mask)."""
    import torch

    def shr(v, k):
        return (v >> k) & ((1 << (64 - k)) - 1)

    def c(u):  # uint64 constant as the int64 with the same bits
        return u - (1 << 64) if u >= (1 << 63) else u

    x = x + c(0x9E3779B97F4A7C15)
    z = (x ^ shr(x, 30)) * c(0xBF58476D1CE4E5B9)
    z = (z ^ shr(z, 27)) * c(0x94D049BB133111EB)
    return z ^ shr(z, 31)


def dyadic_unit_lower_block_torch(seed: int, n: int, r0: int, c0: int, rows: int, cols: int, m: int = 25,
                                  device="cuda"):
    """Rows r0.., columns c0.. of dyadic_unit_lower(seed, n, m) as a torch float64
    tensor (row-major (rows, cols)) on `device`; bit-identical to the numpy form
    (tests/test_synth.py).  For the full-size P2 pins (n up to 65536), generated
    block by block on the GPU."""
    import torch

    p = m - max(1, math.ceil(math.log2(max(n, 2))))
    assert p >= 1, "n too large for this m"
    i = torch.arange(r0, r0 + rows, dtype=torch.int64, device=device)[:, None]
    j = torch.arange(c0, c0 + cols, dtype=torch.int64, device=device)[None, :]
    s = int(splitmix64(np.uint64(seed)))
    s = s - (1 << 64) if s >= (1 << 63) else s
    h = _t_splitmix64(((i << 32) | j) ^ s)
    span = (1 << (p + 1)) - 1
    k = ((h >> 11) & ((1 << 53) - 1)) % span
    kf = k.to(torch.float64) - float((1 << p) - 1)
    L0 = torch.where(i > j, kf * (2.0 ** -m), torch.zeros((), dtype=torch.float64, device=device))
    L0 = torch.where(i == j, torch.ones((), dtype=torch.float64, device=device), L0)
    return L0
