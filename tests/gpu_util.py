"""Helpers shared by the GPU tests: column-major device arrays, error bounds."""
import numpy as np

EPS = np.finfo(np.float64).eps


def to_dev(A, ld=None):
    """numpy (rows, cols) -> torch CUDA tensor whose storage is column-major A
    with leading dimension ld (tensor shape (cols, ld))."""
    import torch

    A = np.asarray(A, dtype=np.float64)
    rows, cols = A.shape
    ld = ld or rows
    buf = np.zeros((cols, ld))
    buf[:, :rows] = A.T
    return torch.from_numpy(buf).cuda()


def from_dev(t, rows):
    return t.cpu().numpy()[:, :rows].T.copy()


def relF(X, Y):
    return float(np.linalg.norm(X - Y) / np.linalg.norm(Y))


def backward_ratio(A, L):
    n = A.shape[0]
    Asym = np.tril(A) + np.tril(A, -1).T
    return float(np.linalg.norm(Asym - L @ L.T) / (np.linalg.norm(Asym) * n * EPS))
