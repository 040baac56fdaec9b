"""The seeded generators in synth/ (no method arithmetic): the torch form of the
P2 dyadic factor equals the numpy form bit for bit, blocks tile the matrix."""
import numpy as np
import torch

import synth
from synth.spd import dyadic_unit_lower_block_torch


def test_dyadic_torch_block_matches_numpy():
    for n, seed in ((300, 101), (1024, 7)):
        L0 = synth.dyadic_unit_lower(seed, n)
        full = dyadic_unit_lower_block_torch(seed, n, 0, 0, n, n, device="cpu").numpy()
        assert np.array_equal(full, L0)
        blk = dyadic_unit_lower_block_torch(seed, n, 64, 32, 100, 77, device="cpu").numpy()
        assert np.array_equal(blk, L0[64:164, 32:109])


def test_dyadic_product_is_exact_at_full_size_bounds():
    """P2 at n = 65536 (m = 25, p = 9): every entry of A = L0 L0^T is a dyadic
    with <= 50 fractional bits and |A_ij| < 2, so 51 significant bits suffice
    and any summation order is exact in FP64."""
    n, m = 65536, 25
    p = m - 16
    assert p == 9
    max_abs = 1 + n * (2 ** p) ** 2 * 2.0 ** (-2 * m)
    assert max_abs < 2
    assert 1 + 2 * m <= 53
    # the largest magnitude a block of the generator produces stays within 2^p - 1 units
    blk = dyadic_unit_lower_block_torch(101, n, n - 64, 0, 64, 4096, device="cpu")
    off = blk[blk != 1.0]
    assert float(off.abs().max()) <= (2 ** p - 1) * 2.0 ** -m
    assert torch.all(torch.remainder(off * 2 ** m, 1) == 0)
