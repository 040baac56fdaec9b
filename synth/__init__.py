"""Seeded synthetic inputs shared by the oracle, the tests and bench.py.

This module holds NO arithmetic of the method (no factorization, no update,
no solve): only counter-based random numbers and the closed-form test
matrices of SURVEY.md §8(c)/(d).  Both the CPU side (this file, numpy) and the
CUDA library (``fill_spd_kernel`` in ``csrc/kernels/panel.cu``) implement the same counter-based
SplitMix64 spec, and a GPU test asserts the two produce identical bits.

Generator spec ("Generator"):
    splitmix64(x): x += 0x9E3779B97F4A7C15; z = (x ^ x>>30) * 0xBF58476D1CE4E5B9;
                   z = (z ^ z>>27) * 0x94D049BB133111EB; return z ^ z>>31   (mod 2^64)
    for i >= j (0-based global):  h = splitmix64(((i<<32) | j) ^ splitmix64(seed))
                                  u = (h >> 11) * 2^-53;  a = 2u - 1   (exact)
    A_ij = A_ji = a (i != j);     A_ii = a + n   (one IEEE add)
Strictly diagonally dominant and symmetric, hence SPD (Gershgorin) -- the
"seeded, diagonally dominant SPD" inputs BASELINE.json's configs name.
"""
from .spd import (  # noqa: F401
    splitmix64,
    spd_block,
    spd_matrix,
    min_matrix,
    diag_matrix,
    kms_matrix,
    dyadic_unit_lower,
    dyadic_spd,
    METRIC_SEED,
)
