"""Reduction oracle — TEST INFRASTRUCTURE, NOT PRODUCT CODE.

The paper's fifth benchmark adds 16M single-precision values (PAPER.md:951-952,
SHOC).  Its plain definition is the exact sum; the oracle
returns that sum correctly rounded to double with math.fsum (a library
primitive: Shewchuk's exact summation).  Pinned in tests/test_reduce.py
against exact rational (fractions.Fraction) sums.
"""
import math

import numpy as np


def sum_exact(x) -> float:
    """Correctly rounded double of the exact sum of the (float32) values."""
    return math.fsum(np.asarray(x, dtype=np.float64).tolist())


def abs_sum(x) -> float:
    return math.fsum(np.abs(np.asarray(x, dtype=np.float64)).tolist())
