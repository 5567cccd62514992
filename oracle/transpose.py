"""Matrix-transpose oracle — TEST INFRASTRUCTURE, NOT PRODUCT CODE.

The paper's transpose (Fig. 10(b), PAPER.md:1132-1138:
``dest[idy][idx] = src[idx][idy]``; the benchmark transposes a 16K x 16K
matrix).  Plain definition: for src of shape (h, w),
dst has shape (w, h) and dst[j][i] = src[i][j].  ``transpose`` uses numpy's
transpose (a library primitive) made contiguous; ``transpose_loops`` is the
definition written out element by element for small inputs.  Pinned in
tests/test_transpose.py (loops vs primitive, involution, a hand-written
example).
"""
import numpy as np


def transpose(src) -> np.ndarray:
    """dst (w x h, row-major) with dst[j, i] = src[i, j]."""
    src = np.asarray(src)
    assert src.ndim == 2
    return np.ascontiguousarray(src.T)


def transpose_loops(src) -> np.ndarray:
    """The same, element by element (Fig. 10(b) as written); small inputs only."""
    src = np.asarray(src)
    h, w = src.shape
    dst = np.empty((w, h), dtype=src.dtype)
    for idx in range(h):
        for idy in range(w):
            dst[idy][idx] = src[idx][idy]
    return dst
