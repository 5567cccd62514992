"""Seeded synthetic workloads for NPB EP — shared by tests, bench.py and smoke().

EP has no input arrays: a workload is fully specified by (M, seed, a)
(SURVEY.md §8(d) "Concrete inputs").  This module holds only those constants
and the class table; it contains none of the method's arithmetic, so both the
oracle-side tests and the CUDA-path callers may import it.

Sources: NPB 3.x EP problem classes (the paper's reference [16],
PAPER.md:1322-1323; classes W..C are the x-axis of Fig. 6, PAPER.md:863-871;
class C is the Fig. 7 size); seed and multiplier from NPB ep.f
and BASELINE.json north_star ("a=5^13, seed 271828183").
"""

NPB_SEED = 271828183          # ep.f  s = 271828183.d0
NPB_A = 1220703125            # ep.f  a = 5^13 = 1220703125.d0
NQ = 10                       # ep.f  nq = 10 annuli
NPB_EPS = 1e-8                # ep.f  epsilon = 1.d-8 (verification tolerance)

# NPB class -> M (2^M pairs, 2^(M+1) uniforms)
CLASSES = {"S": 24, "W": 25, "A": 28, "B": 30, "C": 32, "D": 36, "E": 40}

# BASELINE.json configs: which classes run at which GPU counts
CONFIGS = {
    "S": (1,), "W": (1,), "A": (1,),
    "B": (1, 2, 4, 8), "C": (1, 2, 4, 8), "D": (1, 2, 4, 8),
}
HEADLINE_CLASS = "D"          # BASELINE.json: "class D (M=36) ... FP64-roofline headline"

# robustness seeds for tests only: odd, extreme, all with a = 5^13
ROBUST_SEEDS = (1, (1 << 46) - 1, 0x2B992DDFA23, 5 ** 19 % (1 << 46))


def uniforms(M: int) -> int:
    """Number of uniforms a class-M run draws, the unit of the Mops metric."""
    return 2 << M


def pairs(M: int) -> int:
    return 1 << M


# ---------------------------------------------------------------- F4: spmv
# Fig. 7's spmv size: "a 16K x 16K matrix with a 1% of non zeros"
# (PAPER.md:950-951); Fig. 5's toy: nRows 1024, M = 8.
SPMV_ROWS = 16 * 1024
SPMV_DENSITY = 0.01


def make_csr(n_rows, n_cols, density, seed):
    """Seeded synthetic CSR matrix (numpy): each row gets Binomial(n_cols,
    density) distinct uniformly random sorted columns, values U(-1, 1) float32.
    Returns rowptr (int32, n_rows+1), cols (int32), A (float32)."""
    import numpy as np
    rng = np.random.default_rng(seed)
    counts = rng.binomial(n_cols, density, n_rows)
    rowptr = np.zeros(n_rows + 1, dtype=np.int64)
    np.cumsum(counts, out=rowptr[1:])
    cols = np.empty(int(rowptr[-1]), dtype=np.int32)
    for i in range(n_rows):
        cols[rowptr[i]:rowptr[i + 1]] = np.sort(rng.choice(n_cols, counts[i], replace=False))
    A = rng.uniform(-1.0, 1.0, int(rowptr[-1])).astype(np.float32)
    return rowptr.astype(np.int32), cols, A


# ----------------------------------------------------------- F4: transpose
# Fig. 7's transpose size: "the transposition of a 16K x 16K matrix"
# (PAPER.md:949-950), single precision like the AMD SDK kernel it was taken
# from; Fig. 9's smaller device used 5K x 5K
# (PAPER.md:1087-1088).
TRANSPOSE_N = 16 * 1024
TRANSPOSE_SMALL_N = 5 * 1024


def make_matrix(h, w, seed):
    """Seeded synthetic float32 h x w matrix (row-major), values U(-1, 1);
    distinct values almost surely, so a misplaced element is detected."""
    import numpy as np
    return np.random.default_rng(seed).uniform(-1.0, 1.0, (h, w)).astype(np.float32)
