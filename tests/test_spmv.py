"""F4: CSR spmv, the paper's Fig. 5 kernel, through
hpl_eval("spmv_csr"), bit-exact against the oracle that follows Fig. 5(b)'s
order (oracle/spmv.py), on seeded synthetic matrices of the paper's shapes
(Fig. 5 toy: 1024 rows, NZ 128, M 8; Fig. 7: 16K x 16K, 1 % nonzeros)."""
import ctypes

import numpy as np
import pytest

from ep_workloads import SPMV_DENSITY, SPMV_ROWS, make_csr
from oracle import spmv as osp


# ------------------------------------------------------------ oracle pins
@pytest.mark.parametrize("M", [2, 8, 32])
def test_oracles_agree_with_float64(M):
    rowptr, cols, A = make_csr(300, 500, 0.05, seed=M)
    vec = np.random.default_rng(1).uniform(-1, 1, 500).astype(np.float32)
    ref = np.array([np.dot(A[rowptr[i]:rowptr[i + 1]].astype(np.float64),
                           vec[cols[rowptr[i]:rowptr[i + 1]]].astype(np.float64)) for i in range(300)])
    absd = np.array([np.dot(np.abs(A[rowptr[i]:rowptr[i + 1]]).astype(np.float64),
                            np.abs(vec[cols[rowptr[i]:rowptr[i + 1]]]).astype(np.float64)) for i in range(300)])
    n = np.diff(rowptr).max()
    bound = (n + 2) * 2.0 ** -24 * absd + 1e-30
    for out in (osp.seq_fig5a(rowptr, cols, A, vec), osp.hpl_fig5b(rowptr, cols, A, vec, M)):
        assert np.all(np.abs(out.astype(np.float64) - ref) <= bound)


def test_fig5b_equals_sequential_when_rows_are_short():
    """Rows with <= 1 element per lane and M = 2: both orders coincide."""
    rowptr = np.array([0, 0, 1, 3], dtype=np.int32)
    cols = np.array([2, 0, 1], dtype=np.int32)
    A = np.array([0.5, 1.5, -2.0], dtype=np.float32)
    vec = np.array([1.0, 2.0, 4.0], dtype=np.float32)
    assert np.array_equal(osp.hpl_fig5b(rowptr, cols, A, vec, 2), osp.seq_fig5a(rowptr, cols, A, vec))
    assert np.array_equal(osp.seq_fig5a(rowptr, cols, A, vec), np.array([0.0, 2.0, -2.5], dtype=np.float32))


def test_make_csr_shape():
    rowptr, cols, A = make_csr(1000, 2000, 0.01, seed=3)
    assert rowptr[0] == 0 and len(rowptr) == 1001 and rowptr[-1] == len(cols) == len(A)
    for i in range(0, 1000, 97):
        c = cols[rowptr[i]:rowptr[i + 1]]
        assert np.all(np.diff(c) > 0) and (len(c) == 0 or (c.min() >= 0 and c.max() < 2000))


# ------------------------------------------------------------------- GPU
@pytest.fixture(scope="module")
def gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_bozkusf12_b200 import build
    build.build()
    from paper_conf_ipps_bozkusf12_b200 import hpl
    hpl.hpl_set_device(0)
    return hpl


def _arr(hpl, dtype_code, np_arr):
    n = max(len(np_arr), 1)
    a = hpl.hpl_array_alloc(dtype_code, [n])
    p = hpl.hpl_array_data(a, hpl.HPL_HOST)
    ct = ctypes.c_float if np_arr.dtype == np.float32 else ctypes.c_int32
    if len(np_arr):
        np.ctypeslib.as_array((ct * n).from_address(p))[:] = np_arr
    hpl.hpl_array_sync(a, hpl.HPL_HOST, hpl.HPL_WRITE)
    return a


def run_spmv(hpl, rowptr, cols, A, vec, M):
    rows = len(rowptr) - 1
    hs = [_arr(hpl, hpl.HPL_F32, A), _arr(hpl, hpl.HPL_F32, vec), _arr(hpl, hpl.HPL_I32, cols),
          _arr(hpl, hpl.HPL_I32, rowptr), hpl.hpl_array_alloc(hpl.HPL_F32, [rows])]
    try:
        hpl.hpl_eval("spmv_csr", hs, global_=[rows * M], local=[M])
        hpl.hpl_array_sync(hs[4], hpl.HPL_HOST, hpl.HPL_READ)
        p = hpl.hpl_array_data(hs[4], hpl.HPL_HOST)
        return np.ctypeslib.as_array((ctypes.c_float * rows).from_address(p)).copy()
    finally:
        for h in hs:
            hpl.hpl_array_free(h)


@pytest.mark.gpu
@pytest.mark.parametrize("M", [8, 2, 32])
def test_fig5_toy(gpu, M):
    """Fig. 5(b): nRows 1024, NZ 128 (many empty rows), M 8."""
    rng = np.random.default_rng(5)
    rows = 1024
    r = np.sort(rng.choice(rows, 128))          # 128 nonzeros scattered over rows
    counts = np.bincount(r, minlength=rows)
    rowptr = np.zeros(rows + 1, dtype=np.int32)
    np.cumsum(counts, out=rowptr[1:])
    cols = np.concatenate([np.sort(rng.choice(rows, c, replace=False)) for c in counts]).astype(np.int32)
    A = rng.uniform(-1, 1, 128).astype(np.float32)
    vec = rng.uniform(-1, 1, rows).astype(np.float32)
    got = run_spmv(gpu, rowptr, cols, A, vec, M)
    assert np.array_equal(got, osp.hpl_fig5b(rowptr, cols, A, vec, M))


@pytest.mark.gpu
@pytest.mark.parametrize("M", [8, 32, 2])
def test_fig7_size(gpu, M):
    """Fig. 7's spmv: 16K x 16K, 1 % nonzeros."""
    rowptr, cols, A = make_csr(SPMV_ROWS, SPMV_ROWS, SPMV_DENSITY, seed=16)
    vec = np.random.default_rng(17).uniform(-1, 1, SPMV_ROWS).astype(np.float32)
    got = run_spmv(gpu, rowptr, cols, A, vec, M)
    assert np.array_equal(got, osp.hpl_fig5b(rowptr, cols, A, vec, M))


@pytest.mark.gpu
@pytest.mark.parametrize("M", [4, 32])
def test_vec_too_large_for_shared_memory(gpu, M):
    """A wide matrix (80K columns, 320 KB vec, sparse rows: many CTAs whose
    element ranges are shorter than the 16-byte alignment window)."""
    rowptr, cols, A = make_csr(700, 80_000, 0.002, seed=M + 40)
    vec = np.random.default_rng(M).uniform(-1, 1, 80_000).astype(np.float32)
    got = run_spmv(gpu, rowptr, cols, A, vec, M)
    assert np.array_equal(got, osp.hpl_fig5b(rowptr, cols, A, vec, M))


@pytest.mark.gpu
def test_rows_exceed_one_resident_wave(gpu):
    """Many CTAs (150K rows), a ragged last warp (rows * M not a multiple of
    32), empty rows and rows of 1-2 elements (unaligned chunk ends)."""
    rowptr, cols, A = make_csr(150_001, 3000, 0.001, seed=77)
    vec = np.random.default_rng(78).uniform(-1, 1, 3000).astype(np.float32)
    got = run_spmv(gpu, rowptr, cols, A, vec, 4)
    assert np.array_equal(got, osp.hpl_fig5b(rowptr, cols, A, vec, 4))
