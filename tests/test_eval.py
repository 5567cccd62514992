"""Generic eval over index domains: the paper's own example
kernels run through hpl_eval, checked against oracle/eval_f1.py (plain
definitions of Figs. 2-4 in the paper's order and roundings) and the paper's
Fig. 2 statement about local ids.  The oracle itself is pinned here on CPU:
Fig. 2's printed ids, exact rational arithmetic with correct rounding for
saxpy and for dotp's float32 chain.
"""
import ctypes
import random
from fractions import Fraction

import numpy as np
import pytest

from oracle import eval_f1


@pytest.fixture(scope="module")
def hpl():
    from paper_conf_ipps_bozkusf12_b200 import build
    build.build()
    from paper_conf_ipps_bozkusf12_b200 import hpl as h
    return h


# ------------------------------------------------------------------- CPU
def test_registry(hpl):
    k = hpl.hpl_kernels()
    assert set(k) >= {"domain_ids", "saxpy", "dotp"}
    assert k["saxpy"] == "y:F64:rw,x:F64:r,a:f64"


def test_bad_calls_rejected_without_gpu(hpl):
    for name, args in [("no_such_kernel", []), ("saxpy", [1.0]), ("saxpy", [1.0, 2.0, 3.0]),
                       ("dotp", [("array", None), ("array", None), ("array", None)])]:
        with pytest.raises(hpl.HPLError) as e:
            hpl.hpl_eval(name, args)
        assert e.value.code == hpl.HPL_EINVAL


# ------------------------------------------------------- oracle pins (CPU)
def _rn32(fr: Fraction) -> np.float32:
    """Correctly rounded float32 of an exact rational (ties to even)."""
    f = np.float32(float(fr))
    cands = [f, np.nextafter(f, np.float32(np.inf)), np.nextafter(f, np.float32(-np.inf))]
    best = min(cands, key=lambda c: (abs(Fraction(float(c)) - fr), int(np.float32(c).view(np.int32)) & 1))
    return np.float32(best)


def test_oracle_fig2_ids_as_printed():
    """global 4x8, local 2x4 — the points (1,2), (1,6), (3,2)
    and (3,6) all have local id (1,2); ids partition the domain."""
    ids = eval_f1.domain_ids([4, 8], [2, 4])
    assert ids.shape == (32, 9)
    for (x, y) in [(1, 2), (1, 6), (3, 2), (3, 6)]:
        assert tuple(ids[y * 4 + x, 3:5]) == (1, 2)
    assert np.array_equal(ids[:, 0:3], ids[:, 6:9] * np.array([2, 4, 1]) + ids[:, 3:6])
    assert len({tuple(r[0:3]) for r in ids}) == 32
    assert set(map(tuple, ids[:, 6:8])) == {(gx, gy) for gx in range(2) for gy in range(2)}


def test_oracle_saxpy_two_roundings():
    """y = RN(RN(a x) + y) by exact rationals + correct rounding (float()),
    including inputs where an fma would give a different double."""
    rng = random.Random(5)
    xs = [rng.uniform(-1e3, 1e3) for _ in range(500)] + [1.0 + 2.0 ** -30]
    ys = [rng.uniform(-1e3, 1e3) for _ in range(500)] + [-(1.0 + 2.0 ** -29)]
    a = 1.0 + 2.0 ** -30
    got = eval_f1.saxpy(ys, xs, a)
    for g, x, y in zip(got, xs, ys):
        want = float(Fraction(float(Fraction(a) * Fraction(x))) + Fraction(y))
        assert float(g) == want
    # the constructed last element: an fma keeps a*x's low bits, two roundings lose them
    fused = float(Fraction(a) * Fraction(xs[-1]) + Fraction(ys[-1]))
    assert float(got[-1]) != fused


@pytest.mark.parametrize("M", [1, 4, 32])
def test_oracle_dotp_float32_chain(M):
    """Fig. 4: each partial is lane 0's in-order float32 sum of float32
    products — checked against exact rationals rounded to float32 at every
    step, and against a float64 dot product."""
    rng = np.random.default_rng(M)
    N = 8 * M
    v1 = rng.standard_normal(N).astype(np.float32)
    v2 = rng.standard_normal(N).astype(np.float32)
    got = eval_f1.dotp(v1, v2, M)
    for g in range(N // M):
        acc = np.float32(0.0)
        for i in range(M):
            prod = _rn32(Fraction(float(v1[g * M + i])) * Fraction(float(v2[g * M + i])))
            acc = _rn32(Fraction(float(acc)) + Fraction(float(prod)))
        assert got[g] == acc
    assert abs(float(got.astype(np.float64).sum()) - float(np.dot(v1.astype(np.float64), v2.astype(np.float64)))) \
        < 1e-5 * N


# ------------------------------------------------------------------- GPU
@pytest.fixture(scope="module")
def gpu(hpl):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    hpl.hpl_set_device(0)
    return hpl


def _host(hpl, a, dtype, n):
    p = hpl.hpl_array_data(a, hpl.HPL_HOST)
    return np.ctypeslib.as_array((ctypes.c_byte * (n * np.dtype(dtype).itemsize)).from_address(p)).view(dtype)


@pytest.mark.gpu
def test_fig2_domain_ids(gpu):
    """Fig. 2: global 4x8, local 2x4; threads
    (1,2), (1,6), (3,2), (3,6) all have local id (1,2)."""
    hpl = gpu
    gx, gy, lx, ly = 4, 8, 2, 4
    a = hpl.hpl_array_alloc(hpl.HPL_I32, [gx * gy * 9])
    try:
        hpl.hpl_eval("domain_ids", [a], global_=[gx, gy], local=[lx, ly])
        hpl.hpl_array_sync(a, hpl.HPL_HOST, hpl.HPL_READ)
        ids = _host(hpl, a, np.int32, gx * gy * 9).reshape(gy, gx, 9)
        assert np.array_equal(ids.reshape(-1, 9), eval_f1.domain_ids([gx, gy], [lx, ly]))
        for (x, y) in [(1, 2), (1, 6), (3, 2), (3, 6)]:
            assert tuple(ids[y, x, 3:5]) == (1, 2)
    finally:
        hpl.hpl_array_free(a)


@pytest.mark.gpu
@pytest.mark.parametrize("dims", [[1000], [96, 7], [6, 10, 4], [1 << 20]])
def test_default_local_covers_domain_once(gpu, dims):
    """Library-chosen local domain: every point exactly once,
    ids consistent (g = group * local + lid)."""
    hpl = gpu
    n = int(np.prod(dims))
    a = hpl.hpl_array_alloc(hpl.HPL_I32, [n * 9])
    try:
        hpl.hpl_eval("domain_ids", [a], global_=dims)
        hpl.hpl_array_sync(a, hpl.HPL_HOST, hpl.HPL_READ)
        ids = _host(hpl, a, np.int32, n * 9).reshape(n, 9)
        d3 = list(dims) + [1] * (3 - len(dims))
        gidx = ids[:, 0] + d3[0] * (ids[:, 1] + d3[1] * ids[:, 2])
        assert np.array_equal(gidx, np.arange(n))
        loc = ids[:, 3:6].max(axis=0) + 1
        assert np.array_equal(ids[:, 0:3], ids[:, 6:9] * loc + ids[:, 3:6])
        assert all(d % l == 0 for d, l in zip(d3, loc))
    finally:
        hpl.hpl_array_free(a)


@pytest.mark.gpu
def test_fig3_saxpy(gpu):
    """Fig. 3: y user-owned storage, x library-owned, default
    global domain = dims of y; y[idx] = a*x[idx] + y[idx] (two roundings)."""
    hpl = gpu
    rng = np.random.default_rng(3)
    n = 1000
    myvector = rng.standard_normal(n)
    y0 = myvector.copy()
    x = hpl.hpl_array_alloc(hpl.HPL_F64, [n])
    y = hpl.hpl_array_alloc(hpl.HPL_F64, [n], myvector.ctypes.data)
    try:
        xh = _host(hpl, x, np.float64, n)
        xh[:] = rng.standard_normal(n)
        hpl.hpl_array_sync(x, hpl.HPL_HOST, hpl.HPL_WRITE)  # host copy written
        a = 2.5
        hpl.hpl_eval("saxpy", [y, x, a])
        assert hpl.hpl_array_info(y)["valid"] == hpl.HPL_DEVICE
        assert np.array_equal(myvector, y0)  # host copy untouched until synced
        hpl.hpl_array_sync(y, hpl.HPL_HOST, hpl.HPL_READ)
        assert np.array_equal(myvector, eval_f1.saxpy(y0, xh, a))
        # a second eval reuses the still-valid device copy of x: a host edit
        # not announced with a WRITE sync is (by contract) not uploaded
        x_old, y1 = xh.copy(), myvector.copy()
        xh[:] = 0.0
        hpl.hpl_eval("saxpy", [y, x, a])
        hpl.hpl_array_sync(y, hpl.HPL_HOST, hpl.HPL_READ)
        assert np.array_equal(myvector, eval_f1.saxpy(y1, x_old, a))
        # announcing the edit makes the next eval upload it
        hpl.hpl_array_sync(x, hpl.HPL_HOST, hpl.HPL_WRITE)
        y2 = myvector.copy()
        hpl.hpl_eval("saxpy", [y, x, a])
        hpl.hpl_array_sync(y, hpl.HPL_HOST, hpl.HPL_READ)
        assert np.array_equal(myvector, y2)
    finally:
        hpl.hpl_array_free(x)
        hpl.hpl_array_free(y)


@pytest.mark.gpu
@pytest.mark.parametrize("N,M", [(256, 32), (4096, 128), (1 << 20, 256), (3 * 1024, 1024), (13 * 64, 64), (8, 1)])
def test_fig4_dotp(gpu, N, M):
    """Fig. 4: per-group partial dot products through Local
    memory, lane 0 sums in order into pSums[gidx]; host sums nGroup partials."""
    hpl = gpu
    rng = np.random.default_rng(N)
    ng = N // M
    v1 = hpl.hpl_array_alloc(hpl.HPL_F32, [N])
    v2 = hpl.hpl_array_alloc(hpl.HPL_F32, [N])
    ps = hpl.hpl_array_alloc(hpl.HPL_F32, [ng])
    try:
        a1, a2, p = _host(hpl, v1, np.float32, N), _host(hpl, v2, np.float32, N), _host(hpl, ps, np.float32, ng)
        a1[:] = rng.standard_normal(N).astype(np.float32)
        a2[:] = rng.standard_normal(N).astype(np.float32)
        p[:] = 0
        for h in (v1, v2, ps):
            hpl.hpl_array_sync(h, hpl.HPL_HOST, hpl.HPL_WRITE)
        hpl.hpl_eval("dotp", [v1, v2, ps], global_=[N], local=[M])
        hpl.hpl_array_sync(ps, hpl.HPL_HOST, hpl.HPL_READ)
        assert np.array_equal(p, eval_f1.dotp(a1, a2, M))
        dot = float(np.sum(p.astype(np.float64)))
        assert abs(dot - float(np.dot(a1.astype(np.float64), a2.astype(np.float64)))) < 1e-3 * N ** 0.5
    finally:
        for h in (v1, v2, ps):
            hpl.hpl_array_free(h)


@pytest.mark.gpu
def test_eval_domain_errors(gpu):
    hpl = gpu
    a = hpl.hpl_array_alloc(hpl.HPL_I32, [4 * 8 * 9])
    b = hpl.hpl_array_alloc(hpl.HPL_F32, [16])
    try:
        for g, l in [([4, 8], [3, 4]), ([4, 8], [2, 5]), ([4, 8, 1, 1], None), ([8, 8], [2, 4])]:
            with pytest.raises(hpl.HPLError) as e:
                hpl.hpl_eval("domain_ids", [a], global_=g, local=l)
            assert e.value.code == hpl.HPL_EINVAL
        with pytest.raises(hpl.HPLError):  # wrong dtype for saxpy
            hpl.hpl_eval("saxpy", [b, b, 1.0])
    finally:
        hpl.hpl_array_free(a)
        hpl.hpl_array_free(b)


@pytest.mark.gpu
@pytest.mark.parametrize("dims", [[1], [7], [1001], [33, 31], [(1 << 20) + 3]])
def test_saxpy_sizes(gpu, dims):
    """Any domain size / rank: y = RN(RN(a x) + y) element by element (the
    library may run several consecutive points per CUDA thread)."""
    hpl = gpu
    n = int(np.prod(dims))
    rng = np.random.default_rng(n)
    x = hpl.hpl_array_alloc(hpl.HPL_F64, dims)
    y = hpl.hpl_array_alloc(hpl.HPL_F64, dims)
    try:
        xh, yh = _host(hpl, x, np.float64, n), _host(hpl, y, np.float64, n)
        xh[:] = rng.standard_normal(n)
        yh[:] = rng.standard_normal(n)
        y0 = yh.copy()
        for h in (x, y):
            hpl.hpl_array_sync(h, hpl.HPL_HOST, hpl.HPL_WRITE)
        hpl.hpl_eval("saxpy", [y, x, -0.75])
        hpl.hpl_array_sync(y, hpl.HPL_HOST, hpl.HPL_READ)
        assert np.array_equal(yh, eval_f1.saxpy(y0, xh, -0.75))
    finally:
        hpl.hpl_array_free(x)
        hpl.hpl_array_free(y)
