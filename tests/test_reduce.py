"""F2: the 16M-float reduction benchmark
through hpl_reduce_sum_f32 / hpl_eval("sum_f32"), vs the exact sum.

Tolerance: FP64 accumulation in a fixed order; each partial sum
carries <= 2^-53 relative error per add over <= ~200 sequential adds per
thread plus a ~20-level tree, so |gpu - exact| <= 1e-13 * sum|x| (+1e-300)."""
import ctypes
import random
from fractions import Fraction

import numpy as np
import pytest

from oracle import reduce as red


# ------------------------------------------------------------ oracle pins
@pytest.mark.parametrize("seed", range(5))
def test_oracle_is_the_exact_sum(seed):
    rng = np.random.default_rng(seed)
    x = (rng.standard_normal(3000) * 10.0 ** rng.integers(-8, 8, 3000)).astype(np.float32)
    exact = sum(Fraction(float(v)) for v in x)
    assert red.sum_exact(x) == float(exact)


def test_oracle_cancellation_cases():
    x = np.array([1e30, 1.0, -1e30, 3.0], dtype=np.float32)
    assert red.sum_exact(x) == 4.0
    assert red.sum_exact(np.array([], dtype=np.float32)) == 0.0


# -------------------------------------------------------------- ABI (CPU)
@pytest.fixture(scope="module")
def hpl():
    from paper_conf_ipps_bozkusf12_b200 import build
    build.build()
    from paper_conf_ipps_bozkusf12_b200 import hpl as h
    return h


def test_reduce_argument_checks(hpl):
    lib = hpl.lib()
    assert lib.hpl_reduce_sum_f32(None, -1, 0x1000, None) == hpl.HPL_EINVAL
    assert lib.hpl_reduce_sum_f32(None, 10, 0x1000, None) == hpl.HPL_EINVAL
    assert lib.hpl_reduce_sum_f32(0x1002, 10, 0x1000, None) == hpl.HPL_EINVAL  # misaligned
    assert lib.hpl_reduce_sum_f32(0x1000, 10, None, None) == hpl.HPL_EINVAL


# ------------------------------------------------------------------- GPU
@pytest.fixture(scope="module")
def gpu(hpl):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.set_device(0)
    hpl.hpl_set_device(0)
    return torch, hpl


def gpu_sum(gpu, x_np, offset=0):
    torch, hpl = gpu
    buf = torch.empty(len(x_np) + offset + 4, dtype=torch.float32, device="cuda")
    t = buf[offset:offset + len(x_np)]
    t.copy_(torch.from_numpy(np.ascontiguousarray(x_np)))
    out = torch.full((1,), -1.0, dtype=torch.float64, device="cuda")
    hpl.hpl_reduce_sum_f32(t.data_ptr(), len(x_np), out.data_ptr(), torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    return float(out.item())


@pytest.mark.gpu
@pytest.mark.parametrize("n", [0, 1, 3, 4, 5, 1000, (1 << 20) + 7, 16 * (1 << 20), (1 << 26) + 3])
@pytest.mark.parametrize("offset", [0, 1, 3])
def test_sum_sizes_and_alignment(gpu, n, offset):
    rng = np.random.default_rng(n + offset)
    x = rng.uniform(-1.0, 1.0, n).astype(np.float32)
    got = gpu_sum(gpu, x, offset)
    assert abs(got - red.sum_exact(x)) <= 1e-13 * red.abs_sum(x) + 1e-300


@pytest.mark.gpu
@pytest.mark.parametrize("dist", ["positive", "normal_wide", "cancel"])
def test_sum_distributions(gpu, dist):
    rng = np.random.default_rng(7)
    n = 16 * (1 << 20)  # the paper's 16M values
    if dist == "positive":
        x = rng.uniform(0.0, 1.0, n).astype(np.float32)
    elif dist == "normal_wide":
        x = (rng.standard_normal(n) * 10.0 ** rng.integers(-6, 6, n)).astype(np.float32)
    else:
        h = rng.standard_normal(n // 2).astype(np.float32)
        x = np.concatenate([h, -h[::-1]])
    got = gpu_sum(gpu, x)
    assert abs(got - red.sum_exact(x)) <= 1e-13 * red.abs_sum(x) + 1e-300


@pytest.mark.gpu
def test_sum_deterministic(gpu):
    x = np.random.default_rng(1).standard_normal(10_000_019).astype(np.float32)
    assert gpu_sum(gpu, x) == gpu_sum(gpu, x)


@pytest.mark.gpu
def test_sum_through_eval(gpu):
    torch, hpl = gpu
    n = 1_000_003
    x = np.random.default_rng(2).standard_normal(n).astype(np.float32)
    a = hpl.hpl_array_alloc(hpl.HPL_F32, [n])
    o = hpl.hpl_array_alloc(hpl.HPL_F64, [1])
    try:
        p = hpl.hpl_array_data(a, hpl.HPL_HOST)
        np.ctypeslib.as_array((ctypes.c_float * n).from_address(p))[:] = x
        hpl.hpl_array_sync(a, hpl.HPL_HOST, hpl.HPL_WRITE)
        hpl.hpl_eval("sum_f32", [a, o])
        assert hpl.hpl_array_info(o)["valid"] == hpl.HPL_DEVICE
        hpl.hpl_array_sync(o, hpl.HPL_HOST, hpl.HPL_READ)
        got = (ctypes.c_double * 1).from_address(hpl.hpl_array_data(o, hpl.HPL_HOST))[0]
        assert abs(got - red.sum_exact(x)) <= 1e-13 * red.abs_sum(x)
    finally:
        hpl.hpl_array_free(a)
        hpl.hpl_array_free(o)
