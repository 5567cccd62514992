"""F4: the paper's matrix transpose (Fig. 10(b), PAPER.md:
1132-1138; benchmark size 16K x 16K) through
hpl_transpose_f32 / hpl_eval("transpose_f32"), bit-exact against the oracle
(oracle/transpose.py) on seeded synthetic float32 matrices: ragged shapes that
span several 64 x 64 tiles plus partial edge tiles, degenerate shapes, the
unaligned (scalar) path, and the full 16K x 16K size (sampled)."""
import ctypes

import numpy as np
import pytest

from ep_workloads import TRANSPOSE_N, make_matrix
from oracle import transpose as otr


# ------------------------------------------------------------ oracle pins
def test_oracle_hand_example():
    """Fig. 10(b): dest[idy][idx] = src[idx][idy], on a 2 x 3 example."""
    src = np.array([[1, 2, 3], [4, 5, 6]], dtype=np.float32)
    want = np.array([[1, 4], [2, 5], [3, 6]], dtype=np.float32)
    assert np.array_equal(otr.transpose(src), want)
    assert np.array_equal(otr.transpose_loops(src), want)


@pytest.mark.parametrize("shape", [(1, 1), (1, 7), (7, 1), (13, 29), (64, 65)])
def test_oracle_loops_equal_primitive(shape):
    src = make_matrix(*shape, seed=sum(shape))
    a, b = otr.transpose(src), otr.transpose_loops(src)
    assert a.shape == (shape[1], shape[0]) and a.flags["C_CONTIGUOUS"]
    assert np.array_equal(a, b)


def test_oracle_involution_and_permutation():
    src = make_matrix(37, 53, seed=9)
    t = otr.transpose(src)
    assert np.array_equal(otr.transpose(t), src)
    assert np.array_equal(np.sort(t, axis=None), np.sort(src, axis=None))  # same multiset


def test_make_matrix_seeded_and_distinct():
    a, b = make_matrix(100, 80, seed=1), make_matrix(100, 80, seed=1)
    assert np.array_equal(a, b) and a.dtype == np.float32
    assert len(np.unique(a)) > 0.99 * a.size


# -------------------------------------------------------------- ABI (CPU)
@pytest.fixture(scope="module")
def hpl():
    from paper_conf_ipps_bozkusf12_b200 import build
    build.build()
    from paper_conf_ipps_bozkusf12_b200 import hpl as h
    return h


def test_transpose_argument_checks(hpl):
    lib = hpl.lib()
    assert lib.hpl_transpose_f32(None, 0, 5, None, None) == hpl.HPL_OK   # empty: no-op
    assert lib.hpl_transpose_f32(None, 5, 0, None, None) == hpl.HPL_OK
    assert lib.hpl_transpose_f32(None, -1, 5, None, None) == hpl.HPL_EINVAL
    assert lib.hpl_transpose_f32(None, 3, 4, 0x2000, None) == hpl.HPL_EINVAL
    assert lib.hpl_transpose_f32(0x1002, 3, 4, 0x9000, None) == hpl.HPL_EINVAL   # misaligned
    assert lib.hpl_transpose_f32(0x1000, 3, 4, 0x1010, None) == hpl.HPL_EINVAL   # overlap
    assert lib.hpl_transpose_f32(0x1000, 1 << 40, 1 << 40, 0x9000, None) == hpl.HPL_EINVAL


def test_transpose_registered_for_eval(hpl):
    assert hpl.hpl_kernels().get("transpose_f32") == "dest:F32:w,src:F32:r"


# ------------------------------------------------------------------- GPU
@pytest.fixture(scope="module")
def gpu(hpl):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.set_device(0)
    hpl.hpl_set_device(0)
    return torch, hpl


def gpu_transpose(gpu, src, offset=0):
    torch, hpl = gpu
    h, w = src.shape
    buf = torch.empty(h * w + offset, dtype=torch.float32, device="cuda")
    x = buf[offset:]
    x.copy_(torch.from_numpy(src.reshape(-1)))
    out = torch.full((w * h,), float("nan"), dtype=torch.float32, device="cuda")
    hpl.hpl_transpose_f32(x.data_ptr(), h, w, out.data_ptr(), torch.cuda.current_stream().cuda_stream)
    return out.cpu().numpy().reshape(w, h)


@pytest.mark.gpu
@pytest.mark.parametrize("shape", [(1, 1), (1, 1000), (1000, 1), (64, 64), (128, 192), (65, 63),
                                   (127, 129), (1000, 37), (37, 1000), (513, 2048), (2048, 3001)])
def test_parity_shapes(gpu, shape):
    src = make_matrix(*shape, seed=shape[0] * 7 + shape[1])
    assert np.array_equal(gpu_transpose(gpu, src), otr.transpose(src))


@pytest.mark.gpu
@pytest.mark.parametrize("offset", [1, 2, 3])
def test_parity_unaligned_rows_take_scalar_path(gpu, offset):
    src = make_matrix(200, 256, seed=offset)   # w % 4 == 0 but src not 16-byte aligned
    assert np.array_equal(gpu_transpose(gpu, src, offset), otr.transpose(src))


@pytest.mark.gpu
def test_eval_path_and_coherence(gpu):
    """hpl_eval("transpose_f32") over dest's domain; dest becomes device-valid,
    the host copy is fetched by sync(HOST) (the paper's Array coherence)."""
    torch, hpl = gpu
    h, w = 300, 170
    src = make_matrix(h, w, seed=11)
    a_src = hpl.hpl_array_alloc(hpl.HPL_F32, [h, w])
    a_dst = hpl.hpl_array_alloc(hpl.HPL_F32, [w, h])
    try:
        p = hpl.hpl_array_data(a_src, hpl.HPL_HOST)
        np.ctypeslib.as_array((ctypes.c_float * (h * w)).from_address(p))[:] = src.reshape(-1)
        hpl.hpl_array_sync(a_src, hpl.HPL_HOST, hpl.HPL_WRITE)
        hpl.hpl_eval("transpose_f32", [a_dst, a_src])
        hpl.hpl_array_sync(a_dst, hpl.HPL_HOST, hpl.HPL_READ)
        q = hpl.hpl_array_data(a_dst, hpl.HPL_HOST)
        got = np.ctypeslib.as_array((ctypes.c_float * (h * w)).from_address(q)).reshape(w, h)
        assert np.array_equal(got, otr.transpose(src))
    finally:
        hpl.hpl_array_free(a_src)
        hpl.hpl_array_free(a_dst)


@pytest.mark.gpu
def test_full_size_sampled(gpu):
    """The benchmark size, 16K x 16K, in the launch
    configuration tools/bench_transpose.py times: 2^20 sampled positions
    against the oracle's definition, plus two whole rows and columns."""
    torch, hpl = gpu
    n = TRANSPOSE_N
    g = torch.Generator(device="cuda").manual_seed(16)
    x = torch.rand(n, n, generator=g, device="cuda", dtype=torch.float32)
    out = torch.empty(n, n, device="cuda", dtype=torch.float32)
    hpl.hpl_transpose_f32(x.data_ptr(), n, n, out.data_ptr(), torch.cuda.current_stream().cuda_stream)
    rng = np.random.default_rng(3)
    i = torch.from_numpy(rng.integers(0, n, 1 << 20)).cuda()
    j = torch.from_numpy(rng.integers(0, n, 1 << 20)).cuda()
    src_s = x[i, j].cpu().numpy()
    dst_s = out[j, i].cpu().numpy()
    assert np.array_equal(dst_s, src_s)
    for r in (0, n - 1, 12345):
        row = x[r].cpu().numpy()[None, :]
        assert np.array_equal(out[:, r].cpu().numpy(), otr.transpose(row)[:, 0])
