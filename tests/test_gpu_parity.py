"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle.

Gates: LCG states bit-exact; q[0..9] and gc exact; sx, sy
within T1 = 1e-12 * max(|ref|, sqrt(gc)); NPB verification sums within 1e-8.
Every GPU number comes from libhpl.so kernels; every expected value from
oracle/ (live, or tests/golden/oracle_ep.json written by a script that calls
only oracle/) or from NPB's published sums.
"""
import math
import random

import pytest

from _golden import npb_verify, oracle_golden, sums_close
from ep_workloads import CLASSES, NPB_A, NPB_SEED, ROBUST_SEEDS

pytestmark = pytest.mark.gpu

VARIANTS = [0, 1]  # HPL_EP_LEAN, HPL_EP_LIBDEVICE


@pytest.fixture(scope="module")
def env():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_bozkusf12_b200 import build
    build.build()
    from paper_conf_ipps_bozkusf12_b200 import hpl
    hpl.hpl_set_device(0)
    torch.cuda.set_device(0)
    return torch, hpl


def gpu_range(env, seed, a, begin, n, variant=0, threads=0, bps=0):
    torch, hpl = env
    hpl.hpl_ep_set_config(variant, threads, bps)
    out = torch.full((13,), -7.0, dtype=torch.float64, device="cuda")
    hpl.hpl_ep_run_range(seed, a, begin, n, out.data_ptr(), torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    hpl.hpl_ep_set_config(0, 0, 0)
    return hpl.unpack13(out.cpu().tolist())


def assert_parity(g, r, rel=1e-12):
    assert g["q"] == list(r.q), (g["q"], r.q)
    assert g["gc"] == r.gc
    assert sums_close(g["sx"], r.sx, r.gc, rel), (g["sx"], r.sx)
    assert sums_close(g["sy"], r.sy, r.gc, rel), (g["sy"], r.sy)


# -------------------------------------------------------------- LCG stream
@pytest.mark.parametrize("offset", [0, 1, 2 ** 17 - 3, 2 ** 25 + 7, 2 ** 33 - 1, 2 ** 37 - 5,
                                    2 ** 44 - 100])
def test_lcg_states_bit_exact(env, oracle_mod, offset):
    _, hpl = env
    n = 4096
    assert hpl.hpl_lcg_states(NPB_SEED, NPB_A, offset, n) == oracle_mod.states(NPB_SEED, NPB_A, offset, n)


@pytest.mark.parametrize("a", [NPB_A, 5 ** 19 % 2 ** 46, 2 ** 46 - 1, 3])
def test_lcg_states_other_multipliers(env, oracle_mod, a):
    _, hpl = env
    assert hpl.hpl_lcg_states(12345, a, 999, 1000) == oracle_mod.states(12345, a, 999, 1000)


# ----------------------------------------------------------- small sizes
@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("M", [0, 1, 2, 5, 8, 11, 14, 17, 20])
def test_tiny_M(env, oracle_mod, variant, M):
    g = gpu_range(env, NPB_SEED, NPB_A, 0, 2 ** M, variant)
    assert_parity(g, oracle_mod.run(M, NPB_SEED, NPB_A))


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("begin,n", [(0, 0), (5, 1), (12345, 3), (2 ** 20 + 1, 99991),
                                     (2 ** 35 - 77777, 1_000_003), (2 ** 43 - 600_000, 600_000)])
def test_ragged_ranges(env, oracle_mod, variant, begin, n):
    """Ragged pair ranges: per-thread counts differ by one, ranges start mid-batch."""
    g = gpu_range(env, NPB_SEED, NPB_A, begin, n, variant)
    assert_parity(g, oracle_mod.run_pairs(NPB_SEED, NPB_A, begin, n))


@pytest.mark.parametrize("threads,bps", [(32, 1), (64, 3), (256, 1), (512, 2), (1024, 1)])
def test_launch_shapes(env, oracle_mod, threads, bps):
    """Result independent of the launch shape (counts exact, sums within T1)."""
    g = gpu_range(env, NPB_SEED, NPB_A, 1000, 3_000_017, 0, threads, bps)
    assert_parity(g, oracle_mod.run_pairs(NPB_SEED, NPB_A, 1000, 3_000_017))


@pytest.mark.parametrize("seed", ROBUST_SEEDS)
def test_robust_seeds(env, oracle_mod, seed):
    g = gpu_range(env, seed, NPB_A, 0, 2 ** 20)
    assert_parity(g, oracle_mod.run(20, seed, NPB_A))


@pytest.mark.parametrize("a", [5 ** 19 % 2 ** 46, 2 ** 46 - 1, (2 ** 45) + 12345 * 2 + 1])
def test_wide_multiplier(env, oracle_mod, a):
    """a >= 2^32 takes the general 64-bit multiply path."""
    g = gpu_range(env, 271828183, a, 777, 2 ** 19)
    assert_parity(g, oracle_mod.run_pairs(271828183, a, 777, 2 ** 19))


def test_seed_zero(env):
    g = gpu_range(env, 0, NPB_A, 0, 2 ** 16)
    assert g["gc"] == 0 and g["sx"] == 0.0 and g["sy"] == 0.0


# ---------------------------------------------------------- NPB classes
@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("cls", ["S", "W", "A"])
def test_npb_class_vs_oracle(env, oracle_mod, variant, cls):
    _, hpl = env
    M = CLASSES[cls]
    hpl.hpl_ep_set_config(variant, 0, 0)
    sx, sy, q = hpl.hpl_ep_run(M, NPB_SEED, NPB_A)
    hpl.hpl_ep_set_config(0, 0, 0)
    r = oracle_mod.run(M, NPB_SEED, NPB_A, threads=16, margin=False)
    assert_parity({"sx": sx, "sy": sy, "q": q, "gc": sum(q)}, r)
    _, sxr, syr = npb_verify()[cls]
    assert abs((sx - sxr) / sxr) <= 1e-8 and abs((sy - syr) / syr) <= 1e-8


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("cls", ["B", "C", "D"])
def test_npb_large_class_vs_golden(env, variant, cls):
    """Full-size runs in bench.py's launch configuration vs the stored oracle."""
    _, hpl = env
    gold = oracle_golden().get(cls)
    if gold is None:
        pytest.skip("tests/golden/oracle_ep.json lacks class %s" % cls)
    hpl.hpl_ep_set_config(variant, 0, 0)
    sx, sy, q = hpl.hpl_ep_run(gold["M"], NPB_SEED, NPB_A)
    hpl.hpl_ep_set_config(0, 0, 0)
    assert q == gold["q"] and sum(q) == gold["gc"]
    assert sums_close(sx, gold["sx"], gold["gc"]) and sums_close(sy, gold["sy"], gold["gc"])
    _, sxr, syr = npb_verify()[cls]
    assert abs((sx - sxr) / sxr) <= 1e-8 and abs((sy - syr) / syr) <= 1e-8


def test_class_D_sampled_ranges(env, oracle_mod):
    """Sampled sub-ranges of class D (incl. the last pairs before 2^36) that the
    oracle computes one by one."""
    rng = random.Random(36)
    for begin in [0, 2 ** 36 - 2 ** 21] + [rng.randrange(2 ** 36 - 2 ** 21) for _ in range(2)]:
        g = gpu_range(env, NPB_SEED, NPB_A, begin, 2 ** 21)
        assert_parity(g, oracle_mod.run_pairs(NPB_SEED, NPB_A, begin, 2 ** 21))


# -------------------------------------------------------- multi-GPU math
@pytest.mark.parametrize("G", [2, 4, 8])
def test_fake_multi_gpu_shards(env, oracle_mod, G):
    """Shards r = 0..G-1 run serially on one GPU sum to the whole run (this is
    the arithmetic of the NCCL path minus the allreduce)."""
    torch, hpl = env
    M = 24
    acc = torch.zeros(13, dtype=torch.float64, device="cuda")
    for r in range(G):
        out = torch.empty(13, dtype=torch.float64, device="cuda")
        hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, r, G, out.data_ptr(),
                             torch.cuda.current_stream().cuda_stream)
        acc += out
    torch.cuda.synchronize()
    g = hpl.unpack13(acc.cpu().tolist())
    assert_parity(g, oracle_mod.run(M, NPB_SEED, NPB_A, threads=16, margin=False))


def test_deterministic(env):
    _, hpl = env
    a = hpl.hpl_ep_run(26, NPB_SEED, NPB_A)
    b = hpl.hpl_ep_run(26, NPB_SEED, NPB_A)
    assert a == b  # fixed-order reductions: bitwise reproducible


# ------------------------------------------------------- Array coherence
def test_array_coherence_cycle(env):
    torch, hpl = env
    a = hpl.hpl_array_alloc(hpl.HPL_F64, [13])
    try:
        info = hpl.hpl_array_info(a)
        assert info["valid"] == hpl.HPL_HOST | hpl.HPL_DEVICE and info["nbytes"] == 104
        hpl.hpl_ep_eval(20, NPB_SEED, NPB_A, 0, 1, a)
        assert hpl.hpl_array_info(a)["valid"] == hpl.HPL_DEVICE  # kernel output
        hpl.hpl_array_sync(a, hpl.HPL_HOST, hpl.HPL_READ)
        assert hpl.hpl_array_info(a)["valid"] == hpl.HPL_HOST | hpl.HPL_DEVICE
        host = hpl.hpl_array_data(a, hpl.HPL_HOST)
        import ctypes
        words = list((ctypes.c_double * 13).from_address(host))
        sx, sy, q = hpl.hpl_ep_run(20, NPB_SEED, NPB_A)
        assert words[0] == sx and words[2:12] == [float(v) for v in q]
        hpl.hpl_array_sync(a, hpl.HPL_HOST, hpl.HPL_WRITE)
        assert hpl.hpl_array_info(a)["valid"] == hpl.HPL_HOST
        (ctypes.c_double * 13).from_address(host)[0] = 42.0
        hpl.hpl_array_sync(a, hpl.HPL_DEVICE, hpl.HPL_READ)  # H2D copy, both valid
        hpl.hpl_array_sync(a, hpl.HPL_DEVICE, hpl.HPL_WRITE)  # host copy now stale
        assert hpl.hpl_array_info(a)["valid"] == hpl.HPL_DEVICE
        (ctypes.c_double * 13).from_address(host)[0] = 0.0
        hpl.hpl_array_sync(a, hpl.HPL_HOST, hpl.HPL_READ)  # D2H brings 42 back
        assert (ctypes.c_double * 13).from_address(host)[0] == 42.0
    finally:
        hpl.hpl_array_free(a)


def test_array_user_host_pointer(env):
    _, hpl = env
    import ctypes
    buf = (ctypes.c_double * 6)(*range(6))
    a = hpl.hpl_array_alloc(hpl.HPL_F64, [2, 3], ctypes.addressof(buf))
    try:
        assert hpl.hpl_array_info(a)["valid"] == hpl.HPL_HOST
        hpl.hpl_array_sync(a, hpl.HPL_DEVICE, hpl.HPL_READWRITE)
        assert hpl.hpl_array_info(a)["valid"] == hpl.HPL_DEVICE
        buf[0] = -1.0  # host stale: the sync below must copy the device data back
        hpl.hpl_array_sync(a, hpl.HPL_HOST, hpl.HPL_READ)
        assert list(buf) == [0.0, 1.0, 2.0, 3.0, 4.0, 5.0]
    finally:
        hpl.hpl_array_free(a)


def test_eval_rejects_wrong_array(env):
    _, hpl = env
    a = hpl.hpl_array_alloc(hpl.HPL_F32, [13])
    try:
        with pytest.raises(hpl.HPLError) as e:
            hpl.hpl_ep_eval(10, NPB_SEED, NPB_A, 0, 1, a)
        assert e.value.code == hpl.HPL_EINVAL
    finally:
        hpl.hpl_array_free(a)


# ------------------------------------------------- streams / graph capture
def test_two_streams_concurrently(env, oracle_mod):
    """Per-(device, stream) workspaces: shards launched on two streams at once."""
    torch, hpl = env
    M = 22
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    o1 = torch.empty(13, dtype=torch.float64, device="cuda")
    o2 = torch.empty(13, dtype=torch.float64, device="cuda")
    for _ in range(3):
        hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, 0, 2, o1.data_ptr(), s1.cuda_stream)
        hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, 1, 2, o2.data_ptr(), s2.cuda_stream)
    torch.cuda.synchronize()
    g = hpl.unpack13((o1 + o2).cpu().tolist())
    assert_parity(g, oracle_mod.run(M, NPB_SEED, NPB_A, margin=False))


def test_cuda_graph_replay(env, oracle_mod):
    """The single EP launch is graph-capturable (counter self-resets) and replays exactly."""
    torch, hpl = env
    M = 21
    out = torch.zeros(13, dtype=torch.float64, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, 0, 1, out.data_ptr(), s.cuda_stream)  # warm workspace
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, 0, 1, out.data_ptr(), s.cuda_stream)
    ref = oracle_mod.run(M, NPB_SEED, NPB_A, margin=False)
    for _ in range(3):
        out.zero_()
        g.replay()
        torch.cuda.synchronize()
        assert_parity(hpl.unpack13(out.cpu().tolist()), ref)


def test_launch_count_advances(env):
    _, hpl = env
    c0 = hpl.hpl_ep_launch_count()
    hpl.hpl_ep_run(10, NPB_SEED, NPB_A)
    assert hpl.hpl_ep_launch_count() == c0 + 1


def test_npb_class_E_verification_sums(env):
    """Class E (M = 40, 2^41 uniforms, ~2 s on one B200): no oracle run is
    affordable, so the pin is NPB's published verification sums (1e-8) plus
    the statistical invariants."""
    _, hpl = env
    M, sxr, syr = npb_verify()["E"]
    assert M == 40
    sx, sy, q = hpl.hpl_ep_run(M, NPB_SEED, NPB_A)
    assert abs((sx - sxr) / sxr) <= 1e-8 and abs((sy - syr) / syr) <= 1e-8
    n, p = 2 ** M, math.pi / 4
    gc = sum(q)
    assert abs(gc - n * p) < 5 * math.sqrt(n * p * (1 - p))
    assert q[9] == 0 and q[8] <= 2


def test_class_E_sampled_ranges(env, oracle_mod):
    """Class E q[] parity where the oracle can follow: sampled sub-ranges of the
    M = 40 stream (incl. the first pairs and the last ones before 2^40) through
    the same kernel, q and gc exact, sums within T1."""
    rng = random.Random(40)
    for begin in [0, 2 ** 40 - 2 ** 21] + [rng.randrange(2 ** 40 - 2 ** 21) for _ in range(3)]:
        g = gpu_range(env, NPB_SEED, NPB_A, begin, 2 ** 21)
        assert_parity(g, oracle_mod.run_pairs(NPB_SEED, NPB_A, begin, 2 ** 21))


def test_class_E_shards_add_up(env):
    """Class E split into 8 shards (the 8-GPU layout, run serially here): the
    shards' q and gc add up to the whole run's bit for bit, sums within T1."""
    torch, hpl = env
    M = 40
    sx, sy, q = hpl.hpl_ep_run(M, NPB_SEED, NPB_A)
    acc = torch.zeros(13, dtype=torch.float64, device="cuda")
    for r in range(8):
        out = torch.empty(13, dtype=torch.float64, device="cuda")
        hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, r, 8, out.data_ptr(), torch.cuda.current_stream().cuda_stream)
        acc += out
    torch.cuda.synchronize()
    g = hpl.unpack13(acc.cpu().tolist())
    assert g["q"] == list(q) and g["gc"] == sum(q)
    assert sums_close(g["sx"], sx, sum(q)) and sums_close(g["sy"], sy, sum(q))


@pytest.mark.parametrize("case", range(8))
def test_random_streams(env, oracle_mod, case):
    """Seeded random (seed, a, range) combinations incl. wide multipliers and
    ranges near the 2^43-pair limit, vs the oracle."""
    rng = random.Random(1000 + case)
    seed = rng.randrange(1 << 46)
    if seed == 1 << 45:
        seed += 1
    a = (rng.randrange(1 << 46) | 1) if case % 2 else (rng.randrange(1 << 31) | 1)
    n = rng.randrange(1, 1 << 21)
    begin = rng.randrange((1 << 43) - n)
    g = gpu_range(env, seed, a, begin, n)
    assert_parity(g, oracle_mod.run_pairs(seed, a, begin, n))


def test_acceptance_boundary_pairs(env, oracle_mod):
    """Pairs whose t lies just above 1 (t' shares the high word of 1/4 and is
    rejected: the kernel routes them through the rare path, which rejects
    them exactly) and just below 1 (accepted, top table bucket), located in
    the class-S stream with the oracle's own LCG; each is checked inside a
    2^21-pair range in the bench launch shape (q, gc exact, sums within T1)."""
    import numpy as np
    st = oracle_mod.states_array(NPB_SEED, NPB_A, 0, 1 << 24)   # x_1 .. x_{2^24}: 2^23 pairs
    u = st.astype(np.float64) * 2.0 ** -46
    x1, x2 = 2.0 * u[0::2] - 1.0, 2.0 * u[1::2] - 1.0
    t = x1 * x1 + x2 * x2                                          # NPB roundings (no contraction in numpy)
    above = np.where((t > 1.0) & (t < 1.0 + 2.0 ** -20))[0]
    below = np.where((t <= 1.0) & (t > 1.0 - 2.0 ** -20))[0]
    assert len(above) >= 4 and len(below) >= 4
    for i in list(above[:4]) + list(below[:3]):
        assert oracle_mod.pair_t(float(x1[i]), float(x2[i])) == t[i]
        begin = max(int(i) - (1 << 20), 0)
        g = gpu_range(env, NPB_SEED, NPB_A, begin, 1 << 21)
        assert_parity(g, oracle_mod.run_pairs(NPB_SEED, NPB_A, begin, 1 << 21))


def test_arrays_draw_from_torchs_allocator(env):
    """SURVEY §8(b) memory ownership: with torch loaded, hpl_array device
    memory comes from torch's caching allocator (the binding installs it)."""
    torch, hpl = env
    before = torch.cuda.memory_allocated()
    a = hpl.hpl_array_alloc(hpl.HPL_F64, [1 << 20])
    try:
        assert torch.cuda.memory_allocated() - before >= 8 << 20
    finally:
        hpl.hpl_array_free(a)
    assert torch.cuda.memory_allocated() == before
