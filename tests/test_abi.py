"""CPU tests of the C-ABI boundary: the library loads, exports every symbol
include/hpl.h declares, and its host-side validation works without a GPU."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def hpl():
    from paper_conf_ipps_bozkusf12_b200 import build
    build.build()
    from paper_conf_ipps_bozkusf12_b200 import hpl as h
    return h


def header_functions():
    src = open(os.path.join(ROOT, "include", "hpl.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(hpl_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_what_binding_exports(hpl):
    assert header_functions() == sorted(hpl.EXPORTS)


def test_every_declared_symbol_is_exported(hpl):
    lib = ctypes.CDLL(hpl.LIB_PATH)
    for name in header_functions():
        assert hasattr(lib, name), name


def test_no_oracle_in_product_library(hpl):
    """The product library must not link or embed the oracle."""
    blob = open(hpl.LIB_PATH, "rb").read()
    assert b"ep_oracle" not in blob


def test_strerror_and_version(hpl):
    lib = hpl.lib()
    for code in (0, -1, -2, -3, -4, -5, -6):
        assert lib.hpl_strerror(code)
    assert lib.hpl_strerror(-99) == b"unknown status"
    assert hpl.hpl_version() >> 16 == 1


@pytest.mark.parametrize("seed,a", [(1 << 46, 1220703125), (1 << 45, 1220703125),
                                    (271828183, 1220703124), (271828183, 1 << 46 | 1)])
def test_invalid_parameters_rejected_before_any_cuda_call(hpl, seed, a):
    with pytest.raises(hpl.HPLError) as e:
        hpl.hpl_ep_run_range(seed, a, 0, 16, 0x1000)
    assert e.value.code == hpl.HPL_EINVAL
    with pytest.raises(hpl.HPLError) as e:
        hpl.hpl_lcg_states(seed, a, 0, 4)
    assert e.value.code == hpl.HPL_EINVAL


@pytest.mark.parametrize("M,rank,nranks", [(44, 0, 1), (-1, 0, 1), (10, 0, 3), (10, 2, 2),
                                           (2, 0, 8), (10, -1, 2)])
def test_invalid_shards_rejected(hpl, M, rank, nranks):
    with pytest.raises(hpl.HPLError) as e:
        hpl.hpl_ep_run_shard(M, 271828183, 1220703125, rank, nranks, 0x1000)
    assert e.value.code == hpl.HPL_EINVAL


def test_range_beyond_period_rejected(hpl):
    with pytest.raises(hpl.HPLError) as e:
        hpl.hpl_ep_run_range(271828183, 1220703125, (1 << 43) - 5, 10, 0x1000)
    assert e.value.code == hpl.HPL_EINVAL


def test_config_validation(hpl):
    for args in [(7, 0, 0), (0, 33, 0), (0, 2048, 0), (0, 0, -1)]:
        with pytest.raises(hpl.HPLError):
            hpl.hpl_ep_set_config(*args)
    hpl.hpl_ep_set_config(hpl.HPL_EP_LEAN, 0, 0)


def test_null_outputs_rejected(hpl):
    lib = hpl.lib()
    assert lib.hpl_ep_run(24, 271828183, 1220703125, None, None, None) == hpl.HPL_EINVAL
    assert lib.hpl_array_alloc(None, 0, 1, None, None, -1) == hpl.HPL_EINVAL
    assert lib.hpl_ep_launch_count(None) == hpl.HPL_EINVAL
    assert lib.hpl_array_free(None) == hpl.HPL_OK


def test_launch_counter_readable(hpl):
    assert hpl.hpl_ep_launch_count() >= 0


def test_allocator_hook_validation(hpl):
    """hpl_set_device_allocator: both callbacks or neither (include/hpl.h)."""
    lib = hpl.lib()
    alloc = hpl._ALLOC_T(lambda n, dev, ctx: None)
    assert lib.hpl_set_device_allocator(alloc, hpl._FREE_T(), None) == hpl.HPL_EINVAL
    assert lib.hpl_set_device_allocator(hpl._ALLOC_T(), hpl._FREE_T(lambda p, n, dev, ctx: None), None) == hpl.HPL_EINVAL
    assert b"both" in hpl.lib().hpl_last_error()
