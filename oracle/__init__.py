"""EP oracle — TEST INFRASTRUCTURE, NOT PRODUCT CODE.

ctypes wrapper over ``oracle/ep_oracle.cpp``: a plain single-threaded (or
batch-threaded, order-deterministic) NPB EP in IEEE double, written from NPB
3.x ``ep.f``/``randdp.f`` — the benchmark PAPER.md:789-791 evaluates and cites
as reference [16].  See the C++ header comment for the
step-by-step citations and DESIGN.md "Readings" for every interpretation.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  It
imports nothing from ``paper_conf_ipps_bozkusf12_b200`` and vice versa.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ep_oracle.cpp")
_LIB = os.path.join(_HERE, "libep_oracle.so")

# g++ flags: -ffp-contract=off keeps x1**2 + x2**2 unfused (R5).
CXXFLAGS = ["-O2", "-std=c++17", "-ffp-contract=off", "-fPIC", "-shared", "-pthread"]


def build(force: bool = False) -> str:
    """Compile the oracle shared library in-tree (g++); returns its path."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["g++", *CXXFLAGS, "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


class _Result(ctypes.Structure):
    _fields_ = [
        ("sx", ctypes.c_double),
        ("sy", ctypes.c_double),
        ("q", ctypes.c_uint64 * 10),
        ("gc", ctypes.c_uint64),
        ("qbig", ctypes.c_uint64),
        ("npairs", ctypes.c_uint64),
        ("min_margin_ulp", ctypes.c_double),
    ]


@dataclass
class EPResult:
    sx: float
    sy: float
    q: list = field(default_factory=list)
    gc: int = 0
    qbig: int = 0
    npairs: int = 0
    min_margin_ulp: float = float("inf")


_lib = None


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        d, i, u64, i64 = ctypes.c_double, ctypes.c_int, ctypes.c_uint64, ctypes.c_int64
        R = ctypes.POINTER(_Result)
        lib.ep_oracle_randlc.argtypes = [ctypes.POINTER(d), d]
        lib.ep_oracle_randlc.restype = d
        lib.ep_oracle_pair_t.argtypes = [d, d]
        lib.ep_oracle_pair_t.restype = d
        lib.ep_oracle_states.argtypes = [d, d, u64, u64, ctypes.POINTER(u64)]
        lib.ep_oracle_states.restype = i
        lib.ep_oracle_an.argtypes = [d, i]
        lib.ep_oracle_an.restype = d
        lib.ep_oracle_run_batches.argtypes = [i, d, d, i, i64, i64, i, i, R]
        lib.ep_oracle_run_batches.restype = i
        lib.ep_oracle_run.argtypes = [i, d, d, i, i, i, R]
        lib.ep_oracle_run.restype = i
        lib.ep_oracle_run_pairs.argtypes = [d, d, u64, u64, i, R]
        lib.ep_oracle_run_pairs.restype = i
        lib.ep_oracle_csum.argtypes = [ctypes.c_void_p, u64]
        lib.ep_oracle_csum.restype = d
        lib.ep_oracle_bin_margin.argtypes = [d]
        lib.ep_oracle_bin_margin.restype = d
        lib.ep_oracle_pairs.argtypes = [d, d, u64, u64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        lib.ep_oracle_pairs.restype = i
        _lib = lib
    return _lib


def _conv(r: _Result, rc: int) -> EPResult:
    if rc not in (0, -5):
        raise ValueError("ep_oracle: invalid arguments (rc=%d)" % rc)
    return EPResult(r.sx, r.sy, list(r.q), r.gc, r.qbig, r.npairs, r.min_margin_ulp)


def randlc(x: float, a: float) -> tuple[float, float]:
    """NPB randlc: returns (uniform, new state)."""
    xx = ctypes.c_double(x)
    u = _load().ep_oracle_randlc(ctypes.byref(xx), a)
    return u, xx.value


def pair_t(x1: float, x2: float) -> float:
    """t = x1**2 + x2**2 exactly as the oracle's Gaussian loop evaluates it."""
    return _load().ep_oracle_pair_t(x1, x2)


def states(seed: int, a: int, offset: int, n: int) -> list[int]:
    """x_{offset+1} .. x_{offset+n} of the NPB LCG stream started at x_0 = seed."""
    buf = (ctypes.c_uint64 * max(n, 1))()
    _load().ep_oracle_states(float(seed), float(a), offset, n, buf)
    return list(buf[:n])


def states_array(seed: int, a: int, offset: int, n: int):
    """states() as a numpy uint64 array (same C routine; for scanning large ranges)."""
    import numpy as np
    out = np.empty(max(n, 1), dtype=np.uint64)
    _load().ep_oracle_states(float(seed), float(a), offset, n, out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)))
    return out[:n]


def an(a: int, mk: int = 16) -> int:
    return int(_load().ep_oracle_an(float(a), mk))


def run(M: int, seed: int, a: int, mk: int = -1, threads: int = 1, margin: bool = True) -> EPResult:
    """Whole NPB EP run over 2^M pairs."""
    r = _Result()
    rc = _load().ep_oracle_run(M, float(seed), float(a), mk, threads, int(margin), ctypes.byref(r))
    return _conv(r, rc)


def run_batches(M: int, seed: int, a: int, kk_begin: int, kk_end: int, mk: int = -1,
                threads: int = 1, margin: bool = True) -> EPResult:
    if mk < 0:
        mk = M if M < 16 else 16
    r = _Result()
    rc = _load().ep_oracle_run_batches(M, float(seed), float(a), mk, kk_begin, kk_end, threads,
                                       int(margin), ctypes.byref(r))
    return _conv(r, rc)


def run_pairs(seed: int, a: int, p_begin: int, npairs: int, margin: bool = True) -> EPResult:
    """Pairs [p_begin, p_begin + npairs) of the global stream."""
    r = _Result()
    rc = _load().ep_oracle_run_pairs(float(seed), float(a), p_begin, npairs, int(margin),
                                     ctypes.byref(r))
    return _conv(r, rc)


def csum(values) -> float:
    """The oracle's Neumaier-compensated sum (reading R10) of a float sequence."""
    import numpy as np
    v = np.ascontiguousarray(values, dtype=np.float64)
    return _load().ep_oracle_csum(v.ctypes.data, v.size)


def bin_margin(m: float) -> float:
    """Reading R7: ulps from m to the nearest integer in 1..10 (1e300 if none)."""
    return _load().ep_oracle_bin_margin(m)


def pairs(seed: int, a: int, p_begin: int, n: int):
    """Per-pair deviates (X, Y, l) of pairs [p_begin, p_begin + n) as numpy
    arrays; rejected pairs have X = Y = 0 and l = -1."""
    import numpy as np
    X = np.zeros(max(n, 1)); Y = np.zeros(max(n, 1)); l = np.zeros(max(n, 1), dtype=np.int64)
    _load().ep_oracle_pairs(float(seed), float(a), p_begin, n, X.ctypes.data, Y.ctypes.data, l.ctypes.data)
    return X[:n], Y[:n], l[:n]
