"""Thin ctypes binding of include/hpl.h (libhpl.so) — argument marshalling only.

Every step of EP runs in the CUDA kernels of ``csrc/``; nothing here computes.
If ``libhpl.so`` is missing the import fails loudly (no CPU fallback): build it
with ``python -m paper_conf_ipps_bozkusf12_b200.build`` (or
``__graft_entry__.build()``).

Names mirror the C ABI: ``hpl_array_alloc``, ``hpl_array_sync``,
``hpl_ep_run``, ``hpl_ep_run_shard``, ... .  Functions raise :class:`HPLError`
on a non-zero status; the C status code is ``err.code``.
"""
from __future__ import annotations

import atexit
import ctypes
import os
import sys

_PKG = os.path.dirname(os.path.abspath(__file__))
# HPL_LIB: development override to load an A/B build variant of the library
LIB_PATH = os.environ.get("HPL_LIB") or os.path.join(_PKG, "libhpl.so")

HPL_OK, HPL_EINVAL, HPL_ENOMEM, HPL_ECUDA, HPL_ENODEV, HPL_ERANGE, HPL_ESTATE = 0, -1, -2, -3, -4, -5, -6
HPL_F64, HPL_F32, HPL_U64, HPL_I64, HPL_I32, HPL_U32 = 0, 1, 2, 3, 4, 5
HPL_HOST, HPL_DEVICE = 1, 2
HPL_READ, HPL_WRITE, HPL_READWRITE = 1, 2, 3
HPL_EP_LEAN, HPL_EP_LIBDEVICE = 0, 1

# every symbol include/hpl.h declares (tests/test_abi.py checks the header agrees)
EXPORTS = (
    "hpl_strerror", "hpl_last_error", "hpl_version",
    "hpl_device_count", "hpl_set_device", "hpl_get_device",
    "hpl_array_alloc", "hpl_array_free", "hpl_array_sync", "hpl_array_data",
    "hpl_array_info", "hpl_array_set_stream",
    "hpl_ep_eval", "hpl_ep_run", "hpl_ep_run_shard", "hpl_ep_run_range",
    "hpl_lcg_states", "hpl_ep_set_config", "hpl_ep_launch_shape", "hpl_ep_launch_count",
    "hpl_eval", "hpl_kernel_count", "hpl_kernel_info", "hpl_reduce_sum_f32",
    "hpl_transpose_f32",
    "hpl_ep_pairs_debug",
    "hpl_comm_create", "hpl_comm_open", "hpl_comm_set_timeout", "hpl_comm_free",
    "hpl_ep_run_fused", "hpl_comm_status",
    "hpl_set_device_allocator", "hpl_shutdown",
)
HPL_COMM_HANDLE_BYTES, HPL_COMM_MAX_RANKS = 64, 8
HPL_ARG_ARRAY, HPL_ARG_F64, HPL_ARG_F32, HPL_ARG_I64, HPL_ARG_I32 = 0, 1, 2, 3, 4


# hpl_alloc_fn / hpl_free_fn (include/hpl.h)
_ALLOC_T = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_void_p)
_FREE_T = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_void_p)
_allocator = None  # the installed callbacks
# every callback pair ever installed stays referenced for the life of the
# process: arrays remember the allocator that made them, and one allocated
# under callbacks that were later replaced (or by another thread whose
# per-thread cache outlives hpl_shutdown) still frees through them
_keepalive = []


class HplArg(ctypes.Structure):
    """C struct hpl_arg (include/hpl.h)."""
    _fields_ = [("kind", ctypes.c_int), ("access", ctypes.c_int), ("array", ctypes.c_void_p),
                ("f64", ctypes.c_double), ("f32", ctypes.c_float), ("i64", ctypes.c_int64),
                ("i32", ctypes.c_int32)]


class HPLError(RuntimeError):
    def __init__(self, code: int, func: str, detail: str):
        self.code = code
        super().__init__("%s failed: %s (%d)%s" % (func, _strerror(code), code,
                                                    (": " + detail) if detail else ""))


_lib = None


def _load() -> ctypes.CDLL:
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError("libhpl.so not built at %s — run `python -m paper_conf_ipps_bozkusf12_b200.build`"
                          % LIB_PATH)
    lib = ctypes.CDLL(LIB_PATH)
    c_int, c_u64, c_i64, c_void_p, c_double = (ctypes.c_int, ctypes.c_uint64, ctypes.c_int64,
                                              ctypes.c_void_p, ctypes.c_double)
    P = ctypes.POINTER
    sig = {
        "hpl_strerror": (ctypes.c_char_p, [c_int]),
        "hpl_last_error": (ctypes.c_char_p, []),
        "hpl_version": (c_int, []),
        "hpl_device_count": (c_int, [P(c_int)]),
        "hpl_set_device": (c_int, [c_int]),
        "hpl_get_device": (c_int, [P(c_int)]),
        "hpl_array_alloc": (c_int, [P(c_void_p), c_int, c_int, P(c_i64), c_void_p, c_int]),
        "hpl_array_free": (c_int, [c_void_p]),
        "hpl_array_sync": (c_int, [c_void_p, c_int, c_int]),
        "hpl_array_data": (c_int, [c_void_p, c_int, P(c_void_p)]),
        "hpl_array_info": (c_int, [c_void_p, P(c_int), P(c_int), P(c_i64), P(c_i64), P(c_int)]),
        "hpl_array_set_stream": (c_int, [c_void_p, c_void_p]),
        "hpl_ep_eval": (c_int, [c_int, c_u64, c_u64, c_int, c_int, c_void_p]),
        "hpl_ep_run": (c_int, [c_int, c_u64, c_u64, P(c_double), P(c_double), P(c_u64)]),
        "hpl_ep_run_shard": (c_int, [c_int, c_u64, c_u64, c_int, c_int, c_void_p, c_void_p]),
        "hpl_ep_run_range": (c_int, [c_u64, c_u64, c_u64, c_u64, c_void_p, c_void_p]),
        "hpl_lcg_states": (c_int, [c_u64, c_u64, c_u64, c_u64, P(c_u64)]),
        "hpl_ep_set_config": (c_int, [c_int, c_int, c_int]),
        "hpl_ep_launch_shape": (c_int, [c_u64, P(c_int), P(c_int), P(c_int)]),
        "hpl_ep_launch_count": (c_int, [P(c_u64)]),
        "hpl_eval": (c_int, [ctypes.c_char_p, c_int, P(c_i64), P(c_i64), c_int, P(HplArg)]),
        "hpl_kernel_count": (c_int, [P(c_int)]),
        "hpl_reduce_sum_f32": (c_int, [c_void_p, c_i64, c_void_p, c_void_p]),
        "hpl_transpose_f32": (c_int, [c_void_p, c_i64, c_i64, c_void_p, c_void_p]),
        "hpl_ep_pairs_debug": (c_int, [c_u64, c_u64, c_u64, c_u64, P(c_double)]),
        "hpl_kernel_info": (c_int, [c_int, P(ctypes.c_char_p), P(ctypes.c_char_p)]),
        "hpl_comm_create": (c_int, [P(c_void_p), c_int, c_int, c_int, c_void_p]),
        "hpl_comm_open": (c_int, [c_void_p, c_void_p]),
        "hpl_comm_set_timeout": (c_int, [c_void_p, c_double]),
        "hpl_comm_free": (c_int, [c_void_p]),
        "hpl_ep_run_fused": (c_int, [c_void_p, c_int, c_u64, c_u64, c_void_p, c_void_p]),
        "hpl_comm_status": (c_int, [c_void_p, c_void_p, P(c_u64), P(c_u64)]),
        "hpl_set_device_allocator": (c_int, [_ALLOC_T, _FREE_T, c_void_p]),
        "hpl_shutdown": (c_int, []),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    _lib = lib
    if "torch" in sys.modules:  # the caller uses torch: arrays share its caching allocator
        use_torch_allocator()
    return lib


def _strerror(code: int) -> str:
    return _load().hpl_strerror(code).decode()


def _check(rc: int, func: str) -> None:
    if rc != HPL_OK:
        raise HPLError(rc, func, _load().hpl_last_error().decode())


def lib() -> ctypes.CDLL:
    return _load()


# ------------------------------------------------- device memory / state
def hpl_set_device_allocator(alloc=None, free=None) -> None:
    """Install Python callables alloc(nbytes, device) -> int pointer and
    free(ptr, nbytes, device) as the library's device allocator (both None:
    back to cudaMalloc)."""
    global _allocator
    lib = _load()
    if alloc is None and free is None:
        _check(lib.hpl_set_device_allocator(_ALLOC_T(), _FREE_T(), None), "hpl_set_device_allocator")
        _allocator = None
        return
    cb = (_ALLOC_T(lambda n, dev, ctx: alloc(n, dev) or None),
          _FREE_T(lambda p, n, dev, ctx: free(p, n, dev)))
    _keepalive.append(cb)
    _check(lib.hpl_set_device_allocator(cb[0], cb[1], None), "hpl_set_device_allocator")
    _allocator = cb


def use_torch_allocator() -> None:
    """Route hpl_array device memory through torch's CUDA caching allocator
    (SURVEY §8(b) memory ownership; reading B1).  Installed
    automatically when torch is imported before the library is loaded."""
    import torch

    def alloc(n, dev):
        return torch.cuda.caching_allocator_alloc(n, device=dev)

    def free(p, n, dev):
        torch.cuda.caching_allocator_delete(p)

    hpl_set_device_allocator(alloc, free)


def hpl_shutdown() -> None:
    """Free every library-owned buffer (see include/hpl.h); registered at exit
    so torch-allocated arrays are returned while the interpreter is alive."""
    global _allocator
    if _lib is not None:
        _check(_lib.hpl_shutdown(), "hpl_shutdown")
        _allocator = None


atexit.register(lambda: _lib is not None and _lib.hpl_shutdown())


# ------------------------------------------------------------------ devices
def hpl_version() -> int:
    return _load().hpl_version()


def hpl_device_count() -> int:
    n = ctypes.c_int()
    _check(_load().hpl_device_count(ctypes.byref(n)), "hpl_device_count")
    return n.value


def hpl_set_device(device: int) -> None:
    _check(_load().hpl_set_device(device), "hpl_set_device")


def hpl_get_device() -> int:
    d = ctypes.c_int()
    _check(_load().hpl_get_device(ctypes.byref(d)), "hpl_get_device")
    return d.value


# ------------------------------------------------------------------- arrays
def hpl_array_alloc(dtype: int, dims, host_ptr=None, device: int = -1) -> int:
    dims = list(dims)
    arr = (ctypes.c_int64 * max(len(dims), 1))(*dims)
    h = ctypes.c_void_p()
    _check(_load().hpl_array_alloc(ctypes.byref(h), dtype, len(dims), arr, host_ptr, device),
           "hpl_array_alloc")
    return h.value


def hpl_array_free(a: int) -> None:
    _check(_load().hpl_array_free(a), "hpl_array_free")


def hpl_array_sync(a: int, where: int, mode: int = HPL_READ) -> None:
    _check(_load().hpl_array_sync(a, where, mode), "hpl_array_sync")


def hpl_array_data(a: int, where: int) -> int:
    p = ctypes.c_void_p()
    _check(_load().hpl_array_data(a, where, ctypes.byref(p)), "hpl_array_data")
    return p.value


def hpl_array_info(a: int) -> dict:
    t, nd, nb, v = ctypes.c_int(), ctypes.c_int(), ctypes.c_int64(), ctypes.c_int()
    dims = (ctypes.c_int64 * 3)()
    _check(_load().hpl_array_info(a, ctypes.byref(t), ctypes.byref(nd), dims, ctypes.byref(nb),
                                  ctypes.byref(v)), "hpl_array_info")
    return {"dtype": t.value, "ndim": nd.value, "dims": list(dims[:nd.value]), "nbytes": nb.value,
            "valid": v.value}


def hpl_array_set_stream(a: int, stream: int | None) -> None:
    _check(_load().hpl_array_set_stream(a, stream or None), "hpl_array_set_stream")


# ----------------------------------------------------------------------- EP
def hpl_ep_eval(M: int, seed: int, a: int, rank: int, nranks: int, out13: int) -> None:
    _check(_load().hpl_ep_eval(M, seed, a, rank, nranks, out13), "hpl_ep_eval")


def hpl_ep_run(M: int, seed: int, a: int):
    """Whole EP problem on the current device: returns (sx, sy, q[10])."""
    sx, sy = ctypes.c_double(), ctypes.c_double()
    q = (ctypes.c_uint64 * 10)()
    _check(_load().hpl_ep_run(M, seed, a, ctypes.byref(sx), ctypes.byref(sy), q), "hpl_ep_run")
    return sx.value, sy.value, list(q)


def hpl_ep_run_shard(M: int, seed: int, a: int, rank: int, nranks: int, dev_out13: int,
                     stream: int | None = None) -> None:
    _check(_load().hpl_ep_run_shard(M, seed, a, rank, nranks, dev_out13, stream or None),
           "hpl_ep_run_shard")


def hpl_ep_run_range(seed: int, a: int, pair_begin: int, npairs: int, dev_out13: int,
                     stream: int | None = None) -> None:
    _check(_load().hpl_ep_run_range(seed, a, pair_begin, npairs, dev_out13, stream or None),
           "hpl_ep_run_range")


def hpl_lcg_states(seed: int, a: int, offset: int, n: int) -> list[int]:
    buf = (ctypes.c_uint64 * max(n, 1))()
    _check(_load().hpl_lcg_states(seed, a, offset, n, buf), "hpl_lcg_states")
    return list(buf[:n])


def hpl_ep_pairs_debug(seed: int, a: int, pair_begin: int, n: int):
    """Per-pair (t, X, Y, l) from the production transform code (test hook)."""
    buf = (ctypes.c_double * max(4 * n, 1))()
    _check(_load().hpl_ep_pairs_debug(seed, a, pair_begin, n, buf), "hpl_ep_pairs_debug")
    return buf


def hpl_ep_set_config(variant: int = HPL_EP_LEAN, threads_per_block: int = 0,
                      blocks_per_sm: int = 0) -> None:
    _check(_load().hpl_ep_set_config(variant, threads_per_block, blocks_per_sm), "hpl_ep_set_config")


def hpl_ep_launch_shape(npairs: int):
    b, t, s = ctypes.c_int(), ctypes.c_int(), ctypes.c_int()
    _check(_load().hpl_ep_launch_shape(npairs, ctypes.byref(b), ctypes.byref(t), ctypes.byref(s)),
           "hpl_ep_launch_shape")
    return b.value, t.value, s.value


def hpl_ep_launch_count() -> int:
    c = ctypes.c_uint64()
    _check(_load().hpl_ep_launch_count(ctypes.byref(c)), "hpl_ep_launch_count")
    return c.value


# ------------------------------------------------ fused combine (F3)
def hpl_comm_create(rank: int, nranks: int, device: int = -1) -> tuple[int, bytes]:
    """Create this rank's inbox; returns (comm handle, 64-byte IPC handle)."""
    c = ctypes.c_void_p()
    buf = ctypes.create_string_buffer(HPL_COMM_HANDLE_BYTES)
    _check(_load().hpl_comm_create(ctypes.byref(c), rank, nranks, device, buf), "hpl_comm_create")
    return c.value, buf.raw


def hpl_comm_open(comm: int, handles: bytes) -> None:
    """handles: nranks * 64 bytes in rank order."""
    buf = ctypes.create_string_buffer(bytes(handles), len(handles))
    _check(_load().hpl_comm_open(comm, buf), "hpl_comm_open")


def hpl_comm_set_timeout(comm: int, seconds: float) -> None:
    _check(_load().hpl_comm_set_timeout(comm, seconds), "hpl_comm_set_timeout")


def hpl_comm_free(comm: int) -> None:
    _check(_load().hpl_comm_free(comm), "hpl_comm_free")


def hpl_ep_run_fused(comm: int, M: int, seed: int, a: int, dev_out13: int,
                     stream: int | None = None) -> None:
    _check(_load().hpl_ep_run_fused(comm, M, seed, a, dev_out13, stream or None), "hpl_ep_run_fused")


def hpl_comm_status(comm: int, stream: int | None = None) -> tuple[int, int]:
    """(epoch, timeouts) after synchronizing `stream`; raises if a combine timed out."""
    e, t = ctypes.c_uint64(), ctypes.c_uint64()
    _check(_load().hpl_comm_status(comm, stream or None, ctypes.byref(e), ctypes.byref(t)),
           "hpl_comm_status")
    return e.value, t.value


# ---------------------------------------------------------- reduction (F2)
def hpl_reduce_sum_f32(dev_in: int, n: int, dev_out: int, stream: int | None = None) -> None:
    _check(_load().hpl_reduce_sum_f32(dev_in, n, dev_out, stream or None), "hpl_reduce_sum_f32")


# ---------------------------------------------------------- transpose (F4)
def hpl_transpose_f32(dev_src: int, h: int, w: int, dev_dst: int, stream: int | None = None) -> None:
    """dev_dst (w x h) = transpose of dev_src (h x w), row-major float32, device pointers."""
    _check(_load().hpl_transpose_f32(dev_src, h, w, dev_dst, stream or None), "hpl_transpose_f32")


# ------------------------------------------------------- generic eval (F1)
def _arg(v) -> HplArg:
    a = HplArg()
    if isinstance(v, tuple):
        kind, val = v
        if kind == "array":
            a.kind, a.array = HPL_ARG_ARRAY, val
        elif kind == "f64":
            a.kind, a.f64 = HPL_ARG_F64, val
        elif kind == "f32":
            a.kind, a.f32 = HPL_ARG_F32, val
        elif kind == "i64":
            a.kind, a.i64 = HPL_ARG_I64, val
        elif kind == "i32":
            a.kind, a.i32 = HPL_ARG_I32, val
        else:
            raise ValueError(kind)
    elif isinstance(v, float):
        a.kind, a.f64 = HPL_ARG_F64, v
    else:  # an hpl_array handle
        a.kind, a.array = HPL_ARG_ARRAY, v
    return a


def hpl_eval(name: str, args, global_=None, local=None) -> None:
    """eval(name).global(global_).local(local)(*args); arrays are handles,
    scalars floats (f64) or (kind, value) tuples."""
    arr = (HplArg * max(len(args), 1))(*[_arg(v) for v in args])
    nd = len(global_) if global_ else 0
    gl, ll = list(global_ or []), list(local or [])
    g = (ctypes.c_int64 * max(3, len(gl)))(*(gl + [0] * (3 - len(gl))))
    l = (ctypes.c_int64 * max(3, len(ll)))(*(ll + [0] * (3 - len(ll))))
    _check(_load().hpl_eval(name.encode(), nd, g if nd else None, l if local else None, len(args), arr),
           "hpl_eval")


def hpl_kernels() -> dict:
    n = ctypes.c_int()
    _check(_load().hpl_kernel_count(ctypes.byref(n)), "hpl_kernel_count")
    out = {}
    for i in range(n.value):
        nm, sg = ctypes.c_char_p(), ctypes.c_char_p()
        _check(_load().hpl_kernel_info(i, ctypes.byref(nm), ctypes.byref(sg)), "hpl_kernel_info")
        out[nm.value.decode()] = sg.value.decode()
    return out


def unpack13(words) -> dict:
    """Split the 13-word result [sx, sy, q0..q9, gc] (marshalling helper)."""
    w = list(words)
    return {"sx": float(w[0]), "sy": float(w[1]), "q": [int(v) for v in w[2:12]], "gc": int(w[12])}
