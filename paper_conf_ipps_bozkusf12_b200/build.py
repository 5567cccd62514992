"""Build libhpl.so (the C-ABI EP library) in-tree with nvcc for sm_100a.

    python -m paper_conf_ipps_bozkusf12_b200.build [--force]

No GPU is needed: nvcc cross-compiles.  The .so lands next to this file so
that it travels with the repo snapshot to the GPU box.
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libhpl.so")
SOURCES = [os.path.join(CSRC, f) for f in ("ep_kernel.cu", "eval_kernels.cu", "reduce_kernel.cu", "transpose_kernel.cu",
                                                 "hpl_runtime.cpp")]
HEADERS = [os.path.join(CSRC, f) for f in ("ep_common.cuh", "ep_launch.h", "eval_launch.h", "reduce_launch.h")] + [
    os.path.join(ROOT, "include", "hpl.h")]

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-std=c++17", "-lineinfo",
    "-Xcompiler", "-fPIC", "-Xcompiler", "-O2",
    "-Xptxas", "-v",
    "-shared", "-cudart", "static",
]


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(p) > t for p in SOURCES + HEADERS + [__file__])


def build(force: bool = False, verbose: bool = False, out: str | None = None,
          defines: tuple = (), extra: tuple = ()) -> str:
    """Compile libhpl.so.  `out`/`defines`/`extra` (additional nvcc flags) build
    development A/B variants (e.g. defines=("EP_ILP=4",)) to another path; the
    product is LIB."""
    lib = out or LIB
    if out is None and not defines and not extra and not force and not _stale():
        return LIB
    tmp = lib + ".tmp%d" % os.getpid()
    cmd = [NVCC, *NVCC_FLAGS, *extra, *["-D" + d for d in defines], "-I", os.path.join(ROOT, "include"),
           "-o", tmp, *SOURCES]
    res = subprocess.run(cmd, capture_output=True, text=True)
    log = os.path.join(PKG, "build.log" if out is None else os.path.basename(lib) + ".log")
    with open(log, "w") as f:
        f.write(" ".join(cmd) + "\n" + res.stdout + res.stderr)
    if res.returncode != 0:
        sys.stderr.write(res.stdout + res.stderr)
        raise RuntimeError("nvcc failed (see %s)" % log)
    if verbose:
        sys.stderr.write(res.stderr)
    os.replace(tmp, lib)
    return lib


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
