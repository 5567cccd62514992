"""Measured-and-dropped build variants stay buildable and correct.

DESIGN.md §4.1 (`EP_I2F`: uniforms by I2F.F64.S64 from a signed 64-bit LCG
state, t'' = t' 2^128) and §9 (`SPMV_PIPE`: predicated, software-pipelined
spmv chunks) describe variants that were timed on the B200 and left off.  So
that those records keep describing code that works, each variant is compiled
here (CPU: nvcc cross-compiles sm_100a) and, on a GPU, the parity tests of the
path it changes run against it in a subprocess (HPL_LIB selects the library).
"""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
VARIANTS = {
    "i2f": (("EP_I2F=1",), ["tests/test_gpu_parity.py", "tests/test_edge_pairs.py", "tests/test_gpu_accuracy.py"]),
    "spmvpipe": (("SPMV_PIPE=1",), ["tests/test_spmv.py"]),
}


def _lib(name):
    return os.path.join(ROOT, "paper_conf_ipps_bozkusf12_b200", "variants", "libhpl_%s.so" % name)


def _build(name):
    from paper_conf_ipps_bozkusf12_b200 import build
    os.makedirs(os.path.dirname(_lib(name)), exist_ok=True)
    return build.build(out=_lib(name), defines=VARIANTS[name][0])


@pytest.mark.parametrize("name", sorted(VARIANTS))
def test_variant_builds(name):
    lib = _build(name)
    assert os.path.getsize(lib) > 0
    # the variant really differs where it claims to: its kernels carry the new code
    sass = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
    if name == "i2f":
        assert "I2F.F64.S64" in sass
    else:
        from paper_conf_ipps_bozkusf12_b200 import build
        base = subprocess.run(["cuobjdump", "-sass", build.build()], capture_output=True, text=True).stdout
        assert _fn(sass, "k_spmv_csr") != _fn(base, "k_spmv_csr")


def _fn(sass, name):
    """SASS text of the function whose name contains `name` (addresses stripped)."""
    out, on = [], False
    for ln in sass.splitlines():
        if "Function :" in ln:
            on = name in ln
        elif on and "/*" in ln:
            out.append(ln.split("*/", 1)[-1].split(";")[0].strip())
    return out


@pytest.mark.gpu
@pytest.mark.parametrize("name", sorted(VARIANTS))
def test_variant_parity_on_gpu(name):
    lib = _lib(name) if os.path.exists(_lib(name)) else _build(name)
    env = dict(os.environ, HPL_LIB=lib)
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "-p", "no:cacheprovider",
                        *VARIANTS[name][1]], cwd=ROOT, env=env, capture_output=True, text=True, timeout=1500)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
    assert " passed" in r.stdout
