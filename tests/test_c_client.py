"""Build and run the plain-C client of include/hpl.h (tests/c/hpl_c_client.c)."""
import os
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_ipps_bozkusf12_b200")


@pytest.fixture(scope="module")
def client(tmp_path_factory):
    from paper_conf_ipps_bozkusf12_b200 import build
    build.build()
    exe = str(tmp_path_factory.mktemp("c") / "hpl_c_client")
    cuda = os.environ.get("CUDA_HOME", "/usr/local/cuda")  # the test's own allocator uses cudart
    subprocess.check_call(["gcc", "-O1", "-std=c99", "-Wall", "-I", os.path.join(ROOT, "include"),
                           "-I", os.path.join(cuda, "include"),
                           os.path.join(ROOT, "tests", "c", "hpl_c_client.c"), "-L", PKG, "-lhpl",
                           "-Wl,-rpath," + PKG, "-L", os.path.join(cuda, "lib64"), "-lcudart",
                           "-Wl,-rpath," + os.path.join(cuda, "lib64"), "-lm", "-o", exe])
    return exe


def test_c_client_cpu(client):
    r = subprocess.run([client], capture_output=True, text=True)
    assert r.returncode == 0, r.stdout + r.stderr


@pytest.mark.gpu
def test_c_client_gpu(client):
    r = subprocess.run([client, "gpu"], capture_output=True, text=True)
    assert r.returncode == 0, r.stdout + r.stderr
