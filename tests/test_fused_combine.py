"""F3: the in-kernel cross-GPU combine (hpl_ep_run_fused, include/hpl.h).

The EP kernel's last block stores its 13-word partial into every rank's inbox
(CUDA IPC mappings, peer stores), signals with system-scope atomics, waits for
all partials and sums them in rank order, so each rank holds the whole
problem's result without a separate collective.

CPU tests: argument validation happens before any CUDA call.  GPU tests: one
rank (the combine degenerates to a copy), and two processes sharing GPU 0
(the gpurun box has one GPU; CUDA IPC and the system-scope flag protocol are
the same across processes on one device as across NVLink peers), checked
against the oracle (q exact, sx/sy within T1) over several consecutive calls
(both inbox parities), plus the timeout path when a peer never arrives.
"""
import os
import socket

import pytest

from _golden import sums_close
from ep_workloads import NPB_A, NPB_SEED

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def hpl():
    from paper_conf_ipps_bozkusf12_b200 import build
    build.build()
    from paper_conf_ipps_bozkusf12_b200 import hpl as h
    return h


# ------------------------------------------------------------------ CPU
def test_comm_argument_errors(hpl):
    lib = hpl.lib()
    import ctypes
    c = ctypes.c_void_p()
    buf = ctypes.create_string_buffer(64)
    assert lib.hpl_comm_create(ctypes.byref(c), 0, 0, -1, buf) == hpl.HPL_EINVAL
    assert lib.hpl_comm_create(ctypes.byref(c), 0, 9, -1, buf) == hpl.HPL_EINVAL
    assert lib.hpl_comm_create(ctypes.byref(c), 2, 2, -1, buf) == hpl.HPL_EINVAL
    assert lib.hpl_comm_create(ctypes.byref(c), -1, 2, -1, buf) == hpl.HPL_EINVAL
    assert lib.hpl_comm_create(None, 0, 1, -1, buf) == hpl.HPL_EINVAL
    assert lib.hpl_comm_create(ctypes.byref(c), 0, 1, -1, None) == hpl.HPL_EINVAL
    assert lib.hpl_comm_open(None, buf) == hpl.HPL_EINVAL
    assert lib.hpl_comm_set_timeout(None, 1.0) == hpl.HPL_EINVAL
    assert lib.hpl_ep_run_fused(None, 24, NPB_SEED, NPB_A, None, None) == hpl.HPL_EINVAL
    e, t = ctypes.c_uint64(), ctypes.c_uint64()
    assert lib.hpl_comm_status(None, None, ctypes.byref(e), ctypes.byref(t)) == hpl.HPL_EINVAL
    assert lib.hpl_comm_free(None) == hpl.HPL_OK


# ------------------------------------------------------------------ GPU
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.gpu
def test_fused_single_rank_equals_shard(hpl, oracle_mod):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.set_device(0)
    hpl.hpl_set_device(0)
    comm, handle = hpl.hpl_comm_create(0, 1, 0)
    try:
        hpl.hpl_comm_open(comm, handle)
        s = torch.cuda.current_stream().cuda_stream
        for M in (20, 24):
            a = torch.empty(13, dtype=torch.float64, device="cuda")
            b = torch.empty(13, dtype=torch.float64, device="cuda")
            hpl.hpl_ep_run_fused(comm, M, NPB_SEED, NPB_A, a.data_ptr(), s)
            hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, 0, 1, b.data_ptr(), s)
            torch.cuda.synchronize()
            assert a.cpu().tolist() == b.cpu().tolist()  # 0 + x: bitwise the shard result
        assert hpl.hpl_comm_status(comm, s) == (2, 0)
        with pytest.raises(hpl.HPLError) as ei:
            hpl.hpl_comm_open(comm, handle)
        assert ei.value.code == hpl.HPL_ESTATE
    finally:
        hpl.hpl_comm_free(comm)


def _fused_worker(rank, world, port, M, calls, skip_last, ret):
    import sys
    sys.path.insert(0, ROOT)
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", init_method="tcp://127.0.0.1:%d" % port, rank=rank,
                            world_size=world)
    try:
        from paper_conf_ipps_bozkusf12_b200 import hpl, multi
        torch.cuda.set_device(0)
        hpl.hpl_set_device(0)
        comm = multi.FusedComm(torch.device("cuda", 0), timeout_s=20.0)
        res = []
        for _ in range(calls):
            res.append(multi.ep_run_fused(comm, M, NPB_SEED, NPB_A))
        dist.barrier()
        out = {"results": res}
        if skip_last:
            # rank 0 calls once more, its peers do not: the combine must give up
            hpl.hpl_comm_set_timeout(comm.comm, 1.0)
            if rank == 0:
                o = torch.empty(13, dtype=torch.float64, device="cuda")
                comm.run(M, NPB_SEED, NPB_A, o)
                torch.cuda.synchronize()
                out["timeout_word0"] = o[0].item()
                try:
                    comm.status()
                    out["status"] = "ok"
                except hpl.HPLError as e:
                    out["status"] = e.code
            dist.barrier()
        comm.close()
        ret[rank] = out
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.parametrize("world", [2, 4])
def test_fused_processes_share_gpu(hpl, oracle_mod, world):
    import torch
    import torch.multiprocessing as mp
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    M = 22
    ret = mp.Manager().dict()
    mp.spawn(_fused_worker, args=(world, _free_port(), M, 3, world == 2, ret), nprocs=world, join=True)
    ref = oracle_mod.run(M, NPB_SEED, NPB_A, threads=8, margin=False)
    first = ret[0]["results"][0]
    for r in range(world):
        for res in ret[r]["results"]:
            assert res == first  # identical on every rank and every call (rank-order fold)
    assert first["q"] == list(ref.q) and first["gc"] == ref.gc
    assert sums_close(first["sx"], ref.sx, ref.gc) and sums_close(first["sy"], ref.sy, ref.gc)
    if world == 2:
        assert ret[0]["timeout_word0"] != ret[0]["timeout_word0"]  # NaN
        assert ret[0]["status"] == hpl.HPL_ECUDA
