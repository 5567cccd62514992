"""A9 across real devices: one process per GPU, both combines.

Runs only when at least two CUDA devices are visible (the driver's scaling
runs on an 8-GPU node; this session's gpurun boxes have one GPU, where these
tests skip).  For world = 2, 4, 8 (as many as fit) each rank r drives
cuda:r over an NCCL process group and runs classes B and C, plus class D at
the largest world, through
  * the NCCL combine (kernel, then all_reduce of the 13 words), and
  * the fused combine (hpl_ep_run_fused: peer stores over NVLink, no
    collective launch),
three consecutive calls each (both inbox parities of the fused path).
Checked on every rank: q and gc exactly equal to the oracle goldens
(tests/golden/oracle_ep.json, written by oracle/ only) and to NPB's published
counts, sx/sy within tolerance T1 of the oracle and within 1e-8 of NPB's
verification sums, the fused result identical on all ranks and calls.
"""
import os
import socket

import pytest

from _golden import npb_verify, oracle_golden, sums_close
from ep_workloads import CLASSES, NPB_A, NPB_SEED

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu


def _ndev():
    import torch
    return torch.cuda.device_count() if torch.cuda.is_available() else 0


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, classes, ret):
    import sys
    sys.path.insert(0, ROOT)
    import torch
    import torch.distributed as dist
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", init_method="tcp://127.0.0.1:%d" % port, rank=rank, world_size=world,
                            device_id=torch.device("cuda", rank))
    try:
        from paper_conf_ipps_bozkusf12_b200 import hpl, multi
        hpl.hpl_set_device(rank)
        dev = torch.device("cuda", rank)
        out = {}
        comm = multi.FusedComm(dev, timeout_s=30.0)
        try:
            for cls in classes:
                M = CLASSES[cls]
                out[(cls, "nccl")] = [multi.ep_run_distributed(M, NPB_SEED, NPB_A, dev) for _ in range(3)]
                out[(cls, "fused")] = [multi.ep_run_fused(comm, M, NPB_SEED, NPB_A) for _ in range(3)]
                out[(cls, "fused_status")] = comm.status()
        finally:
            comm.close()
        ret[rank] = out
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4, 8])
def test_combines_across_devices(world):
    n = _ndev()
    if n < 2:
        pytest.skip("needs >= 2 CUDA devices (found %d)" % n)
    if world > n:
        pytest.skip("world %d > %d devices" % (world, n))
    import torch.multiprocessing as mp
    classes = ["B", "C"] + (["D"] if world == min(8, n) or world == 8 else [])
    ret = mp.Manager().dict()
    mp.spawn(_worker, args=(world, _free_port(), classes, ret), nprocs=world, join=True)
    gold, npb = oracle_golden(), npb_verify()
    for cls in classes:
        g = gold[cls]
        fused0 = ret[0][(cls, "fused")][0]
        for r in range(world):
            assert ret[r][(cls, "fused_status")] == (3 * (classes.index(cls) + 1), 0)
            for how in ("nccl", "fused"):
                for res in ret[r][(cls, how)]:
                    assert res["q"] == g["q"] and res["gc"] == g["gc"], (cls, how, r)
                    assert sums_close(res["sx"], g["sx"], g["gc"]) and sums_close(res["sy"], g["sy"], g["gc"])
                    _, sxr, syr = npb[cls]
                    assert abs(res["sx"] - sxr) <= 1e-8 * abs(sxr) and abs(res["sy"] - syr) <= 1e-8 * abs(syr)
            for res in ret[r][(cls, "fused")]:
                assert res == fused0  # rank-order fold: bitwise identical everywhere
