"""Multi-process plumbing of the N>1 path on CPU (gloo, world_size 2 and 4).

The GPU path is: every rank runs hpl_ep_run_shard on its pair range, then one
allreduce(SUM) of the 13-word result (paper_conf_ipps_bozkusf12_b200.multi).
Here the per-rank compute is the oracle (tests may use it) so the sharding
rule, the 13-word packing, the allreduce and the unpacking are exercised
without a GPU; the result must equal the single-process oracle run.
"""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from ep_workloads import NPB_A, NPB_SEED

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _oracle_runner(M, seed, a, rank, nranks, out13):
    import oracle
    from paper_conf_ipps_bozkusf12_b200 import multi
    begin, n = multi.shard_bounds(M, rank, nranks)
    r = oracle.run_pairs(seed, a, begin, n, margin=False)
    out13.copy_(torch.tensor([r.sx, r.sy, *[float(v) for v in r.q], float(r.gc)], dtype=torch.float64))


def _worker(rank, world, port, M, ret):
    import sys
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    dist.init_process_group("gloo", init_method="tcp://127.0.0.1:%d" % port, rank=rank,
                            world_size=world)
    from paper_conf_ipps_bozkusf12_b200 import multi
    res = multi.ep_run_distributed(M, NPB_SEED, NPB_A, device=torch.device("cpu"),
                                   runner=_oracle_runner)
    ret[rank] = res
    dist.barrier()
    dist.destroy_process_group()


@pytest.fixture(scope="module", autouse=True)
def _built():
    from paper_conf_ipps_bozkusf12_b200 import build
    build.build()
    import oracle
    oracle.build()


@pytest.mark.parametrize("world", [2, 4])
def test_gloo_shards_allreduce_equals_single_run(world, oracle_mod):
    M = 18
    mgr = mp.Manager()
    ret = mgr.dict()
    mp.spawn(_worker, args=(world, _free_port(), M, ret), nprocs=world, join=True)
    ref = oracle_mod.run(M, NPB_SEED, NPB_A, margin=False)
    for rank in range(world):
        r = ret[rank]
        assert r["q"] == ref.q and r["gc"] == ref.gc
        assert abs(r["sx"] - ref.sx) <= 1e-12 * max(abs(ref.sx), ref.gc ** 0.5)
        assert abs(r["sy"] - ref.sy) <= 1e-12 * max(abs(ref.sy), ref.gc ** 0.5)


def test_shard_bounds_partition():
    from paper_conf_ipps_bozkusf12_b200 import multi
    for M in (0, 3, 20, 36):
        for n in (1, 2, 4, 8):
            if n > (1 << M):
                continue
            spans = [multi.shard_bounds(M, r, n) for r in range(n)]
            assert spans[0][0] == 0
            assert all(spans[i][0] + spans[i][1] == spans[i + 1][0] for i in range(n - 1))
            assert spans[-1][0] + spans[-1][1] == 1 << M
    with pytest.raises(ValueError):
        multi.shard_bounds(10, 0, 3)
    with pytest.raises(ValueError):
        multi.shard_bounds(1, 0, 4)
