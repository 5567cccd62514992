"""One process per GPU: shard EP by LCG skip-ahead, combine the partials.

SURVEY.md §8(e): rank r of G evaluates pairs [r*2^M/G, (r+1)*2^M/G) with
``hpl_ep_run_shard`` (its kernel jumps the stream to seed*a^(2 r 2^M/G)); the
13-word partials {sx, sy, q0..q9, gc} are combined by a single
``torch.distributed.all_reduce(SUM)`` of 13 float64 (NCCL over NVLink on GPUs;
counts stay exact below 2^53).  The paper runs on one device and names
distributed memory as future work; this is that step for
one NVSwitch box.

Two combines: ``ep_shard_and_reduce`` (kernel, then one NCCL allreduce) and
``FusedComm`` (the EP kernel's last block exchanges the
partials itself over peer memory, ``hpl_ep_run_fused``; torch.distributed only
carries the one-time exchange of the 64-byte IPC handles).

This module is marshalling and plumbing only: the compute is the CUDA kernel
behind ``hpl_ep_run_shard``; ``runner`` exists so the gloo CPU tests can drive
the same plumbing without a GPU.
"""
from __future__ import annotations

from typing import Callable, Optional

import torch
import torch.distributed as dist

from . import hpl

Runner = Callable[[int, int, int, int, int, torch.Tensor], None]


def shard_bounds(M: int, rank: int, nranks: int) -> tuple[int, int]:
    """(first pair, pair count) of shard `rank` — the same rule hpl_ep_run_shard applies."""
    if nranks < 1 or nranks & (nranks - 1) or nranks > (1 << M):
        raise ValueError("nranks must be a power of two <= 2^M")
    if not 0 <= rank < nranks:
        raise ValueError("rank out of range")
    n = (1 << M) // nranks
    return rank * n, n


def gpu_runner(M: int, seed: int, a: int, rank: int, nranks: int, out13: torch.Tensor) -> None:
    """Launch this rank's shard on the current torch stream (asynchronous)."""
    assert out13.is_cuda and out13.dtype == torch.float64 and out13.numel() == 13
    hpl.hpl_ep_run_shard(M, seed, a, rank, nranks, out13.data_ptr(),
                         torch.cuda.current_stream(out13.device).cuda_stream)


def ep_shard_and_reduce(M: int, seed: int, a: int, out13: torch.Tensor,
                        group: Optional[dist.ProcessGroup] = None,
                        runner: Runner = gpu_runner) -> torch.Tensor:
    """Shard of this rank into out13, then allreduce(SUM) across the group."""
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    runner(M, seed, a, rank, world, out13)
    if world > 1:
        dist.all_reduce(out13, op=dist.ReduceOp.SUM, group=group)
    return out13


def ep_run_distributed(M: int, seed: int, a: int, device: Optional[torch.device] = None,
                       group: Optional[dist.ProcessGroup] = None,
                       runner: Runner = gpu_runner) -> dict:
    """Whole EP problem over all ranks; every rank receives the combined result."""
    if device is None:
        device = torch.device("cuda", torch.cuda.current_device()) if runner is gpu_runner \
            else torch.device("cpu")
    out = torch.empty(13, dtype=torch.float64, device=device)
    ep_shard_and_reduce(M, seed, a, out, group, runner)
    words = out.cpu().tolist()  # 104-byte D2H
    if words[0] != words[0]:
        raise hpl.HPLError(hpl.HPL_ERANGE, "ep_run_distributed", "annulus index >= 10")
    return hpl.unpack13(words)


class FusedComm:
    """Peer-memory endpoint for ``hpl_ep_run_fused`` (one per rank and device).

    Construction is collective over ``group``: every rank creates its inbox,
    the 64-byte CUDA IPC handles are all-gathered, and each rank maps its
    peers' inboxes.  Then every rank must call :meth:`run` with the same
    arguments; each call's kernel computes the rank's shard and the combined
    13-word result of the whole problem (identical on all ranks).
    """

    def __init__(self, device: torch.device, group: Optional[dist.ProcessGroup] = None,
                 timeout_s: float = 10.0):
        self.group = group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.device = device
        self.comm, handle = hpl.hpl_comm_create(self.rank, self.world, device.index)
        if self.world > 1:
            backend = dist.get_backend(group)
            on = device if backend == "nccl" else torch.device("cpu")
            mine = torch.tensor(list(handle), dtype=torch.uint8, device=on)
            parts = [torch.empty_like(mine) for _ in range(self.world)]
            dist.all_gather(parts, mine, group=group)
            handles = b"".join(bytes(p.cpu().tolist()) for p in parts)
        else:
            handles = handle
        hpl.hpl_comm_open(self.comm, handles)
        hpl.hpl_comm_set_timeout(self.comm, timeout_s)

    def run(self, M: int, seed: int, a: int, out13: torch.Tensor) -> torch.Tensor:
        """Asynchronous on the current stream of out13's device."""
        assert out13.is_cuda and out13.dtype == torch.float64 and out13.numel() == 13
        hpl.hpl_ep_run_fused(self.comm, M, seed, a, out13.data_ptr(),
                             torch.cuda.current_stream(out13.device).cuda_stream)
        return out13

    def status(self) -> tuple[int, int]:
        return hpl.hpl_comm_status(self.comm, torch.cuda.current_stream(self.device).cuda_stream)

    def close(self) -> None:
        """Collective: every rank drains its own kernels, then a barrier makes
        sure no peer kernel can still be storing into (or reading) any inbox,
        then the mappings and the own inbox are released."""
        if self.comm:
            torch.cuda.synchronize(self.device)
            if self.world > 1 and dist.is_initialized():
                dist.barrier(group=self.group)
            hpl.hpl_comm_free(self.comm)
            self.comm = None


def ep_run_fused(comm: FusedComm, M: int, seed: int, a: int) -> dict:
    """Whole EP problem through the fused combine; host result on every rank."""
    out = torch.empty(13, dtype=torch.float64, device=comm.device)
    comm.run(M, seed, a, out)
    words = out.cpu().tolist()  # 104-byte D2H
    comm.status()
    if words[0] != words[0]:
        raise hpl.HPLError(hpl.HPL_ERANGE, "ep_run_fused", "annulus index >= 10")
    return hpl.unpack13(words)
