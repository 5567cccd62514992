#!/usr/bin/env python
"""Benchmark: NPB EP Mops/s (2^(M+1) uniforms / s) on 1..8 B200 (BASELINE.json).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...        (N > 1, one rank per GPU)

A step = one whole EP problem of class D (M = 36, 2^37 uniforms; the
BASELINE.json headline config) split over the N ranks: each rank runs its
shard kernel; for N > 1 the 13-word partials are combined inside that kernel
over peer memory (--combine fused, hpl_ep_run_fused, the default) or by one
NCCL allreduce after it (--combine nccl).
EP reads no input arrays (only the (M, seed, a) scalars and a 368-B jump table
passed as kernel parameters), so "resident in HBM" is vacuous; L2 is flushed
between timed steps anyway.  Device time: CUDA events per step on the
launching stream, barrier + synchronize around the timed region, max over
ranks.  e2e: the same metric through the public API with host results
(hpl_ep_run / ep_run_distributed incl. the 104-B D2H), wall clock.

--impl reference: the CPU oracle (oracle/, plain NPB EP) on the box's host
cores over a bounded sample of the same workload — the baseline arm.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from ep_workloads import CLASSES, HEADLINE_CLASS, NPB_A, NPB_SEED, uniforms  # noqa: E402

METRIC = "EP Mops/s (2^(M+1)/s) at 1/2/4/8 B200; fraction of FP64 peak"
UNIT = "Mops/s"
PAPER_CONTEXT = {"class": "C", "mops": 3057, "hw": "Tesla C2050/C2070, OpenCL, 2.81 s (PAPER.md:940-942)"}

# Algorithmic FP64 lane-operations per pair: 6 always
# (2 maps, 2 squares, 1 add, 1 compare) + pi/4 * 19 for accepted pairs
# (ln 6, sqrt(L/t) 7, X and Y 2, max 1, sums 2) -- ln: r, 4 Horner, reconstruction (K=9 table).
ALG_OPS_ALWAYS = 6
ALG_OPS_ACCEPTED = 18
P_ACCEPT = 0.7853981633974483
ALG_OPS_PER_PAIR = ALG_OPS_ALWAYS + P_ACCEPT * ALG_OPS_ACCEPTED
# algorithmic-fraction ceiling of the minimal instruction mix (DESIGN.md §5,
# profiles/r02_ceiling.md): 2 / (1.93 + 1.03 * 0.72) of the FP64 pipe x 20.137 / 20
CEILING_FRAC = 0.754
EXEC_FP64_PER_PAIR = 20             # SASS of the hot loop (tools/sass_hot.py): DFMA 10 + DMUL 6 + DADD 4
FP64_LANES_PER_SM_CLK = 64          # measured: tools/probe_fp64.cu (63.9-64.1 lane-DFMA/clk/SM)
EP_PARAM_BYTES = 560                 # EPParams kernel-parameter block (jump table, a^k table, coefs, scalars)


def peaks():
    p = {}
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        p = json.load(open(path))
    return p


def load_profile_field(key):
    """One field of the committed ncu summary of the EP kernel, or None."""
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        return json.load(open(path)).get(key)
    except Exception:
        return None


def load_profile_traffic():
    """dram bytes per launch of the EP kernel from the committed ncu summary, or None."""
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if not os.path.exists(path):
        return None
    try:
        return json.load(open(path)).get("dram_bytes_per_launch")
    except Exception:
        return None


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.sw_power_cap,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None
        self.t0 = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=" + self.FIELDS,
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) == 7:
                self.rows.append((time.time(), parts))

    def mark(self):
        """Start of the timed region: nvidia-smi was started before the
        warm-up (its NVML start-up would otherwise land in the first timed
        step), and only samples from here on count."""
        self.t0 = time.time()

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        rows = [r for t, r in self.rows if self.t0 is None or t >= self.t0] or [r for _, r in self.rows]
        names = ["sw_power_cap", "hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"]
        sm = [float(r[0]) for r in rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        pw = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        active = sorted({names[i] for r in rows for i in range(4) if r[3 + i].lower().startswith("active")})
        loaded = [s for s in sm if mx and s > 0.5 * max(mx)] or sm
        return {"sm_mhz": statistics.median(loaded) if loaded else None,
                "sm_max_mhz": max(mx) if mx else None,
                "power_w_max": max(pw) if pw else None,
                "samples": len(rows), "reasons": active}


# --------------------------------------------------------------- reference
def run_reference(args, M):
    import oracle
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    threads = os.cpu_count() or 1
    nb_total = 1 << (M - 16)
    # bounded sample: `batches` NPB batches (2^16 pairs each) per step
    batches = min(nb_total, args.ref_batches or 64 * threads)
    for _ in range(args.warmup):
        oracle.run_batches(M, NPB_SEED, NPB_A, 0, min(batches, threads), threads=threads, margin=False)
    ts = []
    for s in range(args.steps):
        k0 = (s * batches) % max(nb_total - batches + 1, 1)
        t0 = time.perf_counter()
        oracle.run_batches(M, NPB_SEED, NPB_A, k0, k0 + batches, threads=threads, margin=False)
        ts.append(time.perf_counter() - t0)
    pairs = batches << 16
    tot = sum(ts)
    value = 2 * pairs * args.steps / tot / 1e6
    sample = ("NPB batches [k0, k0+%d) of class %s (2^16 pairs each, %d uniforms per step), "
              "batch-parallel over %d threads, margin tracking off" % (batches, args.cls, 2 * pairs, threads))
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 3), "unit": UNIT,
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(tot / args.steps * 1e3, 3), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic (NPB LCG stream)",
        "config": {"workload": "NPB EP class %s (M=%d)" % (args.cls, M), "M": M, "seed": NPB_SEED,
                   "a": NPB_A, "sampled": True},
        "cpu_baseline": {"value": round(value, 3), "unit": UNIT, "cores": threads, "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": round(value, 3), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def verify_result(cls, M, result, world):
    """Correctness gate of the measured run: the
    printed result against NPB's published verification sums (relative 1e-8,
    ep.f's epsilon) and, where a stored oracle result exists for the class
    (tests/golden/oracle_ep.json, written by a script that calls only oracle/;
    or NPB's reference counts for S/W/A), q[] and gc exactly and sx, sy within
    T1 = 1e-12 * max(|ref|, sqrt(gc)).  Returns the "verified" record."""
    gdir = os.path.join(ROOT, "tests", "golden")
    checks, ok = [], True
    sx, sy, q, gc = result["sx"], result["sy"], result["q"], result["gc"]
    if not (sx == sx and sy == sy) or sum(q) != gc:
        return {"ok": False, "checks": ["result is NaN or sum(q) != gc (combine failed?)"]}
    for line in open(os.path.join(gdir, "npb_ep_verify.txt")):
        f = line.split()
        if f and not f[0].startswith("#") and f[0] == cls:
            good = abs((sx - float(f[2])) / float(f[2])) <= 1e-8 and abs((sy - float(f[3])) / float(f[3])) <= 1e-8
            checks.append("NPB verification sums (1e-8): %s" % ("pass" if good else "FAIL"))
            ok &= good
    gold = json.load(open(os.path.join(gdir, "oracle_ep.json"))).get(cls)
    if gold is not None:
        rs, ry = float.fromhex(gold["sx"]), float.fromhex(gold["sy"])
        tol = 1e-12 * max(abs(rs), abs(ry), gold["gc"] ** 0.5)
        good = q == gold["q"] and gc == gold["gc"]
        checks.append("q, gc exact vs oracle golden: %s" % ("pass" if good else "FAIL"))
        ok &= good
        good = abs(sx - rs) <= 1e-12 * max(abs(rs), gold["gc"] ** 0.5) and \
            abs(sy - ry) <= 1e-12 * max(abs(ry), gold["gc"] ** 0.5)
        checks.append("sx, sy within 1e-12*max(|ref|, sqrt(gc)) of oracle golden: %s (|d| %.2e, %.2e; tol %.2e)"
                      % ("pass" if good else "FAIL", abs(sx - rs), abs(sy - ry), tol))
        ok &= good
    else:
        for line in open(os.path.join(gdir, "npb_ep_counts.txt")):
            f = line.split()
            if f and not f[0].startswith("#") and f[0] == cls:
                good = gc == int(f[2]) and q[:7] == [int(v) for v in f[3:10]]
                checks.append("q, gc exact vs NPB reference counts: %s" % ("pass" if good else "FAIL"))
                ok &= good
    if not checks:
        checks.append("no stored reference for class %s" % cls)
    return {"ok": bool(ok), "world": world, "checks": checks}


def cpu_baseline_sample(M, budget_s, single_s=6.0):
    """Oracle as it stands on the host cores over a bounded sample of class M,
    and (the paper's serial-CPU baseline) the
    same oracle on ONE core over a smaller sample."""
    import oracle
    t0 = time.perf_counter()
    oracle.run_batches(M, NPB_SEED, NPB_A, 0, 1, threads=1, margin=False)
    t_b = max(time.perf_counter() - t0, 1e-3)
    nb1 = max(1, min(int(single_s / t_b), 1 << (M - 16)))
    t0 = time.perf_counter()
    oracle.run_batches(M, NPB_SEED, NPB_A, 0, nb1, threads=1, margin=False)
    dt1 = time.perf_counter() - t0
    single = {"value": round(2 * (nb1 << 16) / dt1 / 1e6, 3), "unit": UNIT, "cores": 1,
              "sample": "first %d NPB batches (%d pairs, %.1f s), one thread" % (nb1, nb1 << 16, dt1)}
    threads = os.cpu_count() or 1
    t0 = time.perf_counter()
    oracle.run_batches(M, NPB_SEED, NPB_A, 0, threads, threads=threads, margin=False)
    t_one = max(time.perf_counter() - t0, 1e-3)  # one batch per thread
    batches = max(threads, int(budget_s / t_one) * threads)
    batches = min(batches, 1 << (M - 16))
    t0 = time.perf_counter()
    oracle.run_batches(M, NPB_SEED, NPB_A, 0, batches, threads=threads, margin=False)
    dt = time.perf_counter() - t0
    pairs = batches << 16
    return {"value": round(2 * pairs / dt / 1e6, 3), "unit": UNIT, "cores": threads, "kind": "oracle",
            "sample": "first %d NPB batches of class-%d stream (%d pairs, %.1f s), batch-parallel over "
                      "%d threads, margin tracking off" % (batches, M, pairs, dt, threads),
            "single_core": single}


# --------------------------------------------------------------------- ours
def run_ours(args, M):
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_bozkusf12_b200 import hpl, multi

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit("--gpus %d but WORLD_SIZE=%d (launch with torchrun for N>1)" % (args.gpus, world))
    # one rank per GPU; --dist-backend gloo lets several ranks share one GPU
    # (code-path test on a 1-GPU box, never a performance number)
    gpu = local % max(torch.cuda.device_count(), 1) if args.dist_backend == "gloo" else local
    torch.cuda.set_device(gpu)
    hpl.hpl_set_device(gpu)
    dev = torch.device("cuda", gpu)
    if world > 1:
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
    stream = torch.cuda.current_stream(dev)
    out = torch.empty(13, dtype=torch.float64, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)  # > 126 MB L2

    # N > 1 combine: "fused" = the kernel's last block exchanges the 13-word
    # partials over peer memory (hpl_ep_run_fused); "nccl" = kernel
    # then one all_reduce.  fused falls back to nccl if peer mapping fails.
    combine, combine_note, fc = ("none" if world == 1 else args.combine), None, None
    if combine == "fused":
        try:
            fc = multi.FusedComm(dev)
        except Exception as e:  # e.g. no CUDA IPC / peer access between these GPUs
            combine, combine_note = "nccl", "fused unavailable: %s" % str(e)[:200]
        if world > 1:  # every rank must agree on the combine
            flag = torch.tensor([1.0 if combine == "fused" else 0.0], device=dev)
            dist.all_reduce(flag, op=dist.ReduceOp.MIN)
            if flag.item() == 0.0 and combine == "fused":
                combine, combine_note = "nccl", "fused unavailable on a peer rank"

    def step():
        if combine == "fused":
            fc.run(M, NPB_SEED, NPB_A, out)
        else:
            hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, rank, world, out.data_ptr(), stream.cuda_stream)

    sampler = ClockSampler(gpu)
    sampler.start()
    for _ in range(args.warmup):
        step()
        if combine == "nccl":
            dist.all_reduce(out)
    torch.cuda.synchronize(dev)
    if combine == "fused":
        # the first multi-GPU execution of the peer-memory combine is here: if a
        # warm-up call timed out, tore a slot or produced a result that fails
        # verification on any rank, every rank switches to the NCCL combine
        # (agreed over NCCL, which does not depend on the fused path)
        try:
            fc.status()
            ok = verify_result(args.cls, M, hpl.unpack13(out.cpu().tolist()), world)["ok"]
            why = "warm-up result failed verification"
        except hpl.HPLError as e:
            ok, why = False, "warm-up combine failed: %s" % str(e)[:160]
        flag = torch.tensor([1.0 if ok else 0.0], device=dev)
        dist.all_reduce(flag, op=dist.ReduceOp.MIN)
        if flag.item() == 0.0:
            combine = "nccl"
            combine_note = why if not ok else "fused combine failed on a peer rank"
            for _ in range(max(args.warmup, 1)):
                step()
                dist.all_reduce(out)
            torch.cuda.synchronize(dev)

    # ---- device-timed region
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    sampler.mark()
    launches0 = hpl.hpl_ep_launch_count()
    step_ms, kern_ms = [], []
    for _ in range(args.steps):
        flush.zero_()  # untimed L2 flush between steps
        e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        e0.record(stream)
        step()
        e1.record(stream)
        if combine == "nccl":
            dist.all_reduce(out)
        e2.record(stream)
        e2.synchronize()
        kern_ms.append(e0.elapsed_time(e1))
        step_ms.append(e0.elapsed_time(e2))
    torch.cuda.synchronize(dev)
    launches = hpl.hpl_ep_launch_count() - launches0
    if world > 1:
        dist.barrier()
    clocks = sampler.stop()
    result = hpl.unpack13(out.cpu().tolist())
    combine_failures = 0
    if combine == "fused":
        try:
            fc.status()  # every timed combine completed (no timeout / torn slot)
        except hpl.HPLError:
            combine_failures = 1
    verified = verify_result(args.cls, M, result, world)
    if combine_failures:
        verified["ok"] = False
        verified["checks"].append("fused combine reported a failed call")

    total_ms = sum(step_ms)
    t = torch.tensor([total_ms, sum(kern_ms), float(launches)], dtype=torch.float64, device=dev)
    if world > 1:
        tmax = t.clone()
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
        tsum = t.clone()
        dist.all_reduce(tsum, op=dist.ReduceOp.SUM)
        total_ms, kern_max_ms, launches_all = tmax[0].item(), tmax[1].item(), int(tsum[2].item())
    else:
        kern_max_ms, launches_all = sum(kern_ms), launches

    # ---- e2e through the public API (host results); one untimed call first
    # (like the device warm-up: it allocates the API's cached pinned result buffer)
    e2e_ms = []
    if world == 1:
        hpl.hpl_ep_run(M, NPB_SEED, NPB_A)
    elif combine == "fused":
        multi.ep_run_fused(fc, M, NPB_SEED, NPB_A)
    else:
        multi.ep_run_distributed(M, NPB_SEED, NPB_A, device=dev)
    if world > 1:
        dist.barrier()
    for _ in range(args.steps):
        t0 = time.perf_counter()
        if world == 1:
            sx, sy, q = hpl.hpl_ep_run(M, NPB_SEED, NPB_A)  # blocking, 104-B D2H inside
        elif combine == "fused":
            multi.ep_run_fused(fc, M, NPB_SEED, NPB_A)
        else:
            multi.ep_run_distributed(M, NPB_SEED, NPB_A, device=dev)
        e2e_ms.append((time.perf_counter() - t0) * 1e3)
    e2e_tot = sum(e2e_ms)
    if combine == "fused":
        fc.status()
    if world == 1:
        e2e_res = {"sx": sx, "sy": sy, "q": q, "gc": sum(q)}
        v2 = verify_result(args.cls, M, e2e_res, world)
        if not v2["ok"]:
            verified["ok"] = False
            verified["checks"].append("e2e (hpl_ep_run) result: " + "; ".join(v2["checks"]))
    if world > 1:
        te = torch.tensor([e2e_tot], dtype=torch.float64, device=dev)
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
        e2e_tot = te.item()

    if rank == 0:
        units = uniforms(M)
        value = units * args.steps / (total_ms / 1e3) / 1e6
        # roofline of the dominant (only) kernel: algorithmic FP64 lane-ops per launch
        pk = peaks()
        sm_max = float(pk.get("sm_max_mhz", 1965.0))
        props = torch.cuda.get_device_properties(dev)
        peak_ops = props.multi_processor_count * FP64_LANES_PER_SM_CLK * sm_max * 1e6
        pairs_per_launch = (1 << M) // world
        kern_avg_s = kern_max_ms / args.steps / 1e3
        achieved = ALG_OPS_PER_PAIR * pairs_per_launch / kern_avg_s
        traffic = load_profile_traffic()
        per_step = sorted(units / (ms / 1e3) / 1e6 for ms in step_ms)  # rank 0's steps
        line = {
            "metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": world,
            "value_stats": {"median": round(statistics.median(per_step), 1), "min": round(per_step[0], 1),
                            "max": round(per_step[-1], 1), "steps": len(per_step),
                            "note": "per-step Mops/s (rank 0); value = all steps / their total time"},
            "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(total_ms / args.steps, 4), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (NPB LCG stream, seed 271828183, a=5^13)",
            "config": {"workload": "NPB EP class %s (M=%d)" % (args.cls, M), "M": M,
                       "global_pairs": 1 << M, "seed": NPB_SEED, "a": NPB_A,
                       "parallelism": ("1 GPU" if world == 1 else
                                       "shard x%d + in-kernel combine (peer stores)" % world
                                       if combine == "fused" else
                                       "shard x%d + allreduce(13 x f64)" % world),
                       "combine": combine if combine_note is None else "%s (%s)" % (combine, combine_note),
                       "l2": "flushed (256 MB write) between timed steps; EP reads no inputs",
                       "kernel_shape": list(hpl.hpl_ep_launch_shape(pairs_per_launch))},
            "paper_context": PAPER_CONTEXT,
            "roofline": {"bound": "alu", "achieved": round(achieved / 1e12, 3),
                         "peak": round(peak_ops / 1e12, 3), "unit": "FP64 Tops/s (lane-ops)",
                         "frac": round(achieved / peak_ops, 4), "traffic": traffic,
                         "alg_ops_per_pair": round(ALG_OPS_PER_PAIR, 3),
                         "peak_basis": "%d SMs x %d FP64 lanes/clk x %.0f MHz (sm_max_mhz)"
                                       % (props.multi_processor_count, FP64_LANES_PER_SM_CLK, sm_max),
                         "kernel_ms": round(kern_avg_s * 1e3, 4),
                         # the FP64-issue view: FP64 instructions the kernel
                         # executes per pair (every pair runs the transform) / peak
                         "executed_fp64_per_pair": EXEC_FP64_PER_PAIR,
                         "fp64_pipe_frac": round(achieved / peak_ops * EXEC_FP64_PER_PAIR / ALG_OPS_PER_PAIR, 4),
                         "ncu_fp64_pipe_active_pct": load_profile_field("fp64_pipe_active_pct"),
                         # counter-backed ceiling of this instruction mix (profiles/r02_ceiling.md):
                         # cycles/FP64 instr = 1.93 + 1.03 rho, rho >= 0.72 non-FP64 instr per FP64
                         "instruction_mix_ceiling_frac": CEILING_FRAC,
                         "frac_of_ceiling": round(achieved / peak_ops / CEILING_FRAC, 4)},
            "e2e": {"value": round(units * args.steps / (e2e_tot / 1e3) / 1e6, 1), "unit": UNIT,
                    "h2d_bytes_per_step": EP_PARAM_BYTES * world, "d2h_bytes_per_step": 104 * world,
                    "note": "h2d = kernel-parameter block (jump table + scalars); d2h = 13-word result"},
            "gpu_launches": launches_all,
            "clocks": clocks,
            "dist_backend": args.dist_backend if world > 1 else None,
            "result": {"sx": result["sx"], "sy": result["sy"], "gc": result["gc"], "q": result["q"]},
            "verified": verified["ok"],
            "verification": verified["checks"],
        }
        if not args.no_cpu_baseline and world == 1:
            line["cpu_baseline"] = cpu_baseline_sample(M, args.cpu_budget)
        print(json.dumps(line), flush=True)
    if fc is not None:
        fc.close()
    ok = torch.tensor([1.0 if verified["ok"] else 0.0], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(ok, op=dist.ReduceOp.MIN)
        dist.barrier()
        dist.destroy_process_group()
    if ok.item() != 1.0:
        sys.stderr.write("bench: result verification FAILED: %s\n" % "; ".join(verified["checks"]))
        return 3
    return 0


def main():
    ap = argparse.ArgumentParser(description=__doc__, formatter_class=argparse.RawDescriptionHelpFormatter)
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--cls", default=HEADLINE_CLASS, choices=sorted(CLASSES))
    ap.add_argument("--cpu-budget", type=float, default=15.0, help="seconds of oracle work for cpu_baseline")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--ref-batches", type=int, default=0, help="NPB batches per --impl reference step")
    ap.add_argument("--combine", choices=["fused", "nccl"], default="fused",
                    help="N>1: in-kernel peer-memory combine (default) or kernel + NCCL all_reduce")
    ap.add_argument("--dist-backend", choices=["nccl", "gloo"], default="nccl",
                    help="gloo only to exercise the N>1 code path with several ranks on one GPU")
    args = ap.parse_args()
    if args.warmup < 3:
        ap.error("--warmup must be >= 3")
    M = CLASSES[args.cls]
    if args.impl == "reference":
        return run_reference(args, M)
    return run_ours(args, M)


if __name__ == "__main__":
    sys.exit(main())
