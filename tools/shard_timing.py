"""Per-shard device time of the EP kernel, i.e. what each of N GPUs runs (dev aid).

python tools/shard_timing.py   (one JSON line per class and N)
For class B, C, D and N = 1, 2, 4, 8 the kernel of shard r of N (r = 0 and
N - 1) is timed alone on this GPU with CUDA events (min of 3 after a warm-up).
Ranks run on separate GPUs, so a step at N GPUs takes the slowest shard plus
the 104-byte combine; the ratio T(1) / max_r T(shard r of N) is the kernel's
strong-scaling ceiling (the driver measures the real multi-GPU number).
Also times every NPB class on one GPU (the whole problem).
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_bozkusf12_b200 import hpl
from ep_workloads import CLASSES, NPB_A, NPB_SEED

torch.cuda.set_device(0); hpl.hpl_set_device(0)
s = torch.cuda.current_stream()
out = torch.empty(13, dtype=torch.float64, device="cuda")


def t_shard(M, r, n, reps=3):
    hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, r, n, out.data_ptr(), s.cuda_stream)
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, r, n, out.data_ptr(), s.cuda_stream)
        e1.record(s); e1.synchronize()
        ts.append(e0.elapsed_time(e1) / 1e3)
    return min(ts)


for cls in ("S", "W", "A", "B", "C", "D", "E"):
    M = CLASSES[cls]
    t = t_shard(M, 0, 1, reps=1 if M >= 40 else 3)
    print(json.dumps({"class": cls, "M": M, "gpus": 1, "s": round(t, 6), "Mops": round((2 << M) / t / 1e6, 1),
                      "gc": int(out[12].item())}), flush=True)
for cls in ("B", "C", "D"):
    M = CLASSES[cls]
    t1 = t_shard(M, 0, 1)
    for n in (2, 4, 8):
        tr = [t_shard(M, r, n) for r in (0, n - 1)]
        print(json.dumps({"class": cls, "M": M, "gpus": n, "shard_s": [round(x, 6) for x in tr],
                          "t1_s": round(t1, 6), "ceiling_speedup": round(t1 / max(tr), 3)}), flush=True)
