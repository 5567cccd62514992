"""Quick device timing of the EP kernel per class / variant / block size (development aid).

python tools/quick_time.py M [M...] [--variants 0,1] [--threads 0,256,...] [--bps 0,...]
"""
import argparse, sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_bozkusf12_b200 import hpl
from ep_workloads import NPB_A, NPB_SEED

ap = argparse.ArgumentParser()
ap.add_argument("M", nargs="*", type=int, default=[32, 36])
ap.add_argument("--variants", default="0")
ap.add_argument("--threads", default="0")
ap.add_argument("--bps", default="0")
ap.add_argument("--reps", type=int, default=3)
a = ap.parse_args()
torch.cuda.set_device(0); hpl.hpl_set_device(0)
s = torch.cuda.current_stream()
out = torch.empty(13, dtype=torch.float64, device="cuda")
for variant in map(int, a.variants.split(",")):
    for thr in map(int, a.threads.split(",")):
        for bps in map(int, a.bps.split(",")):
            hpl.hpl_ep_set_config(variant, thr, bps)
            for M in a.M:
                shape = hpl.hpl_ep_launch_shape(1 << M)
                hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, 0, 1, out.data_ptr(), s.cuda_stream)
                torch.cuda.synchronize()
                ts = []
                for _ in range(a.reps):
                    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
                    e0.record(s)
                    hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, 0, 1, out.data_ptr(), s.cuda_stream)
                    e1.record(s); e1.synchronize()
                    ts.append(e0.elapsed_time(e1) / 1e3)
                t = min(ts)
                print(json.dumps({"variant": variant, "thr": thr, "bps": bps, "M": M, "shape": shape,
                                  "s": round(t, 6), "Mops": round((2 << M) / t / 1e6, 1),
                                  "gc": int(out[12].item()), "sx": out[0].item(), "sy": out[1].item()}), flush=True)
