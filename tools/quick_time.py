"""Quick device timing of the EP kernel per class/variant (development aid)."""
import sys, os, time, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_bozkusf12_b200 import hpl
from ep_workloads import NPB_A, NPB_SEED

torch.cuda.set_device(0); hpl.hpl_set_device(0)
s = torch.cuda.current_stream()
out = torch.empty(13, dtype=torch.float64, device="cuda")
args = sys.argv[1:] or ["30", "32", "36"]
for variant in (0, 1):
    for thr, bps in [(0, 0), (256, 0), (1024, 0)]:
        hpl.hpl_ep_set_config(variant, thr, bps)
        for M in map(int, args):
            shape = hpl.hpl_ep_launch_shape(1 << M)
            hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, 0, 1, out.data_ptr(), s.cuda_stream)
            torch.cuda.synchronize()
            ts = []
            for _ in range(3):
                e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
                e0.record(s)
                hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, 0, 1, out.data_ptr(), s.cuda_stream)
                e1.record(s); e1.synchronize()
                ts.append(e0.elapsed_time(e1) / 1e3)
            t = min(ts)
            print(json.dumps({"variant": variant, "M": M, "shape": shape, "s": round(t, 6),
                              "Mops": round((2 << M) / t / 1e6, 1)}), flush=True)
