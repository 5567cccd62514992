"""Fixed cost per EP launch (dev aid): class S/W/B-shard times by CUDA events,
plain launches and CUDA-graph replays (min over reps), for the library in HPL_LIB.

python tools/fixed_cost.py [M,...]
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_bozkusf12_b200 import hpl
from ep_workloads import NPB_A, NPB_SEED

Ms = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "10,20,24,25,27").split(",")]
torch.cuda.set_device(0); hpl.hpl_set_device(0)
s = torch.cuda.Stream()
out = torch.empty(13, dtype=torch.float64, device="cuda")
tag = os.path.basename(os.environ.get("HPL_LIB", "default"))


def ev_time(fn, reps=20):
    ts = []
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s); fn(); e1.record(s); e1.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    return ts[0], ts[len(ts) // 2]


with torch.cuda.stream(s):
    for M in Ms:
        n = 1 << M
        # M=27 stands for one class-B shard of 8 (2^27 pairs at offset 7 * 2^27)
        run = lambda: hpl.hpl_ep_run_range(NPB_SEED, NPB_A, (7 << 27) if M == 27 else 0, n, out.data_ptr(), s.cuda_stream)
        run(); torch.cuda.synchronize()
        mn, md = ev_time(run)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            run()
        g.replay(); torch.cuda.synchronize()
        gmn, gmd = ev_time(g.replay)
        # 10 replays back to back: per-launch time without the per-event gap
        g10 = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g10, stream=s):
            for _ in range(10):
                run()
        g10.replay(); torch.cuda.synchronize()
        b_mn, _ = ev_time(g10.replay, reps=5)
        print(json.dumps({"lib": tag, "M": M, "pairs": n, "us_min": round(mn, 2), "us_med": round(md, 2),
                          "graph_us_min": round(gmn, 2), "graph10_us_per": round(b_mn / 10, 2),
                          "Mops_graph10": round(2 * n / (b_mn / 10) / 1e6, 1), "gc": int(out[12].item())}), flush=True)
