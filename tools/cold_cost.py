"""Per-launch device time of small EP launches with a cold L2 (bench.py's
setting: a 256 MB write before each launch) vs warm back-to-back launches
(dev aid).  python tools/cold_cost.py [M,...]  (library from HPL_LIB)"""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_bozkusf12_b200 import hpl
from ep_workloads import NPB_A, NPB_SEED

Ms = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "10,24,27").split(",")]
torch.cuda.set_device(0); hpl.hpl_set_device(0)
s = torch.cuda.current_stream()
out = torch.empty(13, dtype=torch.float64, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
tag = os.path.basename(os.environ.get("HPL_LIB", "default"))
for M in Ms:
    run = lambda: hpl.hpl_ep_run_range(NPB_SEED, NPB_A, 0, 1 << M, out.data_ptr(), s.cuda_stream)
    for _ in range(3):
        run()
    res = {}
    for mode in ("cold", "warm"):
        ts = []
        for _ in range(20):
            if mode == "cold":
                flush.zero_()
            else:
                run()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(s); run(); e1.record(s); e1.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e3)
        res[mode] = round(statistics.median(ts), 2)
    print(json.dumps({"lib": tag, "M": M, "cold_us": res["cold"], "warm_us": res["warm"]}), flush=True)
