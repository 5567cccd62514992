import sys, os, time, json
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_ipps_bozkusf12_b200 import hpl
from ep_workloads import NPB_A, NPB_SEED
torch.cuda.set_device(0); hpl.hpl_set_device(0)
s = torch.cuda.current_stream()
out = torch.empty(13, dtype=torch.float64, device="cuda")
for M in (0, 10, 16, 20, 24):
    for _ in range(3): hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, 0, 1, out.data_ptr(), s.cuda_stream)
    torch.cuda.synchronize()
    # host time per call
    t0 = time.perf_counter()
    for _ in range(100): hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, 0, 1, out.data_ptr(), s.cuda_stream)
    torch.cuda.synchronize()
    th = (time.perf_counter() - t0) / 100
    # graph-replayed device time
    g = torch.cuda.CUDAGraph(); gs = torch.cuda.Stream()
    hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, 0, 1, out.data_ptr(), gs.cuda_stream); torch.cuda.synchronize()
    with torch.cuda.graph(g, stream=gs):
        hpl.hpl_ep_run_shard(M, NPB_SEED, NPB_A, 0, 1, out.data_ptr(), gs.cuda_stream)
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(100): g.replay()
    e1.record(s); e1.synchronize()
    print(json.dumps({"M": M, "host_us_per_call": round(th * 1e6, 1), "graph_device_us": round(e0.elapsed_time(e1) * 10, 2)}))
