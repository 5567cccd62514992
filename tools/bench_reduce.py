"""F2 measurement: hpl_reduce_sum_f32 GB/s vs the measured HBM copy peak.

python tools/bench_reduce.py [--n N ...]   (one JSON line per size)
Inputs are resident in HBM; L2 (126 MB) is flushed between timed launches by
a 256 MB write followed by a 256 MB read of another buffer (so the write's
dirty lines are written back before the timed region, not inside it;
--flush write keeps only the write); CUDA events on the launching stream.  Algorithmic bytes =
4 n (each float read once; the 8-byte result and ~5 KB of partials ignored).
"""
import argparse, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_bozkusf12_b200 import hpl

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, nargs="*", default=[16 << 20, 256 << 20])
ap.add_argument("--iters", type=int, default=10)
ap.add_argument("--flush", choices=["write", "write_read"], default="write_read")
a = ap.parse_args()
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pk = json.load(open(os.path.join(root, "MEASURED_PEAKS.json"))) if os.path.exists(os.path.join(root, "MEASURED_PEAKS.json")) else {}
peak = float(pk.get("hbm_gbs", 6650.0))
torch.cuda.set_device(0); hpl.hpl_set_device(0)
s = torch.cuda.current_stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
flush_rd = torch.ones(64 << 20, dtype=torch.float32, device="cuda")  # 256 MB, read to clean L2
for n in a.n:
    x = torch.randn(n, dtype=torch.float32, device="cuda")
    out = torch.empty(1, dtype=torch.float64, device="cuda")
    for _ in range(3):
        hpl.hpl_reduce_sum_f32(x.data_ptr(), n, out.data_ptr(), s.cuda_stream)
    g = torch.cuda.CUDAGraph()  # graph replay: host call overhead not timed
    gs = torch.cuda.Stream()
    hpl.hpl_reduce_sum_f32(x.data_ptr(), n, out.data_ptr(), gs.cuda_stream)  # per-stream workspace
    torch.cuda.synchronize()
    with torch.cuda.graph(g, stream=gs):
        hpl.hpl_reduce_sum_f32(x.data_ptr(), n, out.data_ptr(), gs.cuda_stream)
    ts = []
    for _ in range(a.iters):
        flush.zero_()
        if a.flush == "write_read":
            flush_rd.sum()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        g.replay()
        e1.record(s); e1.synchronize()
        ts.append(e0.elapsed_time(e1) / 1e3)
    t = sorted(ts)[len(ts) // 2]
    gbs = 4 * n / t / 1e9
    # context: torch's own reduction of the same tensor, same flush and timing
    tt = []
    r = torch.empty((), dtype=torch.float64, device="cuda")
    for _ in range(a.iters):
        flush.zero_()
        if a.flush == "write_read":
            flush_rd.sum()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        torch.sum(x, dim=0, dtype=torch.float64, out=r)
        e1.record(s); e1.synchronize()
        tt.append(e0.elapsed_time(e1) / 1e3)
    t_torch = sorted(tt)[len(tt) // 2]
    tf = []
    rf = torch.empty((), dtype=torch.float32, device="cuda")
    for _ in range(a.iters):
        flush.zero_()
        if a.flush == "write_read":
            flush_rd.sum()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        torch.sum(x, dim=0, out=rf)
        e1.record(s); e1.synchronize()
        tf.append(e0.elapsed_time(e1) / 1e3)
    t_torch32 = sorted(tf)[len(tf) // 2]
    print(json.dumps({"workload": "sum of %d f32 (F2)" % n, "flush": a.flush, "median_s": t, "GB/s": round(gbs, 1),
                      "torch_sum_f64_GB/s": round(4 * n / t_torch / 1e9, 1),
                      "torch_sum_f32_GB/s": round(4 * n / t_torch32 / 1e9, 1),
                      "roofline": {"bound": "hbm", "achieved": round(gbs, 1), "peak": peak, "unit": "GB/s",
                                   "frac": round(gbs / peak, 4), "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy)"},
                      "result": out.item(), "torch_sum_f64": float(x.double().sum())}), flush=True)
