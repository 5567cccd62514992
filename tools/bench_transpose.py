"""F4 measurement: hpl_transpose_f32 GB/s vs the measured HBM copy peak.

python tools/bench_transpose.py [--n N ...] [--lib PATH]   (one JSON line per size)
The paper's size is 16K x 16K float32 (1 GiB in, 1 GiB out,
both far above the 126 MB L2).  Inputs resident in HBM; L2 flushed between
timed launches (256 MB write + 256 MB read of other buffers); CUDA events on
the launching stream around a CUDA-graph replay of one launch; median of
--iters.  Algorithmic bytes = 8 h w (each element read once and written once).
"""
import argparse, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_bozkusf12_b200 import hpl

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, nargs="*", default=[16 * 1024, 5 * 1024])
ap.add_argument("--iters", type=int, default=10)
a = ap.parse_args()
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pk_path = os.path.join(root, "MEASURED_PEAKS.json")
pk = json.load(open(pk_path)) if os.path.exists(pk_path) else {}
peak = float(pk.get("hbm_gbs", 6650.0))
torch.cuda.set_device(0); hpl.hpl_set_device(0)
s = torch.cuda.current_stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
flush_rd = torch.ones(64 << 20, dtype=torch.float32, device="cuda")
for n in a.n:
    x = torch.rand(n, n, dtype=torch.float32, device="cuda")
    y = torch.empty(n, n, dtype=torch.float32, device="cuda")
    gs = torch.cuda.Stream()
    for _ in range(3):
        hpl.hpl_transpose_f32(x.data_ptr(), n, n, y.data_ptr(), gs.cuda_stream)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=gs):
        hpl.hpl_transpose_f32(x.data_ptr(), n, n, y.data_ptr(), gs.cuda_stream)
    ts = []
    for _ in range(a.iters):
        flush.zero_()
        flush_rd.sum()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        g.replay()
        e1.record(s); e1.synchronize()
        ts.append(e0.elapsed_time(e1) / 1e3)
    ts.sort()
    t = ts[len(ts) // 2]
    gbs = 8 * n * n / t / 1e9
    ok = bool(torch.equal(y, x.t()))
    # same-size device copy for context (torch's copy kernel, same bytes)
    c = torch.empty_like(x)
    tc = []
    for _ in range(a.iters):
        flush.zero_(); flush_rd.sum()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s); c.copy_(x); e1.record(s); e1.synchronize()
        tc.append(e0.elapsed_time(e1) / 1e3)
    tc.sort()
    print(json.dumps({"workload": "transpose %dx%d f32 (F4)" % (n, n), "median_s": t, "min_s": ts[0], "max_s": ts[-1],
                      "GB/s": round(gbs, 1), "equal_torch_t": ok,
                      "torch_copy_GB/s": round(8 * n * n / tc[len(tc) // 2] / 1e9, 1),
                      "roofline": {"bound": "hbm", "achieved": round(gbs, 1), "peak": peak, "unit": "GB/s",
                                   "frac": round(gbs / peak, 4), "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy)"}}),
          flush=True)
