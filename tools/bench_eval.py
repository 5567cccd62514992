"""F1 measurement: the paper's example kernels through hpl_eval (dev aid).

python tools/bench_eval.py [--log2n 26]   (one JSON line per kernel)
SAXPY (Fig. 3, y = a x + y in f64: 24 B per point) and dotp (Fig. 4, f32
products into Local memory and per-group sums: 8 B per point + 4 B per group)
over 2^log2n points, arrays device-valid (no transfers issued), one eval
captured in a CUDA graph (host-side argument checking not timed), L2 flushed
and cleaned between replays, CUDA events; median of --iters.  Roofline: HBM,
peak = MEASURED_PEAKS.json hbm_gbs (copy).
"""
import argparse, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_bozkusf12_b200 import hpl

ap = argparse.ArgumentParser()
ap.add_argument("--log2n", type=int, default=26)
ap.add_argument("--iters", type=int, default=10)
a = ap.parse_args()
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pk_path = os.path.join(root, "MEASURED_PEAKS.json")
peak = float((json.load(open(pk_path)) if os.path.exists(pk_path) else {}).get("hbm_gbs", 6650.0))
torch.cuda.set_device(0); hpl.hpl_set_device(0)
s = torch.cuda.current_stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
flush_rd = torch.ones(64 << 20, dtype=torch.float32, device="cuda")
n = 1 << a.log2n


def timed(name, arrays, args, global_, local, nbytes):
    gs = torch.cuda.Stream()
    for h in arrays:
        hpl.hpl_array_set_stream(h, gs.cuda_stream)
    for _ in range(3):
        hpl.hpl_eval(name, args, global_=global_, local=local)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=gs):
        hpl.hpl_eval(name, args, global_=global_, local=local)
    ts = []
    for _ in range(a.iters):
        flush.zero_(); flush_rd.sum()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s); g.replay(); e1.record(s); e1.synchronize()
        ts.append(e0.elapsed_time(e1) / 1e3)
    for h in arrays:
        hpl.hpl_array_set_stream(h, None)
    ts.sort()
    t = ts[len(ts) // 2]
    gbs = nbytes / t / 1e9
    print(json.dumps({"workload": "%s over %d points (F1, hpl_eval)" % (name, n), "local": local,
                      "median_s": t, "GB/s": round(gbs, 1),
                      "roofline": {"bound": "hbm", "achieved": round(gbs, 1), "peak": peak, "unit": "GB/s",
                                   "frac": round(gbs / peak, 4), "bytes": nbytes}}), flush=True)


# SAXPY (Fig. 3): y:F64:rw, x:F64:r, a:f64 — library-chosen local domain
y = hpl.hpl_array_alloc(hpl.HPL_F64, [n])
x = hpl.hpl_array_alloc(hpl.HPL_F64, [n])
timed("saxpy", [y, x], [y, x, 1.5], [n], None, 24 * n)
hpl.hpl_array_free(y); hpl.hpl_array_free(x)

# dotp (Fig. 4): v1, v2 f32, pSums one per group of M
for M in [int(x) for x in os.environ.get("EVAL_MS", "32,64,128,256,1024").split(",")]:
    v1 = hpl.hpl_array_alloc(hpl.HPL_F32, [n])
    v2 = hpl.hpl_array_alloc(hpl.HPL_F32, [n])
    ps = hpl.hpl_array_alloc(hpl.HPL_F32, [n // M])
    timed("dotp", [v1, v2, ps], [v1, v2, ps], [n], [M], 8 * n + 8 * (n // M))
    for h in (v1, v2, ps):
        hpl.hpl_array_free(h)
