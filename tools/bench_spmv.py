"""F4 measurement: spmv_csr on Fig. 7's 16K x 16K, 1 % matrix (dev aid).

Device time per hpl_eval with CUDA events (arrays already device-valid, so no
transfers are issued), L2 flushed between launches (256 MB write, then a
256 MB read so the dirty lines are written back before the timed region).  Algorithmic bytes =
A + cols (8 B per nonzero) + rowptr + vec + out (each read/written once).
"""
import ctypes, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_ipps_bozkusf12_b200 import hpl
from ep_workloads import SPMV_DENSITY, SPMV_ROWS, make_csr

root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pk = json.load(open(os.path.join(root, "MEASURED_PEAKS.json"))) if os.path.exists(os.path.join(root, "MEASURED_PEAKS.json")) else {}
peak = float(pk.get("hbm_gbs", 6650.0))
torch.cuda.set_device(0); hpl.hpl_set_device(0)
rowptr, cols, A = make_csr(SPMV_ROWS, SPMV_ROWS, SPMV_DENSITY, seed=16)
vec = np.random.default_rng(17).uniform(-1, 1, SPMV_ROWS).astype(np.float32)
rows, nnz = SPMV_ROWS, len(A)

def arr(code, x, ct):
    a = hpl.hpl_array_alloc(code, [len(x)])
    np.ctypeslib.as_array((ct * len(x)).from_address(hpl.hpl_array_data(a, hpl.HPL_HOST)))[:] = x
    hpl.hpl_array_sync(a, hpl.HPL_HOST, hpl.HPL_WRITE)
    return a

hs = [arr(hpl.HPL_F32, A, ctypes.c_float), arr(hpl.HPL_F32, vec, ctypes.c_float),
      arr(hpl.HPL_I32, cols, ctypes.c_int32), arr(hpl.HPL_I32, rowptr, ctypes.c_int32),
      hpl.hpl_array_alloc(hpl.HPL_F32, [rows])]
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
flush_rd = torch.ones(64 << 20, dtype=torch.float32, device="cuda")  # 256 MB read: writes back the flush's dirty lines
s = torch.cuda.default_stream()
for M in (8, 16, 32):
    for _ in range(3):
        hpl.hpl_eval("spmv_csr", hs, global_=[rows * M], local=[M])
    torch.cuda.synchronize()
    # capture one eval in a CUDA graph so host-side argument checking is not timed
    gs = torch.cuda.Stream()
    for h in hs:
        hpl.hpl_array_set_stream(h, gs.cuda_stream)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=gs):
        hpl.hpl_eval("spmv_csr", hs, global_=[rows * M], local=[M])
    ts = []
    for _ in range(20):
        flush.zero_(); flush_rd.sum(); torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(s)
        g.replay()
        e1.record(s); e1.synchronize()
        ts.append(e0.elapsed_time(e1) / 1e3)
    for h in hs:
        hpl.hpl_array_set_stream(h, None)
    t = sorted(ts)[len(ts) // 2]
    byts = 8 * nnz + 4 * (rows + 1) + 4 * rows + 4 * rows
    print(json.dumps({"workload": "spmv_csr 16Kx16K 1%% nnz=%d M=%d (F4)" % (nnz, M), "median_s": t,
                      "GFLOP/s": round(2 * nnz / t / 1e9, 1),
                      "roofline": {"bound": "hbm", "achieved": round(byts / t / 1e9, 1), "peak": peak, "unit": "GB/s",
                                   "frac": round(byts / t / 1e9 / peak, 4), "bytes": byts}}), flush=True)
# context: cuSPARSE SpMV of the same matrix through torch (CSR @ dense vector),
# same flush and event timing (its order of additions differs: not a parity check)
Acsr = torch.sparse_csr_tensor(torch.from_numpy(rowptr.astype(np.int64)).cuda(), torch.from_numpy(cols.astype(np.int64)).cuda(),
                               torch.from_numpy(A).cuda(), size=(rows, rows))
xv = torch.from_numpy(vec).cuda()
for _ in range(3):
    yv = Acsr @ xv
torch.cuda.synchronize()
tc = []
for _ in range(20):
    flush.zero_(); flush_rd.sum(); torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record(s)
    yv = Acsr @ xv
    e1.record(s); e1.synchronize()
    tc.append(e0.elapsed_time(e1) / 1e3)
t = sorted(tc)[len(tc) // 2]
print(json.dumps({"workload": "context: torch CSR @ vector (cuSPARSE), same matrix", "median_s": t,
                  "GFLOP/s": round(2 * nnz / t / 1e9, 1)}), flush=True)
for h in hs:
    hpl.hpl_array_free(h)
