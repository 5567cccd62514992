#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck on small runs of every
# kernel family: EP (both variants), transpose, reduction, eval (SAXPY, dotp,
# spmv) (dev aid)
cat > /tmp/san.py <<'PY'
import sys, os, ctypes, torch, numpy as np
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_bozkusf12_b200 import hpl
from ep_workloads import NPB_A, NPB_SEED, make_csr, make_matrix
torch.cuda.set_device(0); hpl.hpl_set_device(0)
for v in (0, 1):
    hpl.hpl_ep_set_config(v, 0, 0)
    print(v, hpl.hpl_ep_run(16, NPB_SEED, NPB_A))
    print(v, hpl.hpl_ep_run(12, 1, NPB_A))
hpl.hpl_ep_set_config(0, 0, 0)
print(hpl.hpl_lcg_states(NPB_SEED, NPB_A, 5, 8))
s = torch.cuda.current_stream().cuda_stream
for h, w in ((130, 67), (256, 512)):
    x = torch.from_numpy(make_matrix(h, w, 1)).cuda(); y = torch.empty(w, h, device="cuda")
    hpl.hpl_transpose_f32(x.data_ptr(), h, w, y.data_ptr(), s); torch.cuda.synchronize()
    print("transpose", h, w, bool(torch.equal(y, x.t())))
x = torch.randn(100003, device="cuda"); o = torch.empty(1, dtype=torch.float64, device="cuda")
hpl.hpl_reduce_sum_f32(x.data_ptr(), x.numel(), o.data_ptr(), s); torch.cuda.synchronize(); print("sum", o.item())
def arr(code, a, ct):
    h = hpl.hpl_array_alloc(code, [len(a)])
    np.ctypeslib.as_array((ct * len(a)).from_address(hpl.hpl_array_data(h, hpl.HPL_HOST)))[:] = a
    hpl.hpl_array_sync(h, hpl.HPL_HOST, hpl.HPL_WRITE); return h
for M in (1, 64, 1024):
    n = 4096 if M < 1024 else 3 * 1024
    v1 = arr(hpl.HPL_F32, np.ones(n, np.float32), ctypes.c_float); v2 = arr(hpl.HPL_F32, np.ones(n, np.float32), ctypes.c_float)
    ps = arr(hpl.HPL_F32, np.zeros(n // M, np.float32), ctypes.c_float)
    hpl.hpl_eval("dotp", [v1, v2, ps], global_=[n], local=[M]); hpl.hpl_array_sync(ps, hpl.HPL_HOST, hpl.HPL_READ)
    print("dotp", M, np.ctypeslib.as_array((ctypes.c_float * (n // M)).from_address(hpl.hpl_array_data(ps, hpl.HPL_HOST)))[:2])
rowptr, cols, A = make_csr(300, 400, 0.05, 3)
hs = [arr(hpl.HPL_F32, A, ctypes.c_float), arr(hpl.HPL_F32, np.ones(400, np.float32), ctypes.c_float),
      arr(hpl.HPL_I32, cols, ctypes.c_int32), arr(hpl.HPL_I32, rowptr, ctypes.c_int32), hpl.hpl_array_alloc(hpl.HPL_F32, [300])]
hpl.hpl_eval("spmv_csr", hs, global_=[300 * 8], local=[8]); hpl.hpl_array_sync(hs[4], hpl.HPL_HOST, hpl.HPL_READ); print("spmv ok")
y = arr(hpl.HPL_F64, np.ones(1000), ctypes.c_double); xx = arr(hpl.HPL_F64, np.ones(1000), ctypes.c_double)
hpl.hpl_eval("saxpy", [y, xx, 2.0]); hpl.hpl_array_sync(y, hpl.HPL_HOST, hpl.HPL_READ); print("saxpy ok")
PY
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python /tmp/san.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; tail -2 gpurun_out/sanitize_$tool.log
done
