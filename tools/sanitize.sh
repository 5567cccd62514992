#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck on small EP runs (dev aid)
cat > /tmp/san.py <<'PY'
import sys, os, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_bozkusf12_b200 import hpl
from ep_workloads import NPB_A, NPB_SEED
torch.cuda.set_device(0); hpl.hpl_set_device(0)
for v in (0, 1):
    hpl.hpl_ep_set_config(v, 0, 0)
    print(v, hpl.hpl_ep_run(16, NPB_SEED, NPB_A))
    print(v, hpl.hpl_ep_run(12, 1, NPB_A))
print(hpl.hpl_lcg_states(NPB_SEED, NPB_A, 5, 8))
PY
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python /tmp/san.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; tail -2 gpurun_out/sanitize_$tool.log
done
