#!/bin/bash
# ncu --set full of one class-C EP launch for each A/B variant in build_ab/ (dev aid)
# usage: VARIANTS="a b" THR=512 M=32 bash tools/ncu_ab.sh TAG
TAG=$1; THR=${THR:-512}; M=${M:-32}
mkdir -p gpurun_out
cat > /tmp/one.py <<PY
import sys, os, torch
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_bozkusf12_b200 import hpl
from ep_workloads import NPB_A, NPB_SEED
torch.cuda.set_device(0); hpl.hpl_set_device(0)
hpl.hpl_ep_set_config(0, $THR, 0)
out = torch.empty(13, dtype=torch.float64, device="cuda")
for _ in range(2):
    hpl.hpl_ep_run_shard($M, NPB_SEED, NPB_A, 0, 1, out.data_ptr(), torch.cuda.current_stream().cuda_stream)
torch.cuda.synchronize()
PY
for v in $VARIANTS; do
  HPL_LIB=build_ab/libhpl_$v.so timeout 600 ncu --set full --clock-control none --import-source on -k regex:ep_kernel -s 1 -c 1 \
     -o gpurun_out/${TAG}_$v -f python /tmp/one.py > gpurun_out/${TAG}_$v.log 2>&1
  tail -1 gpurun_out/${TAG}_$v.log
done
