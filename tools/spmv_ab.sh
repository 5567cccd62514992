#!/bin/bash
# spmv A/B (under gpurun): parity tests of each variant, then bench_spmv per variant
#   bash tools/spmv_ab.sh TAG "variants..."
TAG=$1; V=$2
mkdir -p gpurun_out
for v in $V; do
  HPL_LIB=$PWD/ab_ship/libhpl_$v.so timeout 600 python -m pytest tests/test_spmv.py -m gpu -q -x > gpurun_out/${TAG}_spmvtests_$v.log 2>&1; echo "$v tests: $(tail -1 gpurun_out/${TAG}_spmvtests_$v.log)"
done
for p in 0 1; do for v in $V; do
  echo "== $v pass $p" >> gpurun_out/${TAG}_spmv.jsonl
  HPL_LIB=$PWD/ab_ship/libhpl_$v.so timeout 300 python tools/bench_spmv.py >> gpurun_out/${TAG}_spmv.jsonl 2>&1
done; done
python - <<PY
import json
v=None
for l in open("gpurun_out/${TAG}_spmv.jsonl"):
    if l.startswith("=="): v=l.strip(); continue
    if l.startswith("{"):
        d=json.loads(l)
        if "roofline" in d: print(v, d["workload"][-12:], round(d["median_s"]*1e6,2), "us", d["roofline"]["frac"])
PY
