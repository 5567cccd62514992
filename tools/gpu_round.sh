#!/bin/bash
# One GPU session: tests, bench (both arms), ncu launch list + full capture.
# Usage (under gpurun):  bash tools/gpu_round.sh <tag> [what...]
#   what: tests bench ref ncu  (default: all)
TAG=${1:-dev}; shift
WHAT=${@:-tests bench ref ncu}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { echo build failed; tail gpurun_out/${TAG}_build.log; exit 1; }
for w in $WHAT; do
case $w in
tests)
  timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_gpu_tests.log 2>&1; tail -3 gpurun_out/${TAG}_gpu_tests.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; tail -1 gpurun_out/${TAG}_smoke.log ;;
bench)
  timeout 600 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; cat gpurun_out/${TAG}_bench.json ;;
ref)
  timeout 600 python bench.py --impl reference > gpurun_out/${TAG}_ref.json 2> gpurun_out/${TAG}_ref.err; cat gpurun_out/${TAG}_ref.json ;;
probe)
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/probe_fp64 tools/probe_fp64.cu && ./tools/probe_fp64 > gpurun_out/${TAG}_probe.log 2>&1; cat gpurun_out/${TAG}_probe.log ;;
qt)
  python tools/quick_time.py 32 36 --threads ${QT_THREADS:-1024} > gpurun_out/${TAG}_qt.log 2>&1; cat gpurun_out/${TAG}_qt.log ;;
ncu)
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
      python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_ncu_bench.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:ep_kernel -s 3 -c 1 \
      -o gpurun_out/${TAG}_prof -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_ncu_full.log 2>&1
  tail -2 gpurun_out/${TAG}_ncu_full.log ;;
esac
done
