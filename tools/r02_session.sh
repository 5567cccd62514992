#!/bin/bash
# Round-2 GPU session (under gpurun): tests + bench of the default build, A/B of
# the prebuilt variants in ab_ship/, ncu pipe counters of selected variants.
#   bash tools/r02_session.sh TAG "ab variants" "ncu variants" [steps...]
TAG=$1; AB=$2; NCUV=$3; shift 3
WHAT=${@:-tests bench ab ncu}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { echo build failed; exit 1; }
for w in $WHAT; do
case $w in
tests)
  timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_gpu_tests.log 2>&1; tail -3 gpurun_out/${TAG}_gpu_tests.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; tail -1 gpurun_out/${TAG}_smoke.log ;;
bench)
  timeout 600 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; cat gpurun_out/${TAG}_bench.json ;;
ptest)
  HPL_LIB=$PWD/ab_ship/libhpl_${PTV}.so timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_edge_pairs.py tests/test_fused_combine.py tests/test_gpu_accuracy.py -m gpu -x -q > gpurun_out/${TAG}_ptest_${PTV}.log 2>&1; tail -3 gpurun_out/${TAG}_ptest_${PTV}.log ;;
gloo2)
  bash tools/bench_gloo2.sh > gpurun_out/${TAG}_gloo2.log 2>&1; cp gpurun_out/b2_fused.json gpurun_out/${TAG}_b2_fused.json; cp gpurun_out/b2_nccl.json gpurun_out/${TAG}_b2_nccl.json; tail -8 gpurun_out/${TAG}_gloo2.log ;;
san)
  bash tools/sanitize.sh > gpurun_out/${TAG}_sanitize.log 2>&1; for t in memcheck racecheck synccheck; do cp gpurun_out/sanitize_$t.log gpurun_out/${TAG}_sanitize_$t.log; done; cat gpurun_out/${TAG}_sanitize.log ;;
evalb)
  timeout 600 python -m pytest tests/test_eval.py -m gpu -q > gpurun_out/${TAG}_evaltests.log 2>&1; tail -2 gpurun_out/${TAG}_evaltests.log
  timeout 600 python tools/bench_eval.py > gpurun_out/${TAG}_eval.jsonl 2>&1
  HPL_LIB=$PWD/ab_ship/libhpl_nopipe.so timeout 600 python tools/bench_eval.py > gpurun_out/${TAG}_eval_nopipe.jsonl 2>&1
  cat gpurun_out/${TAG}_eval.jsonl gpurun_out/${TAG}_eval_nopipe.jsonl ;;
redb)
  HPL_LIB=$PWD/ab_ship/libhpl_rtma.so timeout 600 python -m pytest tests/test_reduce.py -m gpu -q > gpurun_out/${TAG}_redtests.log 2>&1; tail -2 gpurun_out/${TAG}_redtests.log
  for v in ${REDV:-ship rtma}; do echo "== $v" >> gpurun_out/${TAG}_red.jsonl; HPL_LIB=$PWD/ab_ship/libhpl_$v.so timeout 300 python tools/bench_reduce.py --n 16777216 268435456 >> gpurun_out/${TAG}_red.jsonl 2>&1; done
  for v in ${REDV:-ship rtma}; do HPL_LIB=$PWD/ab_ship/libhpl_$v.so timeout 300 ncu --clock-control none -k regex:reduce_sum --metrics gpu__time_duration.sum,dram__bytes_read.sum --csv python tools/bench_reduce.py --n 16777216 --iters 3 > gpurun_out/${TAG}_red_ncu_$v.csv 2>&1; done
  cat gpurun_out/${TAG}_red.jsonl ;;
classes)
  for c in S W A B C; do timeout 300 python bench.py --cls $c --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/${TAG}_bench_$c.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/${TAG}_bench_$c.json'));print('$c', d['value'], d['ms_per_step'], d['verified'], d['roofline']['frac'])"; done ;;
evalab)
  for v in ${EVV}; do echo "== $v" >> gpurun_out/${TAG}_evalab.jsonl; HPL_LIB=$PWD/ab_ship/libhpl_$v.so timeout 300 python tools/bench_eval.py >> gpurun_out/${TAG}_evalab.jsonl 2>&1; done
  HPL_LIB=$PWD/ab_ship/libhpl_${PTV}.so timeout 600 python -m pytest tests/test_eval.py -m gpu -q > gpurun_out/${TAG}_evaltests.log 2>&1; tail -2 gpurun_out/${TAG}_evaltests.log
  grep -v saxpy gpurun_out/${TAG}_evalab.jsonl | cut -c1-160 ;;
spmvab)
  for v in ${SPV}; do echo "== $v" >> gpurun_out/${TAG}_spmv.jsonl; HPL_LIB=$PWD/ab_ship/libhpl_$v.so timeout 300 python tools/bench_spmv.py >> gpurun_out/${TAG}_spmv.jsonl 2>&1; done
  HPL_LIB=$PWD/ab_ship/libhpl_${PTV}.so timeout 600 python -m pytest tests/test_spmv.py -m gpu -q > gpurun_out/${TAG}_spmvtests.log 2>&1; tail -2 gpurun_out/${TAG}_spmvtests.log ;;
ref)
  timeout 600 python bench.py --impl reference > gpurun_out/${TAG}_ref.json 2> gpurun_out/${TAG}_ref.err; cat gpurun_out/${TAG}_ref.json ;;
ab)
  timeout 1200 python tools/ab_ship.py time 36 512 2 $AB > gpurun_out/${TAG}_ab.jsonl 2>&1
  python tools/ab_summary.py gpurun_out/${TAG}_ab.jsonl ;;
ncu)
  for v in $NCUV; do
    HPL_LIB=$PWD/ab_ship/libhpl_$v.so timeout 300 ncu --clock-control none -k regex:ep_kernel -s 1 -c 1 \
      --metrics gpu__time_duration.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__inst_executed_pipe_fp64.sum,smsp__inst_executed_pipe_fp64.sum,sm__cycles_elapsed.avg,smsp__average_warps_issue_stalled_dispatch_stall_per_issue_active.ratio,smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio,smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio,smsp__average_warps_issue_stalled_wait_per_issue_active.ratio,smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio \
      --csv python tools/quick_time.py 32 --threads 512 --reps 1 > gpurun_out/${TAG}_ncu_$v.csv 2>&1
  done ;;
fc)
  for v in ${FCV:-def}; do
    HPL_LIB=$PWD/ab_ship/libhpl_$v.so timeout 300 python tools/fixed_cost.py ${FCM:-10,24,25,27} >> gpurun_out/${TAG}_fc.jsonl 2>&1
  done
  cat gpurun_out/${TAG}_fc.jsonl ;;
ncufull)
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
      python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_ncu_bench.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:ep_kernel -s 3 -c 1 \
      -o gpurun_out/${TAG}_prof -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_ncu_full.log 2>&1
  tail -2 gpurun_out/${TAG}_ncu_full.log ;;
shard)
  timeout 900 python tools/shard_timing.py > gpurun_out/${TAG}_shard.jsonl 2>&1; tail -4 gpurun_out/${TAG}_shard.jsonl ;;
esac
done
