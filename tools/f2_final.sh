mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_reduce.py -q 2>&1 | tail -1
python tools/bench_reduce.py --n 16777216 268435456 1073741824 > gpurun_out/f2_final.jsonl 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum --clock-control none -k regex:reduce_sum --csv python tools/bench_reduce.py --n 16777216 1073741824 --iters 2 > gpurun_out/f2_final_ncu.csv 2>/dev/null
cat gpurun_out/f2_final.jsonl; grep -E "reduce_sum" gpurun_out/f2_final_ncu.csv | awk -F'","' '{print $(NF-2), $NF}'
