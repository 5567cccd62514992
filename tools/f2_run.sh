mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python tools/bench_reduce.py --n 16777216 268435456 --flush write > gpurun_out/f2_w.jsonl 2>&1
python tools/bench_reduce.py --n 16777216 268435456 --flush write_read > gpurun_out/f2_wr.jsonl 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:reduce --csv python tools/bench_reduce.py --n 16777216 --iters 3 > gpurun_out/f2_ncu.csv 2>&1
cat gpurun_out/f2_w.jsonl gpurun_out/f2_wr.jsonl; grep -E "reduce" gpurun_out/f2_ncu.csv | tail -9
