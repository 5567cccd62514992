#!/bin/bash
# GPU-box probe: hardware facts used by DESIGN.md (host cores, FP64 rate, approx accuracy)
set -x
nproc; lscpu | grep -E "Model name|Socket|Thread|Core"; nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > gpurun_out/probe_clocks.csv &
SMI=$!
./tools/probe_fp64
kill $SMI
