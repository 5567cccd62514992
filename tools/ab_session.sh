#!/bin/bash
# A/B timing session on one GPU (under gpurun):  bash tools/ab_session.sh TAG M "name=DEFS" ...
# Builds each variant on the box (build_ab/ does not travel), then times every
# variant at class M in two passes, the second in reverse order.
TAG=$1; M=$2; shift 2
mkdir -p gpurun_out
names=()
for spec in "$@"; do
  python tools/ab.py build "$spec" >> gpurun_out/${TAG}_abbuild.log 2>&1 &
  names+=("${spec%%=*}")
done
wait
rev=()
for ((i=${#names[@]}-1; i>=0; i--)); do rev+=("${names[i]}"); done
python tools/ab.py time $M 512 "${names[@]}" > gpurun_out/${TAG}_ab.jsonl 2>&1
python tools/ab.py time $M 512 "${rev[@]}" >> gpurun_out/${TAG}_ab.jsonl 2>&1
cat gpurun_out/${TAG}_ab.jsonl
