# development: time A/B builds in build_ab/ (tools/ab.py); THREADS = comma list
mkdir -p gpurun_out
TAG=${TAG:-ab}
for t in ${THREADS:-512}; do python tools/ab.py time ${M:-33} $t ${VARIANTS}; done > gpurun_out/${TAG}.jsonl 2>&1
cat gpurun_out/${TAG}.jsonl
