# dev: F2 reduce A/B variants in build_ab/ (event timing + ncu kernel duration at 16M)
mkdir -p gpurun_out
for v in ${VARIANTS}; do
  echo "== $v"
  HPL_LIB=build_ab/libhpl_$v.so python tools/bench_reduce.py --n 16777216 268435456 | cut -c1-140
  HPL_LIB=build_ab/libhpl_$v.so ncu --metrics gpu__time_duration.sum --clock-control none -k regex:reduce_sum --csv python tools/bench_reduce.py --n 16777216 --iters 3 2>/dev/null | grep gpu__time | tail -2 | awk -F'","' '{print $NF}'
done
