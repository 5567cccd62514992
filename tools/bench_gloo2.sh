mkdir -p gpurun_out
for c in fused nccl; do
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 --cls C --no-cpu-baseline --dist-backend gloo --combine $c > gpurun_out/b2_$c.json 2> gpurun_out/b2_$c.err; echo rc=$?; cat gpurun_out/b2_$c.json; tail -3 gpurun_out/b2_$c.err
done
