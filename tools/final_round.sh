#!/bin/bash
# Final-check GPU session (under gpurun): tests + smoke, bench (both arms),
# ncu launch list + full capture, per-class bench lines, gloo 2-rank runs.
#   bash tools/final_round.sh TAG
TAG=${1:-r02final}
bash tools/gpu_round.sh $TAG tests bench ref ncu
bash tools/r02_session.sh $TAG "" "" classes gloo2
ls -la gpurun_out | tail -30
