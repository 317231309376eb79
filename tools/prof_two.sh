#!/bin/bash
# GPU-box: ncu --set full (with source) of the fused kernel at cfg 3 and cfg 5
# (shortened run), reps read back here with tools/src_stalls.py / prof_regions.py.
mkdir -p gpurun_out
TAG=${TAG:-r2}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_simulate -c 1 \
  -o gpurun_out/prof_${TAG}_cfg3 -f python bench.py --config 3 --steps 1 --warmup 1 --no-cpu-baseline \
  > gpurun_out/ncu_${TAG}_cfg3.log 2>&1; tail -2 gpurun_out/ncu_${TAG}_cfg3.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_simulate -c 1 \
  -o gpurun_out/prof_${TAG}_cfg5 -f python bench.py --config 5 --periods 200 --steps 1 --warmup 1 --no-cpu-baseline \
  > gpurun_out/ncu_${TAG}_cfg5.log 2>&1; tail -2 gpurun_out/ncu_${TAG}_cfg5.log
