#!/bin/bash
# One ncu --set full capture of the dominant kernel of the cfg 4 and cfg 5
# bench commands (DRAM traffic per launch for bench.py's roofline.traffic).
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none -k regex:k_period -s 3 -c 1 -o gpurun_out/prof_cfg4 -f \
  python bench.py --config 4 --steps 1 --warmup 1 --periods 20 --no-cpu-baseline > gpurun_out/prof_cfg4.log 2>&1
tail -1 gpurun_out/prof_cfg4.log
timeout 1200 ncu --set full --clock-control none -k regex:k_simulate -c 1 -o gpurun_out/prof_cfg5 -f \
  python bench.py --config 5 --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/prof_cfg5.log 2>&1
tail -1 gpurun_out/prof_cfg5.log
timeout 900 ncu --set full --clock-control none -k regex:k_simulate -c 1 -o gpurun_out/prof_cfg3c -f \
  python bench.py --config 3 --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/prof_cfg3c.log 2>&1
tail -1 gpurun_out/prof_cfg3c.log
