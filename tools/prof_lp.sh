#!/bin/bash
# GPU-box: ncu --set full (with source) of the lane-parallel kernel at cfg 2; CSV pages back
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_simulate_lp -s 1 -c 1 -o /tmp/prof_lp -f \
  python bench.py --config 2 --steps 1 --warmup 1 --periods 200 --no-cpu-baseline > gpurun_out/ncu_lp.log 2>&1; tail -1 gpurun_out/ncu_lp.log
ncu -i /tmp/prof_lp.ncu-rep --page raw --csv > gpurun_out/lp_raw.csv 2>/dev/null
ncu -i /tmp/prof_lp.ncu-rep --page source --csv --print-source sass > gpurun_out/lp_src.csv 2>/dev/null; gzip -f gpurun_out/lp_src.csv
