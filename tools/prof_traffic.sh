#!/bin/bash
# DRAM traffic per launch of the dominant kernel of the cfg 4 / cfg 5 / cfg 3
# bench commands (bench.py roofline.traffic).  cfg 4 and cfg 3: one
# ncu --set full capture; cfg 5 (an 0.8 s launch): the dram/time metrics only.
# The reports are reduced to CSV on the box (gpurun_out/ must stay < 64 MiB).
mkdir -p gpurun_out
raw() { ncu -i $1.ncu-rep --page raw --csv > $1_raw.csv 2>/dev/null; rm -f $1.ncu-rep; }
timeout 900 ncu --set full --clock-control none -k regex:k_period -s 3 -c 1 -o gpurun_out/prof_cfg4 -f \
  python bench.py --config 4 --steps 1 --warmup 1 --periods 20 --no-cpu-baseline > gpurun_out/prof_cfg4.log 2>&1
raw gpurun_out/prof_cfg4
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_simulate -c 1 -o gpurun_out/prof_cfg3c -f \
  python bench.py --config 3 --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/prof_cfg3c.log 2>&1
ncu -i gpurun_out/prof_cfg3c.ncu-rep --page source --csv --print-source sass > gpurun_out/prof_cfg3c_sass.csv 2>/dev/null
raw gpurun_out/prof_cfg3c
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active \
  --clock-control none -k regex:k_simulate -c 1 --csv --log-file gpurun_out/prof_cfg5_metrics.csv \
  python bench.py --config 5 --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/prof_cfg5.log 2>&1
ls -la gpurun_out/
