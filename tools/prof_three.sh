#!/bin/bash
# GPU-box: ncu --set full (with source) of the SLO-schedule fused kernel, the
# cfg 4 per-period kernel and k_control_step (one launch each); only the raw
# and source pages come back (the reports exceed gpurun's 64 MiB).
mkdir -p gpurun_out
TAG=${TAG:-r2}
cap() {  # name kernel-regex skip bench-args...
  local name=$1 kre=$2 skip=$3; shift 3
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$kre -s $skip -c 1 \
    -o /tmp/prof_$name -f python bench.py "$@" > gpurun_out/ncu_${TAG}_$name.log 2>&1; tail -1 gpurun_out/ncu_${TAG}_$name.log
  ncu -i /tmp/prof_$name.ncu-rep --page raw --csv > gpurun_out/${TAG}_${name}_raw.csv 2>/dev/null
  ncu -i /tmp/prof_$name.ncu-rep --page source --csv --print-source sass > gpurun_out/${TAG}_${name}_src.csv 2>/dev/null
  gzip -f gpurun_out/${TAG}_${name}_src.csv
}
cap slo k_simulate 1 --config slo --periods 200 --steps 1 --warmup 1 --no-cpu-baseline
cap period k_period 20 --config 4 --periods 50 --steps 1 --warmup 1 --no-cpu-baseline
cap cs k_control_step 5 --config 3 --call control_step --steps 3 --warmup 3 --no-cpu-baseline
ls -la gpurun_out
