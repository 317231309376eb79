#!/bin/bash
# GPU-box profiling pass of the fused kernel (cfg 3): phase timing (profiling
# build) + one ncu --set full capture with source, read back here with
# tools/prof_summary.py / tools/src_stalls.py.
set -x
mkdir -p gpurun_out
CFG=${CFG:-3}
python -m paper_conf_icpp_masw25_b200.build --variant=timing > /dev/null 2>&1
CAPGPU_LIB_VARIANT=timing timeout 300 python tools/phase_timing.py $CFG 200 > gpurun_out/phase_cfg$CFG.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_simulate -c 1 \
  -o gpurun_out/prof_cfg$CFG -f python bench.py --config $CFG --steps 1 --warmup 1 --no-cpu-baseline \
  > gpurun_out/ncu_cfg$CFG.log 2>&1
tail -3 gpurun_out/ncu_cfg$CFG.log
