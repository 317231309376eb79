#!/bin/bash
# GPU-box: quick bench lines + one ncu --set full capture (with source) of the
# fused kernel at cfg ${CFG:-3}; rep read back here with tools/prof_regions.py.
mkdir -p gpurun_out
TAG=${TAG:-r2}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
CFGS=${CFGS:-3 5} STEPS=5 bash tools/quick_bench.sh
CFG=${CFG:-3}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KRE:-k_simulate} -c 1 \
  -o gpurun_out/prof_${TAG}_cfg$CFG -f python bench.py --config $CFG --steps 1 --warmup 1 --no-cpu-baseline \
  > gpurun_out/ncu_${TAG}_cfg$CFG.log 2>&1
tail -3 gpurun_out/ncu_${TAG}_cfg$CFG.log
