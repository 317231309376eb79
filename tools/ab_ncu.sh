#!/bin/bash
# ncu --set full (with source) of the fused kernel for each prebuilt library variant (cfg ${CFG:-3})
mkdir -p gpurun_out
CFG=${CFG:-3}
for v in ${VARIANTS:-prod}; do
  lv=$v; [ "$v" = "prod" ] && lv=""
  extra=""; [ "$CFG" = "5" ] && extra="--periods 200"
  CAPGPU_LIB_VARIANT=$lv timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KRE:-k_simulate} -c 1 \
    -o gpurun_out/ncu_${v}_cfg$CFG -f python bench.py --config $CFG --steps 1 --warmup 1 --no-cpu-baseline $extra \
    > gpurun_out/ncu_${v}_cfg$CFG.log 2>&1
  tail -1 gpurun_out/ncu_${v}_cfg$CFG.log
done
