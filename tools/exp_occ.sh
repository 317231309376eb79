#!/bin/bash
# cfg 5 (N = 4) under different resident-warp targets of the fused kernel
mkdir -p gpurun_out
show() { python -c "import json;d=json.load(open('$1'));print('$2', round(d['value']/1e9,3), 'G/s', round(d['ms_per_step'],3), 'ms frac', round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])" || tail -3 ${1%.json}.err; }
for v in "" w12 w20 ""; do
  CAPGPU_LIB_VARIANT=$v timeout 300 python bench.py --config 5 --no-cpu-baseline --steps 3 --warmup 3 --periods 500 > gpurun_out/occ5_$v.json 2>gpurun_out/occ5_$v.err; show gpurun_out/occ5_$v.json "cfg5 lib=$v"
done
