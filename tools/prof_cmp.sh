#!/bin/bash
# ncu --set full of k_simulate (cfg 3) with and without the chunked schedule
mkdir -p gpurun_out
for v in 0 1; do
  CAPGPU_NO_CHUNKING=$v timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_simulate -c 1 \
    -o gpurun_out/prof_nc$v -f python bench.py --config 3 --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/prof_nc$v.log 2>&1
  tail -1 gpurun_out/prof_nc$v.log
done
for v in 0 1; do
  CAPGPU_NO_CHUNKING=$v timeout 300 python bench.py --config 3 --no-cpu-baseline --steps 10 --warmup 3 > gpurun_out/exp_nc$v.json 2>gpurun_out/exp_nc$v.err
  python -c "import json;d=json.load(open('gpurun_out/exp_nc$v.json'));print('nochunk=$v', round(d['value']/1e9,3), 'G/s', round(d['ms_per_step'],3), 'ms frac', round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])" || tail -3 gpurun_out/exp_nc$v.err
done
