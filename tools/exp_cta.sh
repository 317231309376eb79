#!/bin/bash
# A/B of the per-period kernel's CTA size (cfg 4): default library vs the cta32 variant
mkdir -p gpurun_out
show() { python -c "import json;d=json.load(open('$1'));print('$2', round(d['value']/1e9,3), 'G/s', round(d['ms_per_step'],3), 'ms frac', round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])" || tail -3 ${1%.json}.err; }
for v in "" cta32; do
  CAPGPU_LIB_VARIANT=$v timeout 300 python bench.py --config 4 --no-cpu-baseline --steps 5 --warmup 3 --periods 200 > gpurun_out/c4_$v.json 2>gpurun_out/c4_$v.err; show gpurun_out/c4_$v.json "cfg4 variant=$v"
done
CAPGPU_LIB_VARIANT=cta32 timeout 600 python -m pytest tests/test_gpu_budget.py -x -q > gpurun_out/pytest_cta32.log 2>&1; echo "budget tests cta32 rc=$?"; tail -2 gpurun_out/pytest_cta32.log
