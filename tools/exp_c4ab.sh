#!/bin/bash
# cfg 4 A/B: the working tree (libcapgpu_exp.so) against the product library on the per-period kernel
mkdir -p gpurun_out
CAPGPU_LIB_VARIANT=exp timeout 900 python -m pytest tests/test_gpu_budget.py tests/test_gpu_ref.py -x -q > gpurun_out/pytest_c4ab.log 2>&1; echo "pytest(exp) rc=$?"; tail -2 gpurun_out/pytest_c4ab.log
show() { python -c "import json;d=json.load(open('$1'));print('$2', round(d['value']/1e9,4), 'G/s', round(d['ms_per_step'],3), 'ms frac', round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])" || tail -3 ${1%.json}.err; }
for rep in 1 2 3; do
for v in "" exp; do
  CAPGPU_LIB_VARIANT=$v timeout 300 python bench.py --config 4 --no-cpu-baseline --steps 5 --warmup 3 --periods 200 > gpurun_out/c4ab_$v.json 2>gpurun_out/c4ab_$v.err; show gpurun_out/c4ab_$v.json "cfg4 lib=$v"
done
done
