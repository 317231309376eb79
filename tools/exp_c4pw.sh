#!/bin/bash
# cfg 4 A/B: the k_period built for 12 warps per SM (libcapgpu_pw12.so) against the product library on the per-period kernel
mkdir -p gpurun_out
CAPGPU_LIB_VARIANT=pw12 timeout 900 python -m pytest tests/test_gpu_budget.py tests/test_gpu_ref.py -x -q > gpurun_out/pytest_c4pw.log 2>&1; echo "pytest(exp) rc=$?"; tail -2 gpurun_out/pytest_c4pw.log
show() { python -c "import json;d=json.load(open('$1'));print('$2', round(d['value']/1e9,4), 'G/s', round(d['ms_per_step'],3), 'ms frac', round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])" || tail -3 ${1%.json}.err; }
for rep in 1 2; do
for v in "" pw12; do
  CAPGPU_LIB_VARIANT=$v timeout 300 python bench.py --config 4 --no-cpu-baseline --steps 5 --warmup 3 --periods 200 > gpurun_out/c4pw_$v.json 2>gpurun_out/c4pw_$v.err; show gpurun_out/c4pw_$v.json "cfg4 lib=$v"
done
done
