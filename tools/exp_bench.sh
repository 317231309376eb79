#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu_exp.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu_exp.log
show() { python -c "import json;d=json.load(open('$1'));print('$2', round(d['value']/1e9,3), 'G/s', round(d['ms_per_step'],3), 'ms frac', round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])" || tail -3 ${1%.json}.err; }
for v in 0 1; do
  CAPGPU_NO_CHUNKING=$v timeout 300 python bench.py --config 3 --no-cpu-baseline --steps 10 --warmup 3 > gpurun_out/e3_$v.json 2>gpurun_out/e3_$v.err; show gpurun_out/e3_$v.json "cfg3 nochunk=$v"
done
timeout 300 python bench.py --config 5 --no-cpu-baseline --steps 5 --warmup 3 --periods 500 > gpurun_out/e5.json 2>gpurun_out/e5.err; show gpurun_out/e5.json "cfg5"
