#!/bin/bash
# A/B of the working tree (libcapgpu_exp.so) against the product library: parity tests on exp, cfg 3 / 5 / 4 benches (interleaved)
mkdir -p gpurun_out
CAPGPU_LIB_VARIANT=exp timeout 900 python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_ab.log 2>&1; echo "pytest(exp) rc=$?"; tail -2 gpurun_out/pytest_ab.log
show() { python -c "import json;d=json.load(open('$1'));print('$2', round(d['value']/1e9,3), 'G/s', round(d['ms_per_step'],3), 'ms frac', round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])" || tail -3 ${1%.json}.err; }
for rep in 1 2; do
for v in "" exp; do
  CAPGPU_LIB_VARIANT=$v timeout 300 python bench.py --config 3 --no-cpu-baseline --steps 10 --warmup 3 > gpurun_out/ab3_$v.json 2>gpurun_out/ab3_$v.err; show gpurun_out/ab3_$v.json "cfg3 lib=$v"
  CAPGPU_LIB_VARIANT=$v timeout 300 python bench.py --config 5 --no-cpu-baseline --steps 3 --warmup 3 --periods 500 > gpurun_out/ab5_$v.json 2>gpurun_out/ab5_$v.err; show gpurun_out/ab5_$v.json "cfg5 lib=$v"
  CAPGPU_LIB_VARIANT=$v timeout 300 python bench.py --config 4 --no-cpu-baseline --steps 3 --warmup 3 --periods 200 > gpurun_out/ab4_$v.json 2>gpurun_out/ab4_$v.err; show gpurun_out/ab4_$v.json "cfg4 lib=$v"
done
done
