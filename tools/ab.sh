#!/bin/bash
# A/B of prebuilt libraries on the GPU box: VARIANTS="base prod x" (prod = libcapgpu.so,
# others = libcapgpu_<v>.so), CFGS="3 5", REPS=2; optional PYTEST="-k expr" runs the GPU
# tests on the product library first.
mkdir -p gpurun_out
if [ -n "$PYTEST" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q $PYTEST > gpurun_out/pytest_ab.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_ab.log
fi
show() { python -c "import json;d=json.load(open('$1'));print('$2', round(d['value']/1e9,3), 'G/s', round(d['ms_per_step'],3), 'ms frac', round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])" || tail -3 ${1%.json}.err; }
for rep in $(seq 1 ${REPS:-2}); do
for v in ${VARIANTS:-base prod}; do
  lv=$v; [ "$v" = "prod" ] && lv=""
  for c in ${CFGS:-3 5}; do
    extra=""; [ "$c" = "5" ] && extra="--periods 500"; [ "$c" = "4" ] && extra="--periods 200"; [ "$c" = "slo" ] && extra="--periods 400"
    CAPGPU_LIB_VARIANT=$lv timeout 300 python bench.py --config $c --no-cpu-baseline --steps ${STEPS:-5} --warmup 3 $extra > gpurun_out/ab${c}_$v.json 2>gpurun_out/ab${c}_$v.err; show gpurun_out/ab${c}_$v.json "cfg$c lib=$v"
  done
done
done
