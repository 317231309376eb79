#!/bin/bash
# A/B of SLO-schedule builds: VARIANTS="prod s12 s8"
mkdir -p gpurun_out
for rep in 1 2; do for v in ${VARIANTS:-prod}; do lv=$v; [ "$v" = "prod" ] && lv=""
  CAPGPU_LIB_VARIANT=$lv timeout 300 python bench.py --config slo --no-cpu-baseline --steps 3 --warmup 2 --periods 400 > gpurun_out/abslo_$v.json 2>gpurun_out/abslo_$v.err
  python -c "import json;d=json.load(open('gpurun_out/abslo_$v.json'));print('slo lib=$v', round(d['value']/1e9,3), 'G/s', round(d['ms_per_step'],2), 'ms')" || tail -3 gpurun_out/abslo_$v.err
done; done
