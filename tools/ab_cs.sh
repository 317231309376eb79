#!/bin/bash
# A/B of control_step builds: VARIANTS="prod x y" (bench --call control_step at the cfg 3 shape)
for rep in 1 2; do for v in ${VARIANTS:-prod}; do lv=$v; [ "$v" = "prod" ] && lv=""
  CAPGPU_LIB_VARIANT=$lv python bench.py --config 3 --call control_step --no-cpu-baseline --steps 50 2>/dev/null | python -c "import json,sys;d=json.loads(sys.stdin.read());print('cs lib=$v', round(d['value']/1e9,3), round(d['ms_per_step']*1000,2), 'us', round(d['roofline']['frac'],3))"
done; done
