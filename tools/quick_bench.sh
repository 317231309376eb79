#!/bin/bash
# quick perf check on the GPU box: cfg 3 and cfg 5 (shorter), JSON summaries
for c in ${CFGS:-3 5}; do
  extra=""; [ "$c" = "5" ] && extra="--periods 500"
  timeout 400 python bench.py --config $c --no-cpu-baseline --steps ${STEPS:-5} --warmup 3 $extra > gpurun_out/qb_cfg$c.json 2> gpurun_out/qb_cfg$c.err
  python -c "import json;d=json.load(open('gpurun_out/qb_cfg$c.json'));print('cfg$c', round(d['value']/1e9,3), 'G/s', round(d['ms_per_step'],2), 'ms', 'frac', round(d['roofline']['frac'],4), d['clocks'])" || tail -3 gpurun_out/qb_cfg$c.err
done
