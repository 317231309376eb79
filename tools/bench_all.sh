#!/bin/bash
# Every bench config of bench.py on one GPU (short runs), one JSON line each
mkdir -p gpurun_out
for c in 1 2 3 4 5 stab slo fixed safe gpuonly cpuonly move; do
  extra="--steps 5 --warmup 3"
  case $c in 5) extra="--steps 3 --warmup 3";; 4) extra="--steps 3 --warmup 3";; esac
  timeout 600 python bench.py --config $c --no-cpu-baseline $extra > gpurun_out/all_$c.json 2> gpurun_out/all_$c.err
  python -c "import json;d=json.load(open('gpurun_out/all_$c.json'));print('$c', '%.4g' % d['value'], round(d['ms_per_step'],3), 'ms', d['roofline']['bound'], round(d['roofline']['frac'],4))" || tail -2 gpurun_out/all_$c.err
done
