#!/bin/bash
# cfg 4: per-period throughput against the run length (interleaved 1000 / 200 / 500 periods)
mkdir -p gpurun_out
show() { python -c "import json;d=json.load(open('$1'));print('$2', round(d['value']/1e9,4), 'G/s', round(d['ms_per_step'],3), 'ms frac', round(d['roofline']['frac'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 ${1%.json}.err; }
for rep in 1 2; do
for n in 1000 200 500; do
  timeout 300 python bench.py --config 4 --no-cpu-baseline --steps 5 --warmup 3 --periods $n > gpurun_out/c4len_$n.json 2>gpurun_out/c4len_$n.err; show gpurun_out/c4len_$n.json "cfg4 periods=$n"
done
done
