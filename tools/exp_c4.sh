#!/bin/bash
# cfg 4 per-period kernel: budget/ref GPU tests, bench with and without the double-buffered k_period_db
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_budget.py tests/test_gpu_ref.py -x -q > gpurun_out/pytest_c4.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_c4.log
show() { python -c "import json;d=json.load(open('$1'));print('$2', round(d['value']/1e9,3), 'G/s', round(d['ms_per_step'],3), 'ms frac', round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])" || tail -3 ${1%.json}.err; }
for v in 0 1; do
  CAPGPU_NO_PERIOD_DB=$v timeout 300 python bench.py --config 4 --no-cpu-baseline --steps 5 --warmup 3 --periods 200 > gpurun_out/c4_$v.json 2>gpurun_out/c4_$v.err; show gpurun_out/c4_$v.json "cfg4 no_db=$v"
done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:k_period -s 3 -c 2 --csv --log-file gpurun_out/c4_ncu.csv python bench.py --config 4 --steps 1 --warmup 1 --periods 10 --no-cpu-baseline > /dev/null 2>&1; grep -c k_period gpurun_out/c4_ncu.csv
