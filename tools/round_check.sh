#!/bin/bash
# GPU-box round check: full GPU suite, smoke, bench lines (cfg 3 default, cfg 5, cfg 4, cfg 2, slo,
# control_step), ncu launch list of the default bench command.
mkdir -p gpurun_out
TAG=${TAG:-r2}
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke_$TAG.log
timeout 600 python bench.py > gpurun_out/bench_cfg3_$TAG.json 2> gpurun_out/bench_cfg3_$TAG.err; echo "bench rc=$?"; cat gpurun_out/bench_cfg3_$TAG.json
for c in 5 4 2 slo; do
  timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_cfg${c}_$TAG.json 2> gpurun_out/bench_cfg${c}_$TAG.err; cat gpurun_out/bench_cfg${c}_$TAG.json
done
timeout 300 python bench.py --config 3 --call control_step --no-cpu-baseline --steps 50 > gpurun_out/bench_cs_$TAG.json 2> gpurun_out/bench_cs_$TAG.err; cat gpurun_out/bench_cs_$TAG.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_cfg3_$TAG.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_launch_bench_$TAG.log 2>&1; echo "ncu rc=$?"
