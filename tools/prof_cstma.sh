mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_control_step_tma -s 3 -c 1 -o /tmp/prof_cstma -f python bench.py --config 3 --call control_step --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_cstma.log 2>&1; tail -1 gpurun_out/ncu_cstma.log
ncu -i /tmp/prof_cstma.ncu-rep --page raw --csv > gpurun_out/cstma_raw.csv 2>/dev/null
ncu -i /tmp/prof_cstma.ncu-rep --page source --csv --print-source sass > gpurun_out/cstma_src.csv 2>/dev/null; gzip -f gpurun_out/cstma_src.csv
