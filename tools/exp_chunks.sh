for rep in 1 2; do for c in 0 2 3 4 6 8 12 16; do
  if [ $c = 0 ]; then unset CAPGPU_SIM_CHUNKS; else export CAPGPU_SIM_CHUNKS=$c; fi
  python bench.py --config 3 --no-cpu-baseline --steps 8 --warmup 3 2>/dev/null | python -c "import json,sys;d=json.loads(sys.stdin.read());print('chunks=$c', round(d['value']/1e9,3), round(d['ms_per_step'],3))"
done; done
