for rep in 1 2; do for v in prod pf2 pf2plain; do
  lv=$v; unset CAPGPU_CS_PLAIN
  [ "$v" = "prod" ] && lv=""
  [ "$v" = "pf2plain" ] && { lv=pf2; export CAPGPU_CS_PLAIN=1; }
  CAPGPU_LIB_VARIANT=$lv python bench.py --config 3 --call control_step --no-cpu-baseline --steps 50 2>/dev/null | python -c "import json,sys;d=json.loads(sys.stdin.read());print('lib=$v', round(d['value']/1e9,3), round(d['ms_per_step']*1000,2), 'us', round(d['roofline']['frac'],3))"
done; done
