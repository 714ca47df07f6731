for v in 0 1 2 0 1 2; do
  RTM_EV=$v timeout 300 python bench.py --steps 50 --warmup 5 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | \
    python -c "import json,sys;d=json.loads(sys.stdin.read());print('ev=$v', round(d['value']/1e9,2),'G rec/s',round(d['ms_per_step'],3),'ms', {k:round(v*d['ms_per_step']*1e3) for k,v in d['kernel_share'].items()})"
done
