# A/B of the current tree against an older tree unpacked + built under build/oldtree
for i in 1 2 3; do
  (cd build/oldtree && python bench.py --steps 50 --warmup 5 --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('old', round(d['ms_per_step'],4), {k:round(v*d['ms_per_step']*1e3) for k,v in d['kernel_share'].items()})")
  python bench.py --steps 50 --warmup 5 --no-cpu-baseline --no-e2e | python -c "import json,sys;d=json.loads(sys.stdin.read());print('new', round(d['ms_per_step'],4), {k:round(v*d['ms_per_step']*1e3) for k,v in d['kernel_share'].items()})"
done
