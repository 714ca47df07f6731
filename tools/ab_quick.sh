# current tree: gpu parity (fast subset) + 3 bench lines with kernel shares
timeout 900 python -m pytest tests -x -q -m gpu -p no:cacheprovider -k "not full_size" 2>&1 | tail -2
for i in 1 2 3; do
  python bench.py --steps 50 --warmup 5 --no-cpu-baseline --no-e2e | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('new', round(d['ms_per_step'],4), r['kernel'], round(r['frac'],3), {k:round(v*d['ms_per_step']*1e3) for k,v in d['kernel_share'].items()})"
done
