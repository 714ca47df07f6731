# A/B on C2: parity subset, then bench lines (kernel shares) for each RTM_FOLD variant given
# usage: bash tools/ab.sh "chain bkt"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "not c2_full" 2>&1 | tail -2
for v in ${1:-chain bkt}; do
  RTM_FOLD=$v timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | \
    python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('$v', round(d['value']/1e9,2),'G rec/s',round(d['ms_per_step'],3),'ms', {k:round(v*d['ms_per_step']*1e3) for k,v in d['kernel_share'].items()})"
done
