# A/B of runtime experiment switches (RTM_XP bit mask, csrc: p.xp) on C2: GPU parity subset under
# each non-zero variant, then alternating bench lines.   usage: bash tools/ab_xp.sh "0 1"
for v in ${1:-0 1}; do
  [ "$v" != 0 ] && RTM_XP=$v timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "not full" 2>&1 | tail -1
done
for i in 1 2 3; do
  for v in ${1:-0 1}; do
    RTM_XP=$v timeout 300 python bench.py --steps 30 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | \
      python -c "import json,sys;d=json.loads(sys.stdin.read());print('xp=$v', round(d['ms_per_step'],4),'ms', {k:round(v*d['ms_per_step']*1e3) for k,v in d['kernel_share'].items()})"
  done
done
