# A/B of library builds on one bench config: bash tools/ab_cfg.sh <config> <steps> lib1.so lib2.so ...
CFG=${1:?config}; S=${2:?steps}; shift 2
for L in "$@"; do
  RTM_LIB_PATH=$L timeout 600 python bench.py --config $CFG --steps $S --warmup 3 --no-cpu-baseline --no-e2e --no-streaming 2>/dev/null | tail -1 | \
    python -c "import json,sys;d=json.loads(sys.stdin.read());print('$CFG', '$L', round(d['ms_per_step'],2), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()})"
done
