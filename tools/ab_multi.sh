# Timing A/B over several compile-time variants: default librtm.so (A) and each library given as an
# argument, C2 bench lines alternating (3 rounds) + one C3 line each.  usage: bash tools/ab_multi.sh lib1.so ...
run() {  # $1 label, $2 lib ('' = default), $3 config
  if [ -n "$2" ]; then export RTM_LIB_PATH=$2; else unset RTM_LIB_PATH; fi
  timeout 300 python bench.py --config $3 --steps ${STEPS:-20} --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | \
    python -c "import json,sys;d=json.loads(sys.stdin.read());print('$3 $1', round(d['ms_per_step'],4),'ms', {k:round(v*d['ms_per_step']*1e3) for k,v in d['kernel_share'].items()})"
}
for i in 1 2 3; do run A '' C2-1gpu; for l in "$@"; do run $(basename $l) $l C2-1gpu; done; done
STEPS=5; run A '' C3-4gpu; for l in "$@"; do run $(basename $l) $l C3-4gpu; done
unset RTM_LIB_PATH
