# A/B of two builds of librtm on one box: bench lines alternating A, B, A, B ...
#   bash tools/ab.sh <libA.so> <libB.so> [config] [rounds] [steps]
A=${1:?libA}; B=${2:?libB}; CFG=${3:-C2-1gpu}; R=${4:-3}; S=${5:-30}
for i in $(seq 1 $R); do
  for v in A B; do
    if [ $v = A ]; then export RTM_LIB_PATH=$A; else export RTM_LIB_PATH=$B; fi
    timeout 600 python bench.py --config $CFG --steps $S --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | \
      python -c "import json,sys;d=json.loads(sys.stdin.read());print('$v', round(d['ms_per_step'],4), {k:round(v['ms_per_step'],3) for k,v in d['kernels'].items()})"
  done
done
unset RTM_LIB_PATH
