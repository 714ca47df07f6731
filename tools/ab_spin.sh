# A/B of a compile-time variant: default librtm.so (A) vs librtm_b.so (B): GPU parity on A, C2 bench lines alternating, one C3 line each
B=${1:-paper_conf_micro_mosallaeii024_b200/librtm_b.so}
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "not full" 2>&1 | tail -1
for i in 1 2 3; do
  for v in A B; do
    if [ $v = B ]; then export RTM_LIB_PATH=$B; else unset RTM_LIB_PATH; fi
    timeout 300 python bench.py --steps 30 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | \
      python -c "import json,sys;d=json.loads(sys.stdin.read());print('$v', round(d['ms_per_step'],4),'ms', {k:round(v*d['ms_per_step']*1e3) for k,v in d['kernel_share'].items()})"
  done
done
for v in A B; do
  if [ $v = B ]; then export RTM_LIB_PATH=$B; else unset RTM_LIB_PATH; fi
  timeout 300 python bench.py --config C3-4gpu --steps 5 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | \
      python -c "import json,sys;d=json.loads(sys.stdin.read());print('C3 $v', round(d['ms_per_step'],4),'ms', {k:round(v*d['ms_per_step']*1e3) for k,v in d['kernel_share'].items()})"
done
