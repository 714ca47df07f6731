# A/B of the side-stream tail (order check + progress beside the fold, high-priority side stream)
# against RTM_SIDE_PRIO_OFF=1 and RTM_NO_SIDE_TAIL=1: parity, C2 bench, C3, streaming latency
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q -p no:cacheprovider -k "not full" 2>&1 | tail -1
setv() { unset RTM_NO_SIDE_TAIL RTM_SIDE_PRIO_OFF; case $1 in B) export RTM_SIDE_PRIO_OFF=1;; C) export RTM_NO_SIDE_TAIL=1;; esac; }
for i in 1 2 3; do
  for v in A B C; do
    setv $v
    timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | \
      python -c "import json,sys;d=json.loads(sys.stdin.read());print('$v', round(d['ms_per_step'],4),'ms', {k:round(v*d['ms_per_step']*1e3) for k,v in d['kernel_share'].items()})"
  done
done
for v in A C; do
  setv $v
  timeout 300 python bench.py --config C3-4gpu --steps 5 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | \
      python -c "import json,sys;d=json.loads(sys.stdin.read());print('C3 $v', round(d['ms_per_step'],4),'ms', {k:round(v*d['ms_per_step']*1e3) for k,v in d['kernel_share'].items()})"
  for cfg in C2-1gpu C5-long; do
    timeout 300 python tools/latency.py --config $cfg --windows 300 > gpurun_out/lat_${v}_${cfg}.json 2>&1
    python -c "import json;d=json.load(open('gpurun_out/lat_${v}_${cfg}.json'));print('lat $v $cfg', round(d['p50_us'],1), round(d['p99_us'],1), d.get('kernel_us_per_call'))"
  done
done
