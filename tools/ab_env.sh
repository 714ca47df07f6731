# A/B of a runtime switch: default (A) vs the environment variable $1=1 (B): GPU parity on A, C2 bench
# lines alternating, C3 once each, streaming latency C2 / C5.   usage: bash tools/ab_env.sh RTM_NO_SIDE_HANG
VAR=${1:?env var}
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q -p no:cacheprovider -k "not full" 2>&1 | tail -1
setv() { unset $VAR; [ $1 = B ] && export $VAR=1; }
for i in 1 2 3; do
  for v in A B; do
    setv $v
    timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | \
      python -c "import json,sys;d=json.loads(sys.stdin.read());print('$v', round(d['ms_per_step'],4),'ms', {k:round(v*d['ms_per_step']*1e3) for k,v in d['kernel_share'].items()})"
  done
done
for v in A B; do
  setv $v
  timeout 300 python bench.py --config C3-4gpu --steps 5 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | \
      python -c "import json,sys;d=json.loads(sys.stdin.read());print('C3 $v', round(d['ms_per_step'],4),'ms')"
done
for i in 1 2; do for v in A B; do
  setv $v
  for cfg in C2-1gpu C5-long; do
    timeout 300 python tools/latency.py --config $cfg --windows 300 > gpurun_out/lat_${v}_${cfg}.json 2>&1
    python -c "import json;d=json.load(open('gpurun_out/lat_${v}_${cfg}.json'));print('lat $v $cfg', round(d['p50_us'],1), round(d['p99_us'],1))"
  done
done; done
unset $VAR
