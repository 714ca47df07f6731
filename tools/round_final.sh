# r02 closing evidence (one gpurun call, after the last kernel change): GPU suite, smoke, the C2
# bench line, C3 / C4 lines, streaming latency.  ncu captures and the full C5 run: round_measure.sh.
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/r02i_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/r02i_pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/r02i_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/r02i_smoke.log
timeout 900 python bench.py --steps 50 --warmup 5 > gpurun_out/r02i_bench.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/r02i_bench.log | cut -c1-300
for c in C3-4gpu C4-skewed; do timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-streaming --no-cpu-sharded > gpurun_out/r02i_bench_$c.log 2>&1; echo "$c rc=$?"; done
for c in C2-1gpu C5-long; do timeout 400 python tools/latency.py --config $c --windows 1000 > gpurun_out/r02i_latency_$c.json 2>&1; done
timeout 900 python tools/c5_full.py --windows 100000 --batch 1000 > gpurun_out/r02i_c5_100k.log 2>&1; echo "c5 100k rc=$?"; grep '^{' gpurun_out/r02i_c5_100k.log | tail -1 | cut -c1-300
