# r02 final evidence run (one gpurun call): GPU suite (incl. slow full-size configs), smoke, ncu
# launch list + --set full of the C2 step's kernels, bench lines (C2 contract line, C3, C4),
# streaming latency (C2, C5), the full C5 run against the range-parallel oracle.  Outputs in gpurun_out/.
NCU=/usr/local/cuda/bin/ncu
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/r02h_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/r02h_pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/r02h_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/r02h_smoke.log
timeout 900 python bench.py --steps 50 --warmup 5 > gpurun_out/r02h_bench.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/r02h_bench.log | cut -c1-300
for c in C3-4gpu C4-skewed; do timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-streaming --no-cpu-sharded > gpurun_out/r02h_bench_$c.log 2>&1; echo "$c rc=$?"; done
for c in C2-1gpu C5-long; do timeout 400 python tools/latency.py --config $c --windows 1000 > gpurun_out/r02h_latency_$c.json 2>&1; done
timeout 600 $NCU --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02h_launches.csv \
  python tools/prof_step.py --warmup 1 --steps 1 > /dev/null 2>&1; echo "launches rc=$?"
timeout 1200 $NCU --set full --clock-control none --import-source on -k regex:"k_partition|k_fold|k_topk|k_prep|k_hang|k_progress|k_order" \
  -s 7 -c 7 -f -o gpurun_out/r02h_full python tools/prof_step.py --warmup 1 --steps 1 > gpurun_out/r02h_full.log 2>&1; echo "full rc=$?"
timeout 2400 python tools/c5_full.py --windows 1000000 --batch 1000 --oracle --out gpurun_out/r02h_c5_full.json > gpurun_out/r02h_c5_full.log 2>&1; echo "c5 rc=$?"; tail -3 gpurun_out/r02h_c5_full.log
