# Round-end evidence on one B200 (writes gpurun_out/; copy what is judged into profiles/):
# GPU test suite, smoke, the bench line (+ reference arm), ncu launch list of one step and one
# `ncu --set full` launch of each big kernel.
set -x
NCU=/usr/local/cuda/bin/ncu
timeout 2400 python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/bench.jsonl 2> gpurun_out/bench.err; echo "bench rc=$?"
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.jsonl 2>&1; echo "ref rc=$?"
timeout 600 $NCU --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python tools/prof_step.py --warmup 1 --steps 1 > gpurun_out/ncu_launches.log 2>&1; echo "launches rc=$?"
timeout 1500 $NCU --set full --clock-control none --import-source on -k regex:"k_partition|k_fold|k_topk|k_events" \
  -s 3 -c 3 -f -o gpurun_out/prof_full python tools/prof_step.py --warmup 1 --steps 1 > gpurun_out/ncu_full.log 2>&1; echo "full rc=$?"
ls -la gpurun_out/
