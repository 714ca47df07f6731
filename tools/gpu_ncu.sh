# ncu launch list + full capture of the hot kernels (1 GPU; never a multi-rank command)
set -x
NCU=/usr/local/cuda/bin/ncu
timeout 600 $NCU --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python tools/prof_step.py --warmup 1 --steps 1 > gpurun_out/ncu_launches.log 2>&1; echo "launches rc=$?"
timeout 1200 $NCU --set full --clock-control none --import-source on -k regex:"${KREGEX:-k_partition|k_fold|k_topk|k_hang|k_events}" \
  -s ${SKIP:-5} -c ${COUNT:-5} -f -o gpurun_out/prof_full python tools/prof_step.py --warmup 1 --steps 1 > gpurun_out/ncu_full.log 2>&1; echo "full rc=$?"
tail -5 gpurun_out/ncu_full.log
ls -la gpurun_out/
