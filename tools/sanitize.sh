# compute-sanitizer over the C1-shaped workload (tools/sanitize.py); logs in gpurun_out/
CS=/usr/local/cuda/bin/compute-sanitizer
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  arg=""; [ $tool = memcheck ] || arg="--small"
  timeout 1500 $CS --tool $tool --print-limit 50 python tools/sanitize.py $arg > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|sanitize workload OK' gpurun_out/sanitize_$tool.log | tr '\n' ' ')"
done
