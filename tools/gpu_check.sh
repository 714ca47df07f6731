# one GPU round-trip: parity tests, then a short bench (logs under gpurun_out/)
set -x
timeout 1500 python -m pytest tests -x -q -m "gpu" ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -40 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
tail -5 gpurun_out/bench.log
