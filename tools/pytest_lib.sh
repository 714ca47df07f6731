# GPU parity subset against a variant library: bash tools/pytest_lib.sh lib.so [pytest -k expr]
RTM_LIB_PATH=$1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -m "gpu and not slow" ${2:+-k "$2"} 2>&1 | tail -2
