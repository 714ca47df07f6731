# A/B: one-CTA-per-tile partition vs persistent TMA partition (phase timing + bench step time)
RTM_LIB_PATH=$PWD/tools/librtm_timing.so python tools/prof_step.py --warmup 1 --steps 1 2>&1 | grep phase
RTM_TMA=1 RTM_LIB_PATH=$PWD/tools/librtm_timing.so python tools/prof_step.py --warmup 1 --steps 1 2>&1 | grep phase
python bench.py --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('default', d['ms_per_step'], d['kernel_share'])"
RTM_TMA=1 python bench.py --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('tma', d['ms_per_step'], d['kernel_share'])"
