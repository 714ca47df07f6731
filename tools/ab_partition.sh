# A/B: persistent TMA partition vs one-CTA-per-tile partition (ncu launch durations)
NCU=/usr/local/cuda/bin/ncu
RTM_LIB_PATH=$PWD/tools/librtm_timing.so python tools/prof_step.py --warmup 1 --steps 1 2>&1 | grep phase
$NCU --metrics gpu__time_duration.sum -k regex:k_partition -s 1 -c 1 python tools/prof_step.py --warmup 1 --steps 1 2>&1 | grep -E "k_partition|duration"
RTM_NO_TMA=1 $NCU --metrics gpu__time_duration.sum -k regex:k_partition -s 1 -c 1 python tools/prof_step.py --warmup 1 --steps 1 2>&1 | grep -E "k_partition|duration"
