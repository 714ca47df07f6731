"""Phase timing of the persistent partition kernel: build librtm with -DRTM_PHASE_TIMING into
gpurun_out/, point RTM_LIB_PATH at it and run tools/prof_step.py (the library prints a [phase] line
per reduce call on stderr).  On the GPU box:  python tools/phase_timing.py"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
csrc = os.path.join(ROOT, "paper_conf_micro_mosallaeii024_b200", "csrc")
out = os.path.join(ROOT, "gpurun_out", "librtm_pt.so")
os.makedirs(os.path.dirname(out), exist_ok=True)
subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-std=c++17",
                       "-Xcompiler", "-fPIC", "-shared", "--expt-relaxed-constexpr", "-DRTM_PHASE_TIMING",
                       "-I", os.path.join(ROOT, "include"), "-o", out, os.path.join(csrc, "rtm_api.cpp"),
                       os.path.join(csrc, "rtm_kernels.cu")])
env = dict(os.environ, RTM_LIB_PATH=out)
sys.exit(subprocess.call([sys.executable, os.path.join(ROOT, "tools", "prof_step.py"), "--warmup", "1",
                          "--steps", "2"], env=env))
