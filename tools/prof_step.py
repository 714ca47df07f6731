"""Profiling driver: C2 resident in HBM, `--steps` reduce steps after warm-up (for ncu / nsight).

    ncu --set full -k regex:k_partition -s 2 -c 1 -o gpurun_out/prof python tools/prof_step.py
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import gen  # noqa: E402
from paper_conf_micro_mosallaeii024_b200 import Monitor  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--steps", type=int, default=1)
ap.add_argument("--warmup", type=int, default=1)
ap.add_argument("--config", default="C2-1gpu")
args = ap.parse_args()
wl = gen.CONFIGS[args.config]
owner, cap, tot = gen.registry(wl)
ds = torch.empty(wl.n_samples * 16, dtype=torch.uint8, device="cuda")
de = torch.empty(wl.n_events * 16, dtype=torch.uint8, device="cuda")
gen.fill_device("samples", wl, ds.data_ptr(), 0, wl.n_samples)
gen.fill_device("events", wl, de.data_ptr(), 0, wl.n_events)
torch.cuda.synchronize()
mon = Monitor(owner, cap, tot, n_components=wl.n_components, t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k)
t_end = wl.t_end()
for i in range(args.warmup + args.steps):
    mon.reset()
    mon.ingest(ds, de)
    res = mon.window_reduce(t_end)
torch.cuda.synchronize()
print("done", int(res["summary"]["n_samples"].sum()))
