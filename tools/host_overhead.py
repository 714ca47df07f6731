"""Wall-clock breakdown of one bench step (reset / ingest / reduce / results) vs GPU kernel time."""
import os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np, torch
import gen
from paper_conf_micro_mosallaeii024_b200 import Monitor, _native as N
import ctypes
wl = gen.C2
owner, cap, tot = gen.registry(wl)
ds = torch.empty(wl.n_samples * 16, dtype=torch.uint8, device="cuda")
de = torch.empty(wl.n_events * 16, dtype=torch.uint8, device="cuda")
gen.fill_device("samples", wl, ds.data_ptr(), 0, wl.n_samples)
gen.fill_device("events", wl, de.data_ptr(), 0, wl.n_events)
torch.cuda.synchronize()
mon = Monitor(owner, cap, tot, n_components=wl.n_components, t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k)
t_end = np.ascontiguousarray(wl.t_end())
for _ in range(3):
    mon.reset(); mon.ingest(ds, de); mon.window_reduce(t_end)
T = {"reset": 0, "ingest": 0, "reduce_c": 0, "results": 0}
n = 10
summ = np.zeros(len(t_end), N.SUMMARY_DTYPE)
for _ in range(n):
    a = time.perf_counter(); mon.reset(); b = time.perf_counter(); mon.ingest(ds, de); c = time.perf_counter()
    N.check(N.lib().rtm_window_reduce(mon._h, t_end.ctypes.data, len(t_end), summ.ctypes.data), "r")
    d = time.perf_counter(); mon.W = len(t_end); mon.results(); e = time.perf_counter()
    T["reset"] += b - a; T["ingest"] += c - b; T["reduce_c"] += d - c; T["results"] += e - d
mon.profile(True)
for _ in range(n):
    mon.reset(); mon.ingest(ds, de); mon.window_reduce(t_end)
prof = mon.profile_read()
gpu = sum(v["total_ms"] for v in prof.values()) / n
print({k: round(v / n * 1e3, 3) for k, v in T.items()}, "ms; kernels", round(gpu, 3), "ms")
