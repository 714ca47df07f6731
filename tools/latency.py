"""Per-window snapshot latency in streaming mode: one window per
rtm_window_reduce call, its records already in HBM, the call timed on the host from launch to
results on the host (the call blocks until its D2H is done).  Reports p50 / p99 over the first
`--windows` windows of the chosen config.

    python tools/latency.py --config C5-long --windows 2000
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
from paper_conf_micro_mosallaeii024_b200 import Monitor  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C5-long")
ap.add_argument("--windows", type=int, default=2000)
ap.add_argument("--warmup", type=int, default=50)
ap.add_argument("--graphs", type=int, default=1, help="rtm_use_graphs mode: 0 off, 1 auto (default), 2 always")
args = ap.parse_args()
wl = gen.CONFIGS[args.config]
W = args.windows + args.warmup
ns = wl.index_at("samples", wl.t_begin(W))
ne = wl.index_at("events", wl.t_begin(W))
ds = torch.empty(max(1, ns) * 16, dtype=torch.uint8, device="cuda")
de = torch.empty(max(1, ne) * 16, dtype=torch.uint8, device="cuda")
gen.fill_device("samples", wl, ds.data_ptr(), 0, ns)
gen.fill_device("events", wl, de.data_ptr(), 0, ne)
torch.cuda.synchronize()
owner, cap, tot = gen.registry(wl)
mon = Monitor(owner, cap, tot, n_components=wl.n_components, t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k)
mon.use_graphs(args.graphs)
t_end = wl.t_end(0, W)
lat = []
recs = 0
# the windows' record ranges (the generator's index math and the tensor views) are prepared before
# the timed calls: a call is timed from the ingest of its records to its results on the host
views = []
for w in range(W):
    s0, s1 = wl.index_at("samples", wl.t_begin(w)), wl.index_at("samples", wl.t_begin(w + 1))
    e0, e1 = wl.index_at("events", wl.t_begin(w)), wl.index_at("events", wl.t_begin(w + 1))
    views.append((ds[s0 * 16:s1 * 16], de[e0 * 16:e1 * 16], t_end[w:w + 1], (s1 - s0) + (e1 - e0)))
for w in range(W):
    sv, ev, te, nrec = views[w]
    t = time.perf_counter()
    mon.ingest(sv, ev)
    res = mon.window_reduce(te)
    dt = time.perf_counter() - t
    if w >= args.warmup:
        lat.append(dt)
        recs += nrec
    assert int(res["summary"]["n_dropped"][0]) == 0
lat = np.array(lat) * 1e6
# per-kernel device time of a call (CUDA events around each launch, library profiler)
mon.profile(True)
n_prof = min(200, W)
mon.reset()
for w in range(n_prof):
    s0, s1 = wl.index_at("samples", wl.t_begin(w)), wl.index_at("samples", wl.t_begin(w + 1))
    e0, e1 = wl.index_at("events", wl.t_begin(w)), wl.index_at("events", wl.t_begin(w + 1))
    mon.ingest(ds[s0 * 16:s1 * 16], de[e0 * 16:e1 * 16])
    mon.window_reduce(t_end[w:w + 1])
prof = {k: round(v["total_ms"] * 1e3 / n_prof, 2) for k, v in mon.profile_read().items() if v["launches"]}
mon.profile(False)
print(json.dumps({"what": "per-window snapshot latency, one window per call (streaming)", "config": wl.name,
                  "n_buffers": wl.n_buffers, "windows": args.windows, "graphs": args.graphs, "records_per_window": recs / args.windows,
                  "p50_us": float(np.percentile(lat, 50)), "p99_us": float(np.percentile(lat, 99)),
                  "mean_us": float(lat.mean()), "records_per_s": recs / (lat.sum() / 1e6),
                  "kernel_us_per_call": prof}))
