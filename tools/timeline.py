"""Device timeline of reduce calls (CUPTI through torch.profiler): every kernel, memcpy and memset
of the last `--calls` calls with its start, duration and the idle gap before it, so host-side
stalls between launches show up (the per-kernel event timers cannot see them).

    python tools/timeline.py --config C5-long --windows 1000 --calls 2 > gpurun_out/tl.txt
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import gen  # noqa: E402
from paper_conf_micro_mosallaeii024_b200 import Monitor  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C5-long")
ap.add_argument("--windows", type=int, default=1000, help="windows per call")
ap.add_argument("--calls", type=int, default=2)
ap.add_argument("--warmup", type=int, default=2)
ap.add_argument("--trace", default="")
ap.add_argument("--graphs", type=int, default=1, help="rtm_use_graphs mode: 0 off, 1 auto, 2 always")
args = ap.parse_args()
wl = gen.CONFIGS[args.config]
W = args.windows
n_calls = args.warmup + args.calls
ns = wl.index_at("samples", wl.t_begin(W * n_calls))
ne = wl.index_at("events", wl.t_begin(W * n_calls))
ds = torch.empty(max(1, ns) * 16, dtype=torch.uint8, device="cuda")
de = torch.empty(max(1, ne) * 16, dtype=torch.uint8, device="cuda")
gen.fill_device("samples", wl, ds.data_ptr(), 0, ns)
gen.fill_device("events", wl, de.data_ptr(), 0, ne)
torch.cuda.synchronize()
owner, cap, tot = gen.registry(wl)
mon = Monitor(owner, cap, tot, n_components=wl.n_components, t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k)
mon.use_graphs(args.graphs)


def call(i):
    s0, s1 = wl.index_at("samples", wl.t_begin(i * W)), wl.index_at("samples", wl.t_begin((i + 1) * W))
    e0, e1 = wl.index_at("events", wl.t_begin(i * W)), wl.index_at("events", wl.t_begin((i + 1) * W))
    mon.ingest(ds[s0 * 16:s1 * 16], de[e0 * 16:e1 * 16])
    return mon.window_reduce(wl.t_end(i * W, W))


for i in range(args.warmup):
    call(i)
torch.cuda.synchronize()
from torch.profiler import ProfilerActivity, profile  # noqa: E402

with profile(activities=[ProfilerActivity.CPU, ProfilerActivity.CUDA]) as prof:
    for i in range(args.warmup, n_calls):
        call(i)
    torch.cuda.synchronize()
path = args.trace or os.path.join(ROOT, "gpurun_out", "timeline_trace.json")
prof.export_chrome_trace(path)
ev = json.load(open(path))["traceEvents"]
dev = [e for e in ev if e.get("cat") in ("kernel", "gpu_memcpy", "gpu_memset") and "dur" in e]
dev.sort(key=lambda e: e["ts"])
t0 = dev[0]["ts"] if dev else 0
last_end = t0
agg = {}
print(f"{'start_us':>10} {'dur_us':>9} {'gap_us':>8} stream name")
for e in dev:
    gap = e["ts"] - last_end
    name = e["name"].split("(")[0].split("::")[-1][:60]
    print(f"{e['ts'] - t0:10.1f} {e['dur']:9.1f} {gap:8.1f} {e['args'].get('stream', '?'):>6} {name}")
    last_end = max(last_end, e["ts"] + e["dur"])
    a = agg.setdefault(name, [0, 0.0])
    a[0] += 1
    a[1] += e["dur"]
span = last_end - t0
busy = sum(v[1] for v in agg.values())
print(json.dumps({"calls": args.calls, "span_us": round(span, 1), "sum_dur_us": round(busy, 1),
                  "per_name_us": {k: [v[0], round(v[1], 1)] for k, v in sorted(agg.items(), key=lambda x: -x[1][1])}}))
