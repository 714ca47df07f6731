"""Device-timed window_reduce over C2-sized traces with different buffer counts (partition path
selection): python tools/shape_bench.py [n_buffers ...]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import gen  # noqa: E402
from paper_conf_micro_mosallaeii024_b200 import Monitor  # noqa: E402

sizes = [int(x) for x in sys.argv[1:]] or [20480, 32768, 40960, 81920]
for nb in sizes:
    wl = gen.C2.scaled(f"C2-{nb}", n_buffers=nb)
    owner, cap, tot = gen.registry(wl)
    ds = torch.empty(wl.n_samples * 16, dtype=torch.uint8, device="cuda")
    de = torch.empty(wl.n_events * 16, dtype=torch.uint8, device="cuda")
    gen.fill_device("samples", wl, ds.data_ptr(), 0, wl.n_samples)
    gen.fill_device("events", wl, de.data_ptr(), 0, wl.n_events)
    mon = Monitor(owner, cap, tot, n_components=wl.n_components, t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k)
    t_end = wl.t_end()
    for _ in range(3):
        mon.reset(); mon.ingest(ds, de); mon.window_reduce(t_end)
    mon.profile(True)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); a.record()
    for _ in range(10):
        mon.reset(); mon.ingest(ds, de); mon.window_reduce(t_end)
    b.record(); torch.cuda.synchronize()
    ms = a.elapsed_time(b) / 10
    prof = mon.profile_read()
    ks = {k: round(v["total_ms"] / 10, 3) for k, v in prof.items() if v["launches"]}
    print(f"n_buffers={nb} bins={(nb + 255) // 256} {ms:.3f} ms/step {(wl.n_samples + wl.n_events) / ms / 1e6:.1f} G rec/s {ks}")
    del mon, ds, de
    torch.cuda.empty_cache()
