"""Hang-window calibration: for a config, the number of components flagged in
the injection-free trace at each candidate H.  The chosen H is the smallest candidate that flags
nothing; the full-size parity tests then confirm it against the oracle (nothing but the injected
components is ever flagged).

    python tools/calibrate_h.py C3-clean 24 32 40 48 64
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
from paper_conf_micro_mosallaeii024_b200 import Monitor  # noqa: E402

wl = gen.CONFIGS[sys.argv[1]]
Hs = [int(x) for x in sys.argv[2:]] or [8, 16, 32, 48, 64]
owner, cap, tot = gen.registry(wl)
ds = torch.empty(wl.n_samples * 16, dtype=torch.uint8, device="cuda")
de = torch.empty(wl.n_events * 16, dtype=torch.uint8, device="cuda")
gen.fill_device("samples", wl, ds.data_ptr(), 0, wl.n_samples)
gen.fill_device("events", wl, de.data_ptr(), 0, wl.n_events)
torch.cuda.synchronize()
injected = {c for _, cs in wl.deadlock for c in cs}
for H in Hs:
    mon = Monitor(owner, cap, tot, n_components=wl.n_components, t0=wl.t0, hang_windows=H, k=wl.k)
    mon.ingest(ds, de)
    res = mon.window_reduce(wl.t_end())
    flagged = set()
    for w in np.nonzero(res["summary"]["n_hung"])[0]:
        flagged |= set(mon.hang_check(int(w)).tolist())
    print(f"{wl.name} H={H}: flagged components {len(flagged - injected)} (+{len(flagged & injected)} injected), "
          f"component-windows {int(res['summary']['n_hung'].sum())}", flush=True)
    del mon
