"""BASELINE.json configs[4] (C5) at full size on one B200: 16 simulated GPUs, 327 680 buffers,
7.2B samples + 0.8B events (128 GB of records) in 1 000 000 windows.

The trace does not fit in HBM at once, so it is streamed: every batch of `--batch` windows is
generated on the device (counter-based generator, gen/), ingested and reduced with ONE
`rtm_window_reduce` call; the context carries levels, counts and hang runs across calls.  The GPU
pass keeps every window's summary (counts, drops, digest over every touched buffer, n_touched,
n_hung), a hash of every batch's progress table and of its top-k lists, the full top-k / hang lists
of sampled windows and the last window's per-buffer table.

`--oracle` then streams the same trace through the CPU oracle (oracle/, host generator) batch by
batch and checks every window's summary, every batch's progress table (hash), the sampled windows'
top-k and hang lists and the final per-buffer table (the oracle's full-sort top-k of 327 680
buffers is its slow part, so it runs on sampled windows only).  Test infrastructure: this tool is
one of the places allowed to call oracle/.

    python tools/c5_full.py --windows 1000000 --batch 1000 --oracle --out gpurun_out/c5_full.json
"""
from __future__ import annotations

import argparse
import hashlib
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gen  # noqa: E402

SUM_FIELDS = ("t_begin", "t_end", "n_samples", "n_events", "n_dropped", "digest", "n_touched", "n_hung")


def batches(n_windows, batch):
    for w0 in range(0, n_windows, batch):
        yield w0, min(n_windows, w0 + batch)


def ranges(wl, w0, w1):
    s_lo, s_hi = wl.index_at("samples", wl.t_begin(w0)), wl.index_at("samples", wl.t_begin(w1))
    e_lo, e_hi = wl.index_at("events", wl.t_begin(w0)), wl.index_at("events", wl.t_begin(w1))
    return s_lo, s_hi, e_lo, e_hi


def h(a) -> str:
    return hashlib.blake2b(np.ascontiguousarray(a).tobytes(), digest_size=16).hexdigest()


def gpu_pass(wl, n_windows, batch, sampled, checkpoints):
    import torch

    from paper_conf_micro_mosallaeii024_b200 import Monitor

    owner, cap, tot = gen.registry(wl)
    mon = Monitor(owner, cap, tot, n_components=wl.n_components, t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k)
    if os.environ.get("C5_PROFILE"):
        mon.profile(True)
    max_s = max(ranges(wl, a, b)[1] - ranges(wl, a, b)[0] for a, b in [(0, batch), (n_windows - batch, n_windows)])
    max_e = max(ranges(wl, a, b)[3] - ranges(wl, a, b)[2] for a, b in [(0, batch), (n_windows - batch, n_windows)])
    ds = torch.empty((max_s + 4096) * 16, dtype=torch.uint8, device="cuda")
    de = torch.empty((max_e + 4096) * 16, dtype=torch.uint8, device="cuda")
    summ = []
    prog_h, top_h, tops, hung, prog = [], [], {}, {}, {}
    t_reduce = 0.0
    t_gen = 0.0
    n_rec = 0
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    dev_ms = 0.0
    for w0, w1 in batches(n_windows, batch):
        s_lo, s_hi, e_lo, e_hi = ranges(wl, w0, w1)
        t = time.perf_counter()
        gen.fill_device("samples", wl, ds.data_ptr(), s_lo, s_hi - s_lo)
        gen.fill_device("events", wl, de.data_ptr(), e_lo, e_hi - e_lo)
        torch.cuda.synchronize()
        t_gen += time.perf_counter() - t
        t = time.perf_counter()
        ev0.record()
        mon.ingest(ds[:(s_hi - s_lo) * 16], de[:(e_hi - e_lo) * 16])
        got = mon.window_reduce(wl.t_end(w0, w1 - w0))
        ev1.record()
        torch.cuda.synchronize()
        t_reduce += time.perf_counter() - t
        dev_ms += ev0.elapsed_time(ev1)
        n_rec += (s_hi - s_lo) + (e_hi - e_lo)
        summ.append(np.array(got["summary"]))
        prog_h.append(h(got["progress"]))
        for w in range(w0, w1):
            if w in checkpoints:
                prog[w] = np.array(got["progress"][w - w0])
        top_h.append(h(np.concatenate([got["topk_n"].view(np.uint8), got["topk"].view(np.uint8).ravel()])))
        for w in sampled:
            if w0 <= w < w1:
                n = int(got["topk_n"][w - w0])
                tops[w] = np.array(got["topk"][w - w0][:n])
                hung[w] = mon.hang_check(w - w0)
    stats = mon.buffer_stats()
    summ = np.concatenate(summ)
    if os.environ.get("C5_PROFILE"):
        print(json.dumps({k: round(v["total_ms"], 2) for k, v in mon.profile_read().items() if v["launches"]}))
    out = {
        "records": n_rec, "windows": n_windows, "batch": batch, "calls": len(prog_h),
        "reduce_wall_s": t_reduce, "reduce_device_s": dev_ms / 1e3, "gen_s": t_gen,
        "records_per_s_device": n_rec / (dev_ms / 1e3), "records_per_s_wall": n_rec / t_reduce,
        "n_hung_total": int(summ["n_hung"].sum()), "windows_with_hung": int((summ["n_hung"] > 0).sum()),
        "n_touched_mean": float(summ["n_touched"].mean()),
    }
    return out, summ, prog, top_h, tops, hung, stats


def _oracle_range(args):
    """One worker of the parallel oracle pass: windows [a, b) of the trace.  The oracle's context
    is brought to window a by replaying the prefix: records before window a - H as coarse windows
    of `coarse` real windows each (levels, cumulative START / END counts and t_prev only depend on
    the records, not on how they are cut into windows), then the H windows before a one by one, so
    every hang run that matters (run >= H decides a flag) is rebuilt exactly.  Then [a, b) in
    batches; sampled windows get their own call with top-k and hang lists."""
    wl, a, b, batch, sampled, checkpoints, coarse, n_total = args
    import oracle

    owner, cap, tot = gen.registry(wl)
    orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, t0=wl.t0, hang_windows=wl.hang_windows,
                        k=wl.k)
    H = wl.hang_windows
    ws = max(0, a - H)

    def run(w0, w1, t_end, **kw):
        s_lo, s_hi, e_lo, e_hi = ranges(wl, w0, w1)
        ref = orc.reduce(gen.samples(wl, s_lo, s_hi - s_lo), gen.events(wl, e_lo, e_hi - e_lo), t_end, **kw)
        assert ref["rc"] == 0, (w0, ref["rc"])
        return ref

    for c0 in range(0, ws, coarse):  # prefix as coarse windows
        c1 = min(ws, c0 + coarse)
        run(c0, c1, np.array([wl.t_begin(c1)], np.int64), want_hung=False, want_topk=False)
    for w0 in range(ws, a, batch):  # hang-run warm-up
        w1 = min(a, w0 + batch)
        run(w0, w1, wl.t_end(w0, w1 - w0), want_hung=False, want_topk=False)
    summ, prog, tops, hung, stats = [], {}, {}, {}, None
    cuts = sorted({a, b} | set(range(a - a % batch + batch, b, batch)) | {w for w in sampled if a <= w < b}
                  | {w + 1 for w in sampled if a <= w < b})
    for w0, w1 in zip(cuts[:-1], cuts[1:]):
        samp = w0 in sampled
        ref = run(w0, w1, wl.t_end(w0, w1 - w0), want_hung=samp, want_topk=samp)
        summ.append(ref["summary"])
        for w in range(w0, w1):
            if w in checkpoints:
                prog[w] = np.array(ref["progress"][w - w0])
        if samp:
            n = int(ref["topk_n"][0])
            tops[w0] = np.array(ref["topk"][0][:n])
            hung[w0] = np.nonzero(ref["hung"][0])[0].astype(np.uint32)
        if w1 == n_total:
            stats = ref["stats"]
    return a, b, np.concatenate(summ), prog, tops, hung, stats


def oracle_pass(wl, n_windows, batch, sampled, checkpoints, g_summ, g_prog, g_tops, g_hung, g_stats, workers):
    import multiprocessing as mp

    bounds = [round(i * n_windows / workers) for i in range(workers + 1)]
    jobs = [(wl, bounds[i], bounds[i + 1], batch, set(sampled), set(checkpoints), 2000, n_windows)
            for i in range(workers) if bounds[i] < bounds[i + 1]]
    bad = []
    with mp.get_context("spawn").Pool(len(jobs)) as pool:
        outs = pool.map(_oracle_range, jobs)
    for a, b, summ, prog, tops, hung, stats in outs:
        for f in SUM_FIELDS:
            if not np.array_equal(g_summ[f][a:b], summ[f]):
                i = int(np.nonzero(g_summ[f][a:b] != summ[f])[0][0])
                bad.append(("summary", f, a + i))
        for w, row in prog.items():
            if not np.array_equal(g_prog[w], row):
                bad.append(("progress", w))
        for w, t in tops.items():
            if not np.array_equal(g_tops[w], t):
                bad.append(("topk", w))
        for w, x in hung.items():
            if not np.array_equal(g_hung[w], x):
                bad.append(("hung", w))
        if stats is not None:
            for f in ("integral", "last", "max", "min", "capacity", "n_samples"):
                if not np.array_equal(g_stats[f], stats[f]):
                    bad.append(("stats", f))
            if not np.array_equal(g_stats["mean_occ"], stats["mean_occ"]):
                bad.append(("stats", "mean_occ"))
    return {"oracle_ok": not bad, "mismatches": [list(map(str, x)) for x in bad[:20]],
            "topk_windows_checked": sum(len(o[4]) for o in outs),
            "progress_windows_checked": sum(len(o[3]) for o in outs),
            "summary_windows_checked": sum(len(o[2]) for o in outs), "oracle_workers": len(jobs)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--windows", type=int, default=gen.C5.n_windows)
    ap.add_argument("--batch", type=int, default=1000)
    ap.add_argument("--hang-windows", type=int, default=0)
    ap.add_argument("--oracle", action="store_true")
    ap.add_argument("--workers", type=int, default=max(1, (os.cpu_count() or 2) - 1))
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    wl = gen.C5
    if a.hang_windows:
        wl = wl.scaled(wl.name, hang_windows=a.hang_windows)
    W = a.windows
    sampled = sorted({0, 1, a.batch - 1, a.batch, W // 3, W // 2 + 7, W - 2, W - 1} & set(range(W)))
    t = time.perf_counter()
    checkpoints = set(range(a.batch - 1, W, a.batch)) | set(sampled) | {W - 1}
    res, summ, prog, top_h, tops, hung, stats = gpu_pass(wl, W, a.batch, sampled, checkpoints)
    res["gpu_pass_s"] = time.perf_counter() - t
    res["hang_windows"] = wl.hang_windows
    res["sampled_windows"] = sampled
    print(json.dumps(res), flush=True)
    if a.oracle:
        t = time.perf_counter()
        res.update(oracle_pass(wl, W, a.batch, sampled, checkpoints, summ, prog, tops, hung, stats, a.workers))
        res["oracle_pass_s"] = time.perf_counter() - t
        print(json.dumps({k: v for k, v in res.items() if k.startswith(("oracle", "mismatch")) or k.endswith("checked")}),
              flush=True)
    if a.out:
        with open(a.out, "w") as f:
            json.dump(res, f, indent=1)
    return 0 if res.get("oracle_ok", True) else 1


if __name__ == "__main__":
    sys.exit(main())
