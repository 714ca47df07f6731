"""Workload for compute-sanitizer (SURVEY.md §4 "Sanitizers", §5): a C1-shaped trace through the
C-ABI in the launch configurations the tests use — one multi-window call (partition, fold with
look-back, top-k, hang, progress), single-window calls (top-k slices + merge), rank modes SIZE and
MEAN, invalid records, a very sparse call (sequential fold, prefix hang), a windowed call with the
compacted finalize, a two-pass call over window ranges — every result compared with the oracle so
a silent corruption also fails.

    compute-sanitizer --tool memcheck python tools/sanitize.py [--small]
"""
from __future__ import annotations

import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import gen  # noqa: E402
import oracle  # noqa: E402
from paper_conf_micro_mosallaeii024_b200 import Monitor  # noqa: E402


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a).view(np.uint8)).cuda()


def check(got, ref, n_windows):
    for f in ("n_samples", "n_events", "n_dropped", "digest", "n_touched", "n_hung"):
        assert np.array_equal(got["summary"][f], ref["summary"][f]), f
    for w in range(n_windows):
        n = int(ref["topk_n"][w])
        assert np.array_equal(got["topk"][w][:n], ref["topk"][w][:n]), w
    for f in ("started", "finished", "in_flight"):
        assert np.array_equal(got["progress"][f], ref["progress"][f]), f


def main():
    small = "--small" in sys.argv
    ns = 60_000 if small else 300_000
    base = gen.C1_INVALID.scaled("C1-sanitize", n_samples=ns, n_events=ns // 10, n_windows=6)
    owner, cap, tot = gen.registry(base)
    s, e = gen.samples(base), gen.events(base)
    t_end = base.t_end()
    for mode in (0, 1, 2):
        kw = dict(t0=base.t0, hang_windows=2, k=base.k, rank_mode=mode)
        orc = oracle.Oracle(owner, cap, tot, n_components=base.n_components, **kw)
        mon = Monitor(owner, cap, tot, n_components=base.n_components, **kw)
        # one multi-window call, then one window per call
        lo_s, lo_e = base.index_at("samples", base.t_begin(4)), base.index_at("events", base.t_begin(4))
        ref = orc.reduce(s[:lo_s], e[:lo_e], t_end[:4])
        mon.ingest(_dev(s[:lo_s]), _dev(e[:lo_e]))
        check(mon.window_reduce(t_end[:4]), ref, 4)
        for w in (4, 5):
            hs, he = base.index_at("samples", base.t_begin(w + 1)), base.index_at("events", base.t_begin(w + 1))
            ref = orc.reduce(s[lo_s:hs], e[lo_e:he], t_end[w:w + 1])
            mon.ingest(_dev(s[lo_s:hs]), _dev(e[lo_e:he]))
            check(mon.window_reduce(t_end[w:w + 1]), ref, 1)
            lo_s, lo_e = hs, he
        mon.buffer_stats()
        mon.close()
    # a very sparse call (sequential fold) with a long H (prefix hang kernel), 128-buffer bins
    nb = 140_000
    owner2 = (np.arange(nb) // 4).astype(np.uint32)
    cap2 = np.full(nb, 8, np.uint16)
    tot2 = np.full(2, 100, np.int64)
    rng = np.random.default_rng(7)
    m = 4000 if small else 20_000
    ts = np.sort(rng.integers(0, 200_000, m))
    sp = np.zeros(m, gen.SAMPLE_DTYPE)
    sp["ts"], sp["buffer_id"] = ts, rng.integers(0, nb, m)
    sp["level"], sp["capacity"] = rng.integers(0, 9, m), 8
    ends = np.arange(1, 201, dtype=np.int64) * 1000
    kw = dict(t0=0, hang_windows=300, k=16)
    orc = oracle.Oracle(owner2, cap2, tot2, n_components=nb // 4, **kw)
    mon = Monitor(owner2, cap2, tot2, n_components=nb // 4, **kw)
    ref = orc.reduce(sp, np.zeros(0, gen.EVENT_DTYPE), ends)
    mon.ingest(_dev(sp), None)
    check(mon.window_reduce(ends), ref, len(ends))
    # a windowed call with fewer samples than buffer-windows (compacted finalize, 32-bit D)
    cf = gen.C1.scaled("C1-cf-sanitize", n_samples=40_000 if small else 120_000, n_events=4_000, n_buffers=20_000,
                       n_windows=8)
    owner3, cap3, tot3 = gen.registry(cf)
    kw = dict(t0=cf.t0, hang_windows=2, k=cf.k)
    orc = oracle.Oracle(owner3, cap3, tot3, n_components=cf.n_components, **kw)
    mon = Monitor(owner3, cap3, tot3, n_components=cf.n_components, **kw)
    ref = orc.reduce(gen.samples(cf), gen.events(cf), cf.t_end())
    mon.ingest(_dev(gen.samples(cf)), _dev(gen.events(cf)))
    check(mon.window_reduce(cf.t_end()), ref, 8)
    # a very sparse two-pass call of >= 128 windows: the sequential fold over window ranges
    # (k_subpart's end keys) with its batched finalize queue
    nb4 = 262_144
    owner4 = (np.arange(nb4) // 4).astype(np.uint32)
    cap4 = np.full(nb4, 16, np.uint16)
    m4 = 6000 if small else 20_000
    ts4 = np.sort(rng.integers(0, 130_000, m4))
    s4 = np.zeros(m4, gen.SAMPLE_DTYPE)
    s4["ts"], s4["buffer_id"] = ts4, rng.integers(0, nb4, m4)
    s4["level"], s4["capacity"] = rng.integers(0, 17, m4), 16
    ends4 = np.arange(1, 131, dtype=np.int64) * 1000
    kw = dict(t0=0, hang_windows=4, k=16)
    orc = oracle.Oracle(owner4, cap4, tot2, n_components=nb4 // 4, **kw)
    mon = Monitor(owner4, cap4, tot2, n_components=nb4 // 4, **kw)
    ref = orc.reduce(s4, np.zeros(0, gen.EVENT_DTYPE), ends4)
    mon.ingest(_dev(s4), None)
    check(mon.window_reduce(ends4), ref, len(ends4))
    mon.close()
    print("sanitize workload OK")


if __name__ == "__main__":
    main()
