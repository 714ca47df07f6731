"""GPU parity on BASELINE.json configs C3 (injected deadlock) and C4 (Zipf skew).

The CUDA path runs each trace in ONE `rtm_window_reduce` call over all windows (the launch
configuration bench.py times); the oracle then streams the same trace window batch by window
batch (its context carries state across calls, so the batching does not change its results) and
every window is compared: summaries (counts, drops, digest over every touched buffer), progress
bars, hang lists; top-k lists on every window of the small variants and on a fixed sample of
windows at full size (a full-sort top-k of 80k / 1M buffers per window is the oracle's slow
part); the per-buffer table of the last window in full.
"""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_micro_mosallaeii024_b200 import Monitor  # noqa: E402

SUM_FIELDS = ("t_begin", "t_end", "n_samples", "n_events", "n_dropped", "digest", "n_touched", "n_hung")


def _device_trace(wl):
    ds = torch.empty(wl.n_samples * 16, dtype=torch.uint8, device="cuda")
    de = torch.empty(wl.n_events * 16, dtype=torch.uint8, device="cuda")
    gen.fill_device("samples", wl, ds.data_ptr(), 0, wl.n_samples)
    gen.fill_device("events", wl, de.data_ptr(), 0, wl.n_events)
    torch.cuda.synchronize()
    return ds, de


def _host_slice(dev, lo, hi, dtype):
    """Records [lo, hi) of a device trace as a host structured array (input copy, not a result)."""
    return dev[lo * 16:hi * 16].cpu().numpy().view(dtype)


def run_config(wl, *, batch, topk_windows=None, rank_mode=0):
    """GPU: one call over all windows.  Oracle: batches of `batch` windows.  Returns the
    per-window hang lists of the oracle for property checks.  When every window's top-k is
    compared, the windows-in-top-k counter (persistence) is compared too."""
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k, rank_mode=rank_mode)
    ds, de = _device_trace(wl)
    # the device generator writes the same records as the host one (spot check)
    idx = np.random.default_rng(1).integers(0, wl.n_samples, 2048)
    assert np.array_equal(ds.view(-1, 16)[torch.from_numpy(idx).cuda()].cpu().numpy().view(gen.SAMPLE_DTYPE).ravel(),
                          gen.samples(wl)[idx] if wl.n_samples <= 20_000_000 else
                          np.concatenate([gen.samples(wl, int(i), 1) for i in idx]))
    mon = Monitor(owner, cap, tot, n_components=wl.n_components, **kw)
    mon.ingest(ds, de)
    t_end = wl.t_end()
    got = mon.window_reduce(t_end)
    gsum, gtop, gtopn, gprog = got["summary"], got["topk"], got["topk_n"], got["progress"]
    stats = mon.buffer_stats()
    _, comps = mon.progress(wl.n_windows - 1, comps=True)
    ghung = [mon.hang_check(w) for w in range(wl.n_windows)]
    gpersist = mon.topk_persistence()
    del mon

    orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, **kw)
    hung_ref = []
    want = set(range(wl.n_windows)) if topk_windows is None else set(topk_windows)
    for w0 in range(0, wl.n_windows, batch):
        w1 = min(wl.n_windows, w0 + batch)
        s_lo, s_hi = wl.index_at("samples", wl.t_begin(w0)), wl.index_at("samples", wl.t_begin(w1))
        e_lo, e_hi = wl.index_at("events", wl.t_begin(w0)), wl.index_at("events", wl.t_begin(w1))
        s = _host_slice(ds, s_lo, s_hi, gen.SAMPLE_DTYPE)
        e = _host_slice(de, e_lo, e_hi, gen.EVENT_DTYPE)
        tk = any(w in want for w in range(w0, w1))
        ref = orc.reduce(s, e, t_end[w0:w1], want_topk=tk)
        assert ref["rc"] == 0
        for f in SUM_FIELDS:
            assert np.array_equal(gsum[f][w0:w1], ref["summary"][f]), (f, w0)
        for f in ("total", "started", "finished", "in_flight", "not_started"):
            assert np.array_equal(gprog[f][w0:w1], ref["progress"][f]), (f, w0)
        for w in range(w0, w1):
            hr = np.nonzero(ref["hung"][w - w0])[0].astype(np.uint32)
            assert np.array_equal(ghung[w], hr), w
            hung_ref.append(hr)
            if tk and w in want:
                n = int(ref["topk_n"][w - w0])
                assert int(gtopn[w]) == n, w
                assert np.array_equal(gtop[w][:n], ref["topk"][w - w0][:n]), w
        if w1 == wl.n_windows:
            rs = ref["stats"]
            for f in ("integral", "last", "max", "min", "capacity", "n_samples"):
                assert np.array_equal(stats[f], rs[f]), f
            assert np.array_equal(stats["mean_occ"], rs["mean_occ"])
            for f in ("started", "finished", "in_flight"):
                assert np.array_equal(comps[f], ref["comps"][f]), f
    if topk_windows is None:
        assert np.array_equal(gpersist, orc.persistence())
    return hung_ref


def check_deadlock_flags(wl, hung):
    """Case study 2: every injected component is flagged from window
    w_d + H - 1 on (it may be flagged up to `deadlock_lead` windows earlier when it happened to be
    silent while its buffers were already held full), never before w_d + H - 1 - lead; nothing
    else is ever flagged (H is large enough that the injection-free trace flags nothing)."""
    H, lead = wl.hang_windows, wl.deadlock_lead
    injected = {c for _, cs in wl.deadlock for c in cs}
    for w_d, cs in wl.deadlock:
        for c in cs:
            first = next(w for w in range(wl.n_windows) if c in hung[w])
            assert w_d + H - 1 - lead <= first <= w_d + H - 1, (c, first)
            assert all(c in hung[w] for w in range(w_d + H - 1, wl.n_windows)), c
    others = set().union(*[set(h.tolist()) for h in hung]) - injected
    assert not others, sorted(others)[:10]


def test_c3_small_deadlock_parity():
    hung = run_config(gen.C3_SMALL, batch=25)
    check_deadlock_flags(gen.C3_SMALL, hung)


@pytest.mark.parametrize("rank_mode", [0, 1, 2])
def test_c4_small_zipf_parity(rank_mode):
    """C4's shape (2^20 buffers, Zipf 0.99, k = 1024) in every rank mode: MEAN ranks 1M 64-bit
    order keys per window (k_topk64's uncompacted large-n path)."""
    run_config(gen.C4_SMALL, batch=5, rank_mode=rank_mode)


@pytest.mark.slow
def test_c3_full_size_parity():
    """BASELINE configs[2] at full size: 1B records, 81920 buffers, 10k windows, deadlock at 6000."""
    wl = gen.C3
    sample = sorted(set(range(0, wl.n_windows, 250)) | {5999, 6000, 6005, 6038, 6039, 6044, wl.n_windows - 1})
    hung = run_config(wl, batch=250, topk_windows=sample)
    check_deadlock_flags(wl, hung)


@pytest.mark.slow
def test_c4_full_size_parity():
    """BASELINE configs[3] at full size: 2B records, 1M buffers (Zipf 0.99), k = 1024."""
    wl = gen.C4
    sample = [0, 1, 999, 1000, wl.n_windows - 1]
    run_config(wl, batch=50, topk_windows=sample)


def test_c5_first_windows_parity():
    """BASELINE configs[4] (16 simulated GPUs, 327680 buffers, 1M windows of ~8k records): its
    first 1000 windows (8M records) in one call, every window checked.  The full 1M-window run
    (128 GB, streamed in 1000 calls) is `tools/c5_full.py` against a range-parallel oracle
    (~10 min on 15 cores; profiles/r01_c5_full.json)."""
    wl = gen.C5
    n_win = 1000
    ns = wl.index_at("samples", wl.t_begin(n_win))
    ne = wl.index_at("events", wl.t_begin(n_win))
    part = wl.scaled("C5-slice", n_samples=ns, n_events=ne)
    # the slice's records are the full trace's first records (index-addressed generator)
    ds = torch.empty(ns * 16, dtype=torch.uint8, device="cuda")
    de = torch.empty(ne * 16, dtype=torch.uint8, device="cuda")
    gen.fill_device("samples", wl, ds.data_ptr(), 0, ns)
    gen.fill_device("events", wl, de.data_ptr(), 0, ne)
    torch.cuda.synchronize()
    s, e = gen.samples(wl, 0, ns), gen.events(wl, 0, ne)
    assert np.array_equal(ds.cpu().numpy().view(gen.SAMPLE_DTYPE)[:4096], s[:4096])
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k)
    t_end = wl.t_end(0, n_win)
    mon = Monitor(owner, cap, tot, n_components=wl.n_components, **kw)
    mon.ingest(ds, de)
    got = mon.window_reduce(t_end)
    ref = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, **kw).reduce(s, e, t_end)
    assert ref["rc"] == 0
    for f in SUM_FIELDS:
        assert np.array_equal(got["summary"][f], ref["summary"][f]), f
    assert np.array_equal(got["topk_n"], ref["topk_n"])
    assert np.array_equal(got["topk"], ref["topk"])
    for f in ("total", "started", "finished", "in_flight", "not_started"):
        assert np.array_equal(got["progress"][f], ref["progress"][f]), f
    for w in range(0, n_win, 37):
        assert np.array_equal(mon.hang_check(w), np.nonzero(ref["hung"][w])[0].astype(np.uint32)), w
    st = mon.buffer_stats()
    for f in ("integral", "last", "max", "min", "capacity", "n_samples"):
        assert np.array_equal(st[f], ref["stats"][f]), f
    del part
