"""GPU parity: the CUDA path (through the C-ABI) vs the CPU oracle, element by element.

Integer outputs must be bit-exact; mean occupancy must agree within 1e-12 relative
(BASELINE.json north_star) — the path uses the same single IEEE division, so it is exact.
"""
from __future__ import annotations

import numpy as np
import pytest

import gen
import oracle
from tests.helpers import event_array, random_tiny_case, sample_array

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_micro_mosallaeii024_b200 import Monitor, RTMError  # noqa: E402
from paper_conf_micro_mosallaeii024_b200 import _native as N  # noqa: E402

SUM_FIELDS = ("t_begin", "t_end", "n_samples", "n_events", "n_dropped", "digest", "n_touched", "n_hung")


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a).view(np.uint8)).cuda()


def _pair(owner, cap, tot, nc, **kw):
    orc = oracle.Oracle(owner, cap, tot, n_components=nc, **kw)
    mon = Monitor(owner, cap, tot, n_components=nc, **kw)
    return orc, mon


def assert_same(got, ref, mon, *, stats=True, comps=True, hung=True):
    W = len(ref["summary"])
    for f in SUM_FIELDS:
        assert np.array_equal(got["summary"][f], ref["summary"][f]), (f, got["summary"][f], ref["summary"][f])
    assert np.array_equal(got["topk_n"], ref["topk_n"])
    for w in range(W):
        n = int(ref["topk_n"][w])
        assert np.array_equal(got["topk"][w][:n], ref["topk"][w][:n]), w
    for f in ("total", "started", "finished", "in_flight", "not_started"):
        assert np.array_equal(got["progress"][f], ref["progress"][f]), f
    for w in (0, W - 1):  # single-window accessors agree with the bulk one
        assert np.array_equal(mon.topk(w), got["topk"][w][: int(got["topk_n"][w])])
        assert np.array_equal(mon.progress(w), got["progress"][w])
    if hung:
        for w in range(W):
            assert np.array_equal(mon.hang_check(w), np.nonzero(ref["hung"][w])[0].astype(np.uint32)), w
    if stats:
        st = mon.buffer_stats()
        rs = ref["stats"]
        for f in ("integral", "last", "max", "min", "capacity", "n_samples"):
            assert np.array_equal(st[f], rs[f]), f
        np.testing.assert_allclose(st["mean_occ"], rs["mean_occ"], rtol=1e-12, atol=0)
        assert np.array_equal(st["mean_occ"], rs["mean_occ"])  # same single IEEE division
    if comps:
        _, cs = mon.progress(W - 1, comps=True)
        for f in ("started", "finished", "in_flight"):
            assert np.array_equal(cs[f], ref["comps"][f]), f


# ---------------------------------------------------------------------------------------------
@pytest.mark.parametrize("seed", range(40))
def test_random_tiny_traces(seed):
    rng = np.random.default_rng(5000 + seed)
    case = random_tiny_case(rng, allow_disorder=(seed % 5 == 4))
    kw = dict(t0=case["t0"], hang_windows=case["H"], k=case["k"], rank_mode=case["mode"])
    orc, mon = _pair(case["owner"], case["caps"], case["totals"], case["nc"], **kw)
    for srows, erows, ends in case["calls"]:
        s, e = sample_array(srows), event_array(erows)
        ref = orc.reduce(s, e, ends)
        mon.ingest(_dev(s) if len(s) else None, _dev(e) if len(e) else None)
        if ref["rc"] == -4:
            with pytest.raises(RTMError) as ei:
                mon.window_reduce(ends)
            assert ei.value.code == N.RTM_E_ORDER
            break
        got = mon.window_reduce(ends)
        assert_same(got, ref, mon)


def test_fig3_and_size_mode():
    size = [8, 8, 8, 8, 8, 8, 7, 4, 4, 4, 4, 4]
    cap = np.array([8] * 7 + [4] * 5, np.uint16)
    s = sample_array([(i, i, size[i], int(cap[i])) for i in range(12)])
    for mode, expected in ((1, list(range(12))), (0, [0, 1, 2, 3, 4, 5, 7, 8, 9, 10, 11, 6])):
        mon = Monitor(np.arange(12, dtype=np.uint32), cap, np.ones(1, np.int64), n_components=12, t0=0,
                      hang_windows=1, k=12, rank_mode=mode)
        mon.ingest(_dev(s), None)
        got = mon.window_reduce([100])
        assert [int(x) for x in got["topk"][0]["buffer_id"]] == expected


def test_c1_full_parity():
    wl = gen.C1
    owner, cap, tot = gen.registry(wl)
    s, e = gen.samples(wl), gen.events(wl)
    kw = dict(t0=wl.t0, hang_windows=2, k=wl.k)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    ref = orc.reduce(s, e, wl.t_end())
    mon.ingest(_dev(s), _dev(e))
    got = mon.window_reduce(wl.t_end())
    assert_same(got, ref, mon)
    assert int(ref["summary"]["n_hung"].sum()) >= 0


def test_c1_invalid_records_parity():
    wl = gen.C1_INVALID
    owner, cap, tot = gen.registry(wl)
    s, e = gen.samples(wl), gen.events(wl)
    orc, mon = _pair(owner, cap, tot, wl.n_components, t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k)
    # windows starting after t0 and ending before the trace end: late and early drops too
    ends = wl.t_end()[2:8]
    orc.reduce(s[:0], e[:0], [wl.t_end()[1]])
    mon.ingest(None, None)
    mon.window_reduce([wl.t_end()[1]])
    ref = orc.reduce(s, e, ends)
    mon.ingest(_dev(s), _dev(e))
    got = mon.window_reduce(ends)
    assert int(ref["summary"]["n_dropped"].sum()) > 0
    assert_same(got, ref, mon)


def test_windows_one_call_each_full_tables():
    """Every window's full per-buffer table (reduce one window per call) and batch invariance."""
    wl = gen.C1.scaled("C1-small", n_samples=300_000, n_events=30_000, n_buffers=900, n_windows=12)
    owner, cap, tot = gen.registry(wl)
    s, e = gen.samples(wl), gen.events(wl)
    kw = dict(t0=wl.t0, hang_windows=2, k=wl.k)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    ref = orc.reduce(s, e, wl.t_end(), want_all_stats=True)
    ends = wl.t_end()
    for w in range(wl.n_windows):
        lo = wl.t0 if w == 0 else ends[w - 1]
        ss = s[(s["ts"] >= lo) & (s["ts"] < ends[w])]
        ee = e[(e["ts"] >= lo) & (e["ts"] < ends[w])]
        mon.ingest(_dev(ss) if len(ss) else None, _dev(ee) if len(ee) else None)
        got = mon.window_reduce(ends[w:w + 1])
        st = mon.buffer_stats()
        for f in ("integral", "last", "max", "min", "n_samples"):
            assert np.array_equal(st[f], ref["all_stats"][w][f]), (w, f)
        for f in ("n_samples", "digest", "n_touched", "n_hung"):
            assert got["summary"][f][0] == ref["summary"][f][w], (w, f)
        assert np.array_equal(got["topk"][0], ref["topk"][w])


def test_edge_cases_empty_zero_length_and_k_above_n():
    owner = np.array([0, 0, 1], np.uint32)
    cap = np.array([4, 8, 16], np.uint16)
    tot = np.array([10, 3], np.int64)
    kw = dict(t0=0, hang_windows=1, k=8)
    orc, mon = _pair(owner, cap, tot, 2, **kw)
    # no records at all, zero-length windows included
    ends = [0, 5, 5, 9]
    ref = orc.reduce(sample_array([]), event_array([]), ends)
    mon.ingest(None, None)
    got = mon.window_reduce(ends)
    assert_same(got, ref, mon)
    # only dropped records (late, early, invalid)
    s = sample_array([(3, 0, 1, 4), (10, 9, 1, 4), (12, 1, 9, 8), (20, 2, 1, 16)])
    ref = orc.reduce(s, event_array([]), [15, 18])
    mon.ingest(s, None)  # host ingest path
    got = mon.window_reduce([15, 18])
    assert_same(got, ref, mon)


def test_multiple_ingest_chunks_host_and_device():
    wl = gen.C1.scaled("C1-chunks", n_samples=100_000, n_events=10_000, n_windows=5)
    owner, cap, tot = gen.registry(wl)
    s, e = gen.samples(wl), gen.events(wl)
    orc, mon = _pair(owner, cap, tot, wl.n_components, t0=wl.t0, hang_windows=2, k=wl.k)
    ref = orc.reduce(s, e, wl.t_end())
    mon.ingest(_dev(s[:30000]), _dev(e[:1000]))
    mon.ingest(s[30000:70000], e[1000:5000])
    mon.ingest(_dev(s[70000:]), _dev(e[5000:]))
    got = mon.window_reduce(wl.t_end())
    assert_same(got, ref, mon)


def test_order_violation_is_sticky_until_reset():
    owner = np.zeros(2, np.uint32)
    cap = np.array([4, 4], np.uint16)
    mon = Monitor(owner, cap, np.ones(1, np.int64), n_components=1, t0=0, hang_windows=1, k=2)
    mon.ingest(_dev(sample_array([(5, 0, 1, 4), (3, 1, 2, 4)])), None)
    with pytest.raises(RTMError) as ei:
        mon.window_reduce([10])
    assert ei.value.code == N.RTM_E_ORDER
    with pytest.raises(RTMError):
        mon.window_reduce([20])
    mon.reset()
    mon.ingest(_dev(sample_array([(3, 1, 2, 4), (5, 0, 1, 4)])), None)
    got = mon.window_reduce([10])
    assert int(got["summary"]["n_samples"][0]) == 2


def test_invalid_arguments():
    mon = Monitor(np.zeros(1, np.uint32), np.array([4], np.uint16), np.ones(1, np.int64), n_components=1, t0=10,
                  hang_windows=1, k=1)
    for ends in ([5], [20, 15], [10 + (1 << 40)]):
        with pytest.raises(RTMError) as ei:
            mon.window_reduce(ends)
        assert ei.value.code == N.RTM_E_INVALID
    got = mon.window_reduce([20])  # state unchanged by the rejected calls
    assert int(got["summary"]["t_begin"][0]) == 10


def test_case_study_deadlock_on_gpu():
    from tests.test_oracle import _deadlock_trace

    caps, S, E = _deadlock_trace()
    owner = np.arange(5, dtype=np.uint32)
    orc, mon = _pair(owner, np.array(caps, np.uint16), np.array([100], np.int64), 5, t0=0, hang_windows=2, k=5)
    ends = [100 * (w + 1) for w in range(6)]
    ref = orc.reduce(sample_array(S), event_array(E), ends)
    mon.ingest(_dev(sample_array(S)), _dev(event_array(E)))
    got = mon.window_reduce(ends)
    assert_same(got, ref, mon)
    assert [list(mon.hang_check(w)) for w in range(6)] == [[], [], [], [], [1, 2], [0, 1, 2, 3]]


def _merge_shards(mons, packs, n_windows):
    """The exchange of the two-phase API for shard contexts on one GPU: every shard merges the
    concatenated per-call packs (rtm_merge), then the on-demand tables (rtm_tables_local /
    rtm_tables_merge).  Returns each shard's merged results."""
    import ctypes

    from paper_conf_micro_mosallaeii024_b200 import _copy_from_ptr

    G = len(mons)
    gathered = torch.cat(packs)
    outs = []
    for m in mons:
        summ = np.zeros(n_windows, N.SUMMARY_DTYPE)
        N.check(N.lib().rtm_merge(m._h, gathered.data_ptr(), G, summ.ctypes.data), "merge")
        m.W = n_windows
        outs.append((m.results(), summ))
    tabs = []
    for m in mons:
        pack, nbytes = ctypes.c_void_p(), ctypes.c_uint64()
        N.check(N.lib().rtm_tables_local(m._h, ctypes.byref(pack), ctypes.byref(nbytes)), "tables_local")
        t = torch.empty(int(nbytes.value), dtype=torch.uint8, device="cuda")
        _copy_from_ptr(t, pack.value, int(nbytes.value))
        tabs.append(t)
    torch.cuda.synchronize()
    tg = torch.cat(tabs)
    for m in mons:
        N.check(N.lib().rtm_tables_merge(m._h, tg.data_ptr(), G), "tables_merge")
        m._synced = True
    return outs


SHARD_RANKINGS = [(0, None), (1, None), (2, None), (2, 512)]  # (rank_mode, k); k=512 > owned per rank


@pytest.mark.parametrize("mode,k", SHARD_RANKINGS)
def test_virtual_shards_merge_equals_whole(mode, k):
    """Three shard contexts on one GPU (owner-component sharding) + the library's merge kernels, in
    every rank mode (MEAN: the packs carry the 64-bit order keys, include/rtm.h RTM_RANK_MEAN)."""
    import ctypes

    from paper_conf_micro_mosallaeii024_b200 import _copy_from_ptr

    wl = gen.C1.scaled("C1-vshard", n_samples=200_000, n_events=20_000, n_windows=6)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=2, k=k or wl.k, rank_mode=mode)
    orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, **kw)
    ref = orc.reduce(gen.samples(wl), gen.events(wl), wl.t_end())
    G = 3
    mons, packs = [], []
    for r in range(G):
        owned = (np.arange(wl.n_components) % G == r).astype(np.uint8)
        m = Monitor(owner, cap, tot, n_components=wl.n_components, rank=r, world=G, owned_components=owned, **kw)
        m.ingest(_dev(gen.samples(wl, shard=(G, r))), _dev(gen.events(wl, shard=(G, r))))
        ends = np.ascontiguousarray(wl.t_end())
        pack, nbytes = ctypes.c_void_p(), ctypes.c_uint64()
        N.check(N.lib().rtm_window_reduce_local(m._h, ends.ctypes.data, len(ends), ctypes.byref(pack),
                                                ctypes.byref(nbytes)), "local")
        t = torch.empty(int(nbytes.value), dtype=torch.uint8, device="cuda")
        _copy_from_ptr(t, pack.value, int(nbytes.value))
        torch.cuda.synchronize()
        mons.append(m)
        packs.append(t)
    for m, (got, summ) in zip(mons, _merge_shards(mons, packs, wl.n_windows)):
        assert np.array_equal(got["summary"], summ)
        assert_same(got, ref, m)
        assert np.array_equal(m.topk_persistence(), orc.persistence())  # counted from the merged lists


@pytest.mark.slow
@pytest.mark.parametrize("rank_mode", [0, 1, 2])
def test_c2_full_size_parity(rank_mode):
    """BASELINE configs[1] at full size, in the launch configuration bench.py times, in every
    rank mode (PERCENT is the bench's; SIZE and MEAN rank the same 20480 buffers by level and by
    64-bit mean-occupancy keys); the persistence counter too."""
    wl = gen.C2
    owner, cap, tot = gen.registry(wl)
    ds = torch.empty(wl.n_samples * 16, dtype=torch.uint8, device="cuda")
    de = torch.empty(wl.n_events * 16, dtype=torch.uint8, device="cuda")
    gen.fill_device("samples", wl, ds.data_ptr(), 0, wl.n_samples)
    gen.fill_device("events", wl, de.data_ptr(), 0, wl.n_events)
    torch.cuda.synchronize()
    kw = dict(t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k, rank_mode=rank_mode)
    mon = Monitor(owner, cap, tot, n_components=wl.n_components, **kw)
    mon.ingest(ds, de)
    got = mon.window_reduce(wl.t_end())
    # device generator == host generator (spot check), then the oracle on the host copy
    s = gen.samples(wl)
    e = gen.events(wl)
    idx = np.random.default_rng(0).integers(0, wl.n_samples, 4096)
    assert np.array_equal(ds.view(-1, 16)[torch.from_numpy(idx).cuda()].cpu().numpy().view(gen.SAMPLE_DTYPE).ravel(),
                          s[idx])
    orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, **kw)
    ref = orc.reduce(s, e, wl.t_end())
    assert_same(got, ref, mon)
    assert np.array_equal(mon.topk_persistence(), orc.persistence())


@pytest.mark.parametrize("n_top", [0, 10, 63, 64, 65, 200])
@pytest.mark.parametrize("at_cap", [True, False])
def test_topk_paths_top_tie_and_radix(n_top, at_cap):
    """k=64 over 3000 buffers where exactly n_top buffers share the largest fullness (100 % full, or
    7/8 with everything else lower): n_top >= k takes the top-tie shortcut, fewer takes the radix
    select; both must match the oracle's sort (ties by buffer id)."""
    rng = np.random.default_rng(77 + n_top + 1000 * at_cap)
    nb = 3000
    caps = rng.choice(np.array([4, 8, 16, 128, 1024], np.uint16), nb)
    top = rng.choice(nb, n_top, replace=False)
    caps[top] = 8
    lv = np.minimum(rng.integers(0, 1024, nb), caps // 2).astype(np.uint16)  # <= 50 % full
    lv[top] = 8 if at_cap else 7
    s = sample_array([(i, b, int(lv[b]), int(caps[b])) for i, b in enumerate(rng.permutation(nb))])
    owner = (np.arange(nb) // 4).astype(np.uint32)
    kw = dict(t0=0, hang_windows=4, k=64, rank_mode=0)
    orc, mon = _pair(owner, caps, np.ones(2, np.int64), int(owner[-1]) + 1, **kw)
    ref = orc.reduce(s, event_array([]), [nb + 10])
    mon.ingest(_dev(s), None)
    got = mon.window_reduce([nb + 10])
    assert int(got["topk_n"][0]) == int(ref["topk_n"][0]) == 64
    assert np.array_equal(got["topk"][0], ref["topk"][0])


@pytest.mark.parametrize("placement", ["slice0", "later_slices", "split_k_minus_1", "kth_at_slice_end",
                                       "none", "scattered"])
@pytest.mark.parametrize("n_windows", [1, 200])
def test_topk_full_prefix_shortcut(placement, n_windows):
    """Percent-mode top-k scans ids in order for 100 %-full buffers and stops at k (DESIGN.md §4
    K5); with few windows the buffers are split into id slices and the merge takes slice 0's list
    when all its k candidates are full.  Full buffers are placed so that the scan succeeds in
    slice 0, only in later slices, misses by one, ends exactly at a slice boundary, never
    succeeds, or is scattered; every window must equal the oracle's full sort."""
    rng = np.random.default_rng(hash(placement) % 1000 + n_windows)
    nb, k = 20480, 64
    caps = rng.choice(np.array([4, 8, 16, 128, 1024], np.uint16), nb)
    if placement == "slice0":
        full = rng.choice(1024, 100, replace=False)
    elif placement == "later_slices":
        full = 8192 + rng.choice(8192, 100, replace=False)
    elif placement == "split_k_minus_1":
        full = np.concatenate([rng.choice(1024, k - 1, replace=False), [nb - 1]])
    elif placement == "kth_at_slice_end":
        full = np.concatenate([rng.choice(2047, k - 1, replace=False), [2047]])
    elif placement == "none":
        full = np.array([], np.int64)
    else:
        full = rng.choice(nb, 300, replace=False)
    lv = np.minimum(rng.integers(0, 1024, nb), caps - 1).astype(np.uint16)
    lv[full] = caps[full]
    rows = []
    for w in range(n_windows):  # every window re-samples a random subset; fulls stay full
        ids = rng.choice(nb, nb // 4 if w else nb, replace=False)
        lvw = lv.copy()
        if w:
            lvw[ids] = np.where(np.isin(ids, full), caps[ids], np.minimum(rng.integers(0, 1024, len(ids)), caps[ids] - 1))
            lv = lvw
        rows += [(w * 100000 + i, int(b), int(lvw[b]), int(caps[b])) for i, b in enumerate(ids)]
    s = sample_array(rows)
    owner = (np.arange(nb) // 4).astype(np.uint32)
    kw = dict(t0=0, hang_windows=4, k=k, rank_mode=0)
    orc, mon = _pair(owner, caps, np.ones(2, np.int64), int(owner[-1]) + 1, **kw)
    t_end = [(w + 1) * 100000 for w in range(n_windows)]
    ref = orc.reduce(s, event_array([]), t_end)
    mon.ingest(_dev(s), None)
    got = mon.window_reduce(t_end)
    assert np.array_equal(got["topk_n"], ref["topk_n"])
    for w in range(n_windows):
        assert np.array_equal(got["topk"][w], ref["topk"][w]), w


@pytest.mark.parametrize("H", [65, 100, 160])
def test_long_hang_window_across_calls(H):
    """H above the per-(window, word) AND loop's range takes the two-pass sliding-window AND
    (DESIGN.md §4 K6); quiet components (few events) and held-full buffers make long runs that
    cross call boundaries, so windows w < H-1 of every call depend on the carried run.  Flags and
    n_hung of every window must equal the oracle's."""
    wl = gen.C1.scaled("C1-longH", n_samples=300_000, n_events=3_000, n_windows=600, hang_windows=H)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=H, k=wl.k)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    s, e = gen.samples(wl), gen.events(wl)
    t_end = wl.t_end()
    w0, total_hung = 0, 0
    for m in (50, 1, 120, 7, 300, 122):
        w1 = w0 + m
        sl = slice(wl.index_at("samples", wl.t_begin(w0)), wl.index_at("samples", wl.t_begin(w1)))
        el = slice(wl.index_at("events", wl.t_begin(w0)), wl.index_at("events", wl.t_begin(w1)))
        ref = orc.reduce(s[sl], e[el], t_end[w0:w1])
        mon.ingest(_dev(s[sl]), _dev(e[el]))
        got = mon.window_reduce(t_end[w0:w1])
        assert_same(got, ref, mon, stats=False, comps=False)
        total_hung += int(ref["summary"]["n_hung"].sum())
        w0 = w1
    assert w0 == wl.n_windows and total_hung > 0  # the long-run path was exercised


def test_long_hang_block_edges():
    """Long H with calls of H - 1, H, H + 1 and 2H windows: the prefix path (W < H) and the
    block-parallel van Herk path at its edges (one full block, a one-window second block, two full
    blocks), runs carried across all of them."""
    H = 100
    wl = gen.C1.scaled("C1-longH-edges", n_samples=400_000, n_events=2_000, n_windows=500, hang_windows=H)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=H, k=wl.k)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    s, e = gen.samples(wl), gen.events(wl)
    t_end = wl.t_end()
    w0, total_hung = 0, 0
    for m in (H - 1, H, H + 1, 2 * H):
        w1 = w0 + m
        sl = slice(wl.index_at("samples", wl.t_begin(w0)), wl.index_at("samples", wl.t_begin(w1)))
        el = slice(wl.index_at("events", wl.t_begin(w0)), wl.index_at("events", wl.t_begin(w1)))
        ref = orc.reduce(s[sl], e[el], t_end[w0:w1])
        mon.ingest(_dev(s[sl]), _dev(e[el]))
        assert_same(mon.window_reduce(t_end[w0:w1]), ref, mon, stats=False, comps=False)
        total_hung += int(ref["summary"]["n_hung"].sum())
        w0 = w1
    assert total_hung > 0


@pytest.mark.parametrize("disorder", [False, True])
@pytest.mark.parametrize("stream", ["samples", "events"])
def test_order_check_across_tiles_with_invalid_gap(disorder, stream):
    """The cross-tile order check compares each tile with the nearest EARLIER tile that has a
    field-valid record: here three 4096-record tiles, the middle one entirely field-invalid, and
    (disorder) the third starting below the first tile's last ts.  Oracle and GPU must agree."""
    nb, n = 8, 4096
    owner = np.zeros(nb, np.uint32)
    cap = np.full(nb, 4, np.uint16)
    ts = np.concatenate([np.arange(n), np.full(n, 5000), np.arange(n) + (n - 10 if disorder else n)])
    if stream == "samples":
        rows = [(int(t), i % nb, 1, 4) for i, t in enumerate(ts)]
        for i in range(n, 2 * n):
            rows[i] = (int(ts[i]), nb + 3, 1, 4)  # buffer id out of range: field-invalid
        s, e = sample_array(rows), event_array([])
    else:
        rows = [(int(t), i, 0 | (0 << 20) | ((i & 1) << 31)) for i, t in enumerate(ts)]
        for i in range(n, 2 * n):
            rows[i] = (int(ts[i]), i, 7)  # component 7 >= n_components: field-invalid
        s, e = sample_array([]), event_array(rows)
    kw = dict(t0=0, hang_windows=2, k=4)
    orc, mon = _pair(owner, cap, np.full(1, 10 ** 6, np.int64), 1, **kw)
    ends = [3 * n + 100]
    ref = orc.reduce(s, e, ends)
    mon.ingest(_dev(s) if len(s) else None, _dev(e) if len(e) else None)
    if disorder:
        assert ref["rc"] == -4
        with pytest.raises(RTMError) as ei:
            mon.window_reduce(ends)
        assert ei.value.code == N.RTM_E_ORDER
    else:
        assert ref["rc"] == 0
        assert_same(mon.window_reduce(ends), ref, mon)


@pytest.mark.parametrize("mode,k", SHARD_RANKINGS)
def test_rank_local_numbering_shards_merge_equals_whole(mode, k):
    """Owner sharding with RANK-LOCAL buffer numbering (include/rtm.h buffer_global_id): each
    shard registers only its own buffers (dense local ids, records remapped to them), results
    carry global ids; the merged top-k, digests, progress, hang flags and the per-buffer table
    (by global id) must equal the whole-trace oracle."""
    import ctypes

    from paper_conf_micro_mosallaeii024_b200 import _copy_from_ptr

    wl = gen.C1.scaled("C1-lshard", n_samples=200_000, n_events=20_000, n_windows=6)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=2, k=k or wl.k, rank_mode=mode)
    orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, **kw)
    ref = orc.reduce(gen.samples(wl), gen.events(wl), wl.t_end())
    G = 3
    gids = [np.nonzero(owner % G == r)[0].astype(np.uint32) for r in range(G)]
    pack_nb = max(len(g) for g in gids)
    mons, packs = [], []
    ends = np.ascontiguousarray(wl.t_end())
    for r in range(G):
        gid = gids[r]
        m = Monitor(owner[gid], cap[gid], tot, n_components=wl.n_components, rank=r, world=G,
                    buffer_global_id=gid, n_global_buffers=len(owner), pack_buffers=pack_nb, **kw)
        s = gen.samples(wl, shard=(G, r)).copy()
        loc = np.searchsorted(gid, s["buffer_id"])
        ok = (loc < len(gid)) & (gid[np.minimum(loc, len(gid) - 1)] == s["buffer_id"])
        s["buffer_id"] = np.where(ok, loc, 0xFFFFFFF0).astype(np.uint32)
        m.ingest(_dev(s), _dev(gen.events(wl, shard=(G, r))))
        pack, nbytes = ctypes.c_void_p(), ctypes.c_uint64()
        N.check(N.lib().rtm_window_reduce_local(m._h, ends.ctypes.data, len(ends), ctypes.byref(pack),
                                                ctypes.byref(nbytes)), "local")
        t = torch.empty(int(nbytes.value), dtype=torch.uint8, device="cuda")
        _copy_from_ptr(t, pack.value, int(nbytes.value))
        torch.cuda.synchronize()
        mons.append(m)
        packs.append(t)
    assert len({int(t.numel()) for t in packs}) == 1  # equal-size packs (pack_buffers)
    for m, (got, summ) in zip(mons, _merge_shards(mons, packs, wl.n_windows)):
        assert np.array_equal(got["summary"], summ)
        assert_same(got, ref, m)
        assert np.array_equal(m.topk_persistence(), orc.persistence())  # counted from the merged lists


def test_rank_local_numbering_rejects_unsorted_ids():
    owner = np.zeros(3, np.uint32)
    cap = np.full(3, 4, np.uint16)
    with pytest.raises(RTMError):
        Monitor(owner, cap, np.ones(1, np.int64), n_components=1, buffer_global_id=np.array([5, 3, 9], np.uint32),
                n_global_buffers=10)
    with pytest.raises(RTMError):
        Monitor(owner, cap, np.ones(1, np.int64), n_components=1, buffer_global_id=np.array([1, 3, 10], np.uint32),
                n_global_buffers=10)


@pytest.mark.parametrize("n_buffers", [32768, 33000, 43521, 81920, 261888, 262144])
def test_many_bins_partition_paths(n_buffers):
    """Every partition path against the oracle (short trace): <= 170 bins the lane-major partition
    in one ranking pass (128, 129 bins), 171 .. 1023 bins in passes of <= 170 bins (171: a
    one-bin second pass; 320 as C3; 1023: one CTA per SM), 1024 bins the two-pass path."""
    wl = gen.C1.scaled("C1-bins", n_samples=400_000, n_events=40_000, n_buffers=n_buffers, n_windows=5)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=2, k=wl.k)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    s, e = gen.samples(wl), gen.events(wl)
    ref = orc.reduce(s, e, wl.t_end())
    mon.ingest(_dev(s), _dev(e))
    got = mon.window_reduce(wl.t_end())
    assert_same(got, ref, mon)


@pytest.mark.parametrize("n_buffers", [1000, 327680])
def test_graph_replay_equals_direct_launches(n_buffers):
    """rtm_use_graphs: a context replaying captured CUDA graphs (RTM_GRAPHS_ALWAYS) and one
    launching directly (RTM_GRAPHS_OFF) stream the same trace in calls of 1, 1, 3, 1, 2, 1, 1
    windows (shapes repeat, so most calls are replays with new arguments) with watched buffers;
    both equal the oracle call by call, including the value-monitor rings.  327680 buffers take the
    two-pass partition; 1000 the lane-major one."""
    wl = gen.C1.scaled("C1-graph", n_samples=300_000, n_events=30_000, n_buffers=n_buffers, n_windows=10)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=2, k=wl.k)
    orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, **kw)
    mons = [Monitor(owner, cap, tot, n_components=wl.n_components, **kw) for _ in range(2)]
    mons[0].use_graphs(N.RTM_GRAPHS_OFF)
    mons[1].use_graphs(N.RTM_GRAPHS_ALWAYS)
    watched = [0, 7, n_buffers - 1]
    for m in mons:
        m.watch(watched)
    s, e = gen.samples(wl), gen.events(wl)
    t_end = wl.t_end()
    w0 = 0
    launches = []
    for m_w in (1, 1, 3, 1, 2, 1, 1):
        w1 = w0 + m_w
        sl = slice(wl.index_at("samples", wl.t_begin(w0)), wl.index_at("samples", wl.t_begin(w1)))
        el = slice(wl.index_at("events", wl.t_begin(w0)), wl.index_at("events", wl.t_begin(w1)))
        ref = orc.reduce(s[sl], e[el], t_end[w0:w1], want_all_stats=True)
        for i, m in enumerate(mons):
            k0 = N.lib().rtm_kernel_launches()
            m.ingest(_dev(s[sl]), _dev(e[el]))
            got = m.window_reduce(t_end[w0:w1])
            launches.append((i, int(N.lib().rtm_kernel_launches() - k0)))
            assert_same(got, ref, m)
        w0 = w1
    for q in range(len(watched)):
        a, b = mons[0].watch_series(q), mons[1].watch_series(q)
        assert np.array_equal(a.view(np.uint8), b.view(np.uint8))
    captured, replayed = mons[1].graph_stats()
    assert captured >= 1 and replayed >= 1 and captured + replayed == 7, (captured, replayed)
    assert mons[0].graph_stats() == (0, 0)
    # a replay launches (and counts) the same kernels as a direct call of the same shape
    direct = [n for i, n in launches if i == 0]
    graph = [n for i, n in launches if i == 1]
    assert direct == graph


@pytest.mark.parametrize("case", ["ragged_invalid", "mean_1m", "very_sparse_bl7", "wide_windows"])
def test_two_pass_partition_paths(case):
    """Registries of >= 1024 bins take the two-pass partition (lane-major by 16384-buffer superbin,
    then k_subpart sorts every (window, superbin) by bin into (window, bin)-contiguous staging)
    when every window is shorter than 2^32 ticks; wider windows keep the match-based partition.
    Cases: a ragged last superbin (262444 buffers) with 1 % invalid records and empty windows;
    2^20 buffers in rank mode MEAN (windowed fold + 64-bit keys); 327680 buffers (bins of 128)
    in a very sparse call (sequential fold); a window of 2^33 ticks (fallback partition)."""
    n_buffers = {"ragged_invalid": 262444, "mean_1m": 1 << 20, "very_sparse_bl7": 327680,
                 "wide_windows": 262144}[case]
    n_samples = 60_000 if case == "very_sparse_bl7" else 500_000
    wl = gen.C1.scaled("C1-2p", n_samples=n_samples, n_events=n_samples // 10, n_buffers=n_buffers, n_windows=6,
                       invalid_ppm=10_000 if case == "ragged_invalid" else 0)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=2, k=wl.k)
    if case == "mean_1m":
        kw["rank_mode"] = 2  # RTM_RANK_MEAN
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    s, e = gen.samples(wl), gen.events(wl)
    t_end = wl.t_end()
    if case == "ragged_invalid":  # empty windows: repeated ends
        t_end = np.array([t_end[0], t_end[0], t_end[1], t_end[2], t_end[2], t_end[3], t_end[4], t_end[5]], np.int64)
    elif case == "very_sparse_bl7":  # 60k samples over 327680 buffers x 40 windows: sequential fold
        t_end = np.linspace(wl.t0 + 1, int(t_end[-1]), 40).astype(np.int64)
        assert len(s) * 8 < n_buffers * len(t_end)
    elif case == "wide_windows":
        t_end = np.array([int(t_end[2]), int(t_end[2]) + (1 << 33)], np.int64)
    ref = orc.reduce(s, e, t_end, want_all_stats=True)
    mon.ingest(_dev(s), _dev(e))
    got = mon.window_reduce(t_end)
    assert_same(got, ref, mon)
    if case == "ragged_invalid":
        assert int(np.sum(ref["summary"]["n_dropped"])) > 0


@pytest.mark.parametrize("n_buffers,k,calls", [(20480, 64, (1, 1, 3, 37, 1)), (65536, 1024, (1, 2)),
                                                (16384, 16, (5, 1)), (20482, 64, (1, 2))])
def test_topk_slices_few_window_calls(n_buffers, k, calls):
    """Calls with fewer windows than SMs split each window's buffers into id slices (one top-k
    CTA per slice, then a merge of the slices' candidates); every call must still equal the
    oracle's full sort (n_buffers not a multiple of 8 takes the one-CTA path)."""
    n_win = sum(calls)
    wl = gen.C1.scaled("C1-slices", n_samples=600_000, n_events=60_000, n_buffers=n_buffers, n_windows=n_win, k=k)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=2, k=k)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    s, e = gen.samples(wl), gen.events(wl)
    t_end = wl.t_end()
    w0 = 0
    for m in calls:
        w1 = w0 + m
        sl = slice(wl.index_at("samples", wl.t_begin(w0)), wl.index_at("samples", wl.t_begin(w1)))
        el = slice(wl.index_at("events", wl.t_begin(w0)), wl.index_at("events", wl.t_begin(w1)))
        ref = orc.reduce(s[sl], e[el], t_end[w0:w1])
        mon.ingest(_dev(s[sl]), _dev(e[el]))
        got = mon.window_reduce(t_end[w0:w1])
        assert_same(got, ref, mon)
        w0 = w1


def test_value_monitor_rings_last_300_windows():
    """Value monitor (up to 5 values, the last 300 points): 5 watched buffers
    over 400 windows in 40 calls; each ring holds the last 300 windows' statistics of its
    buffer, equal to the oracle's per-window table; invalid watch sets are rejected."""
    wl = gen.C1.scaled("C1-watch", n_samples=400_000, n_events=40_000, n_windows=400)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=2, k=wl.k)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    ids = [0, 7, 999, 500, 123]
    with pytest.raises(RTMError):
        mon.watch(list(range(6)))
    with pytest.raises(RTMError):
        mon.watch([3, 3])
    with pytest.raises(RTMError):
        mon.watch([wl.n_buffers])
    mon.watch(ids)
    s, e = gen.samples(wl), gen.events(wl)
    t_end = wl.t_end()
    ref_rows = []
    for w0 in range(0, wl.n_windows, 10):
        w1 = w0 + 10
        sl = slice(wl.index_at("samples", wl.t_begin(w0)), wl.index_at("samples", wl.t_begin(w1)))
        el = slice(wl.index_at("events", wl.t_begin(w0)), wl.index_at("events", wl.t_begin(w1)))
        ref = orc.reduce(s[sl], e[el], t_end[w0:w1], want_all_stats=True)
        ref_rows.append(ref["all_stats"])
        mon.ingest(_dev(s[sl]), _dev(e[el]))
        mon.window_reduce(t_end[w0:w1])
        if w0 == 0:
            assert len(mon.watch_series(0)) == 10
    A = np.concatenate(ref_rows)  # [400, n_buffers]
    for q, b in enumerate(ids):
        ser = mon.watch_series(q)
        assert len(ser) == 300
        assert np.array_equal(ser["t_end"], t_end[100:])
        for f in ("integral", "last", "max", "min", "capacity", "n_samples", "mean_occ"):
            assert np.array_equal(ser[f], A[100:, b][f]), (b, f)
    mon.reset()
    assert len(mon.watch_series(0)) == 0
    mon.watch([])
    with pytest.raises(RTMError):
        mon.watch_series(0)


@pytest.mark.parametrize("seed", range(30))
def test_mean_ranking_random_tiny_traces(seed):
    """Rank mode MEAN (persistence ranking): random tiny traces, GPU vs oracle, plus the
    windows-in-top-k counter after every call."""
    rng = np.random.default_rng(7000 + seed)
    case = random_tiny_case(rng)
    kw = dict(t0=case["t0"], hang_windows=case["H"], k=case["k"], rank_mode=2)
    orc, mon = _pair(case["owner"], case["caps"], case["totals"], case["nc"], **kw)
    for srows, erows, ends in case["calls"]:
        ref = orc.reduce(sample_array(srows), event_array(erows), ends)
        mon.ingest(sample_array(srows), event_array(erows))
        got = mon.window_reduce(np.array(ends, np.int64))
        assert_same(got, ref, mon, comps=False)
        assert np.array_equal(mon.topk_persistence(), orc.persistence())


@pytest.mark.parametrize("mode", [0, 1, 2])
def test_ranking_modes_c1_and_persistence(mode):
    """C1 (1M samples, 1000 buffers, 10 windows) in every rank mode: top-k lists and the
    persistence counter equal the oracle's."""
    wl = gen.C1
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k, rank_mode=mode)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    s, e = gen.samples(wl), gen.events(wl)
    for lo, hi in ((0, 4), (4, 5), (5, 10)):
        sl = slice(wl.index_at("samples", wl.t_begin(lo)), wl.index_at("samples", wl.t_begin(hi)))
        el = slice(wl.index_at("events", wl.t_begin(lo)), wl.index_at("events", wl.t_begin(hi)))
        ref = orc.reduce(s[sl], e[el], wl.t_end()[lo:hi])
        mon.ingest(_dev(s[sl]), _dev(e[el]))
        got = mon.window_reduce(wl.t_end()[lo:hi])
        assert_same(got, ref, mon)
    assert np.array_equal(mon.topk_persistence(), orc.persistence())


def test_mean_mode_rejects_long_windows():
    owner, cap = np.zeros(2, np.uint32), np.array([4, 8], np.uint16)
    mon = Monitor(owner, cap, np.ones(1, np.int64), n_components=1, t0=0, k=2, rank_mode=2)
    with pytest.raises(RTMError):
        mon.window_reduce(np.array([1 << 33], np.int64))
    got = mon.window_reduce(np.array([10], np.int64))  # state unchanged: the next call works
    assert int(got["summary"]["t_begin"][0]) == 0


@pytest.mark.parametrize("seed", range(25))
def test_dynamic_progress_bars_random(seed):
    """Bars created / updated / destroyed between calls: GPU vs oracle on random
    tiny traces, including the dropped events of destroyed ids and zero entries."""
    from tests.test_oracle import _apply, _bar_ops
    rng = np.random.default_rng(9000 + seed)
    case = random_tiny_case(rng)
    kw = dict(t0=case["t0"], hang_windows=case["H"], k=case["k"], rank_mode=case["mode"])
    orc, mon = _pair(case["owner"], case["caps"], case["totals"], case["nc"], **kw)
    for srows, erows, ends in case["calls"]:
        for op, arg in _bar_ops(rng, case["nk"]):
            assert _apply(orc, op, arg) == _apply(mon, op, arg)
        ref = orc.reduce(sample_array(srows), event_array(erows), ends)
        mon.ingest(sample_array(srows), event_array(erows))
        got = mon.window_reduce(np.array(ends, np.int64))
        assert_same(got, ref, mon)


def test_dynamic_progress_bars_c1_kernels_retired():
    """C1 with its 4 kernel bars: after window 4 bar 0 is destroyed (its remaining thread blocks
    become invalid records) and re-created for a new kernel with another total; the GPU matches
    the oracle on every window, and rtm_reset restores the registry."""
    wl = gen.C1
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    s, e = gen.samples(wl), gen.events(wl)
    for lo, hi in ((0, 4), (4, 7), (7, 10)):
        if lo == 4:
            for x in (orc, mon):
                x.bar_destroy(0)
                x.bar_update(3, 12345)
        if lo == 7:
            assert orc.bar_create(777) == mon.bar_create(777) == 0
        sl = slice(wl.index_at("samples", wl.t_begin(lo)), wl.index_at("samples", wl.t_begin(hi)))
        el = slice(wl.index_at("events", wl.t_begin(lo)), wl.index_at("events", wl.t_begin(hi)))
        ref = orc.reduce(s[sl], e[el], wl.t_end()[lo:hi])
        mon.ingest(_dev(s[sl]), _dev(e[el]))
        got = mon.window_reduce(wl.t_end()[lo:hi])
        assert_same(got, ref, mon)
    with pytest.raises(RTMError):
        mon.bar_create(1)  # every id live again
    mon.reset()
    orc.reset()
    ref = orc.reduce(s[:1000], e[:100], wl.t_end()[:1])
    mon.ingest(_dev(s[:1000]), _dev(e[:100]))
    assert_same(mon.window_reduce(wl.t_end()[:1]), ref, mon)


@pytest.mark.parametrize("hang_mode", [0, 1])
def test_case_study_deadlock_roots(hang_mode):
    """Case study 2 with the component connection graph (L1 -> L2 write buffer <-> local storage
    <- DRAM controller, CU -> L1): the GPU's flags equal the oracle's in both hang modes, and the
    root causes are the circular wait {1, 2} — the backed-up L1 and DRAM controller are not."""
    from oracle import brute
    from tests.test_oracle import _deadlock_trace

    caps, S, E = _deadlock_trace()
    owner = np.arange(5, dtype=np.uint32)
    kw = dict(t0=0, hang_windows=2, k=5, hang_mode=hang_mode)
    orc, mon = _pair(owner, np.array(caps, np.uint16), np.array([100], np.int64), 5, **kw)
    src, dst = [0, 2, 1, 3, 4], [2, 1, 2, 1, 0]
    mon.set_links(src, dst)
    ends = [100 * (w + 1) for w in range(6)]
    ref = orc.reduce(sample_array(S), event_array(E), ends)
    mon.ingest(_dev(sample_array(S)), _dev(event_array(E)))
    got = mon.window_reduce(ends)
    assert_same(got, ref, mon)
    for w in range(6):
        flagged = np.nonzero(ref["hung"][w])[0]
        assert mon.hang_roots(w).tolist() == brute.hang_roots(flagged, src, dst), w
    assert mon.hang_roots(5).tolist() == [1, 2]


@pytest.mark.parametrize("seed", range(20))
def test_nonempty_hang_mode_and_roots_random(seed):
    """RTM_HANG_NONEMPTY on random tiny traces with random connection graphs: flags equal the
    oracle's, root causes equal the brute-force reachability definition on them."""
    from oracle import brute

    rng = np.random.default_rng(12000 + seed)
    case = random_tiny_case(rng)
    kw = dict(t0=case["t0"], hang_windows=case["H"], k=case["k"], rank_mode=case["mode"], hang_mode=1)
    orc, mon = _pair(case["owner"], case["caps"], case["totals"], case["nc"], **kw)
    nl = int(rng.integers(0, 3 * case["nc"]))
    src, dst = rng.integers(0, case["nc"], nl), rng.integers(0, case["nc"], nl)
    mon.set_links(src, dst)
    for srows, erows, ends in case["calls"]:
        ref = orc.reduce(sample_array(srows), event_array(erows), ends)
        mon.ingest(sample_array(srows), event_array(erows))
        got = mon.window_reduce(np.array(ends, np.int64))
        assert_same(got, ref, mon)
        for w in range(len(ends)):
            assert mon.hang_roots(w).tolist() == brute.hang_roots(np.nonzero(ref["hung"][w])[0], src, dst)


def test_limits_max_sizes_wide_windows_and_hot_buffer():
    """Registry and record limits in one trace: 2^20 components, 2048 progress bars, k = 1024,
    capacities 1 .. 65534 with levels up to 65534, windows of 2^33 and ~2^39 ticks next to 0- and
    5-tick ones (the 64-bit offset paths), and one buffer with more than 65535 samples in a
    window (the per-window sample counter's wide path); t0 far below zero."""
    rng = np.random.default_rng(31337)
    nb, nc, nk = 3000, 1 << 20, 2048
    owner = ((np.arange(nb, dtype=np.int64) * 349) % nc).astype(np.uint32)
    cap = rng.choice([1, 2, 8, 1024, 65534], size=nb).astype(np.uint16)
    t0 = -(1 << 41)
    lens = [1 << 33, 5, 0, (1 << 39) + 12345, 1000]
    ends = list(np.cumsum([t0] + lens)[1:].astype(np.int64))
    n = 300_000
    ts = np.sort(rng.integers(t0, ends[-1], n))
    b = rng.integers(0, nb, n).astype(np.uint32)
    hot = (ts >= ends[2]) & (ts < ends[3]) & (rng.random(n) < 0.6)  # > 65535 samples in window 3
    b[hot] = 7
    lvl = (rng.random(n) * (cap[b].astype(np.float64) + 1)).astype(np.int64)
    lvl = np.minimum(lvl, cap[b]).astype(np.uint16)
    s = np.zeros(n, gen.SAMPLE_DTYPE)
    s["ts"], s["buffer_id"], s["level"], s["capacity"] = ts, b, lvl, cap[b]
    ne = 50_000
    ets = np.sort(rng.integers(t0, ends[-1], ne))
    comp = rng.integers(0, nc, ne).astype(np.uint32)
    kern = rng.integers(0, nk, ne).astype(np.uint32)
    kind = rng.integers(0, 2, ne).astype(np.uint32)
    e = np.zeros(ne, gen.EVENT_DTYPE)
    e["ts"], e["task_id"], e["meta"] = ets, np.arange(ne), comp | (kern << 20) | (kind << 31)
    tot = rng.integers(0, 100, nk).astype(np.int64)
    assert int(hot.sum()) > 65535
    for mode in (0, 2):
        if mode == 2:  # mean-occupancy keys need windows < 2^32 ticks: those calls are rejected
            mon = Monitor(owner, cap, tot, n_components=nc, t0=t0, hang_windows=2, k=1024, rank_mode=2)
            with pytest.raises(RTMError):
                mon.window_reduce(np.array(ends, np.int64))
            continue
        orc, mon = _pair(owner, cap, tot, nc, t0=t0, hang_windows=2, k=1024, rank_mode=mode)
        ref = orc.reduce(s, e, np.array(ends, np.int64))
        assert ref["rc"] == 0
        mon.ingest(_dev(s), _dev(e))
        got = mon.window_reduce(np.array(ends, np.int64))
        assert_same(got, ref, mon)  # window 3's digest covers the hot buffer's > 65535-sample count


@pytest.mark.parametrize("dense", [True, False])
def test_narrow_integral_boundary(dense):
    """The fold keeps its integral term D in 32 bits when every capacity times every window length
    of the call is below 2^32 (D lies in [0, cap * Wlen]).  Capacities up to 65534 at levels near
    capacity, a call whose windows are 65538 ticks (65534 * 65538 = 2^32 - 4: the 32-bit path at
    its edge, one buffer with more than 65535 samples in a window) and a call with 65539-tick
    windows (just past it: the 64-bit path), dense and sparse, then very sparse calls of 40 such
    windows (the sequential fold, both layouts), against the oracle."""
    rng = np.random.default_rng(4242 + dense)
    nb, nc, nk = 2000 if dense else 60_000, 500, 4
    owner = (np.arange(nb) % nc).astype(np.uint32)
    cap = rng.choice([1, 1024, 65534], size=nb).astype(np.uint16)
    tot = np.full(nk, 10, np.int64)
    orc, mon = _pair(owner, cap, tot, nc, t0=0, hang_windows=2, k=16)
    t = 0
    # windowed fold (32-bit D at its edge, then 64-bit), then very sparse calls (sequential fold)
    for lens, n in (([65538, 1000, 0, 65538], 400_000), ([65539, 70000, 3], 400_000), ([65539] * 40, 500),
                    ([65538] * 40, 500)):
        ends = np.cumsum([t] + lens)[1:].astype(np.int64)
        ts = np.sort(rng.integers(t, ends[-1], n))
        b = rng.integers(0, nb, n).astype(np.uint32)
        if n > 1000 and lens[0] == 65538:  # > 65535 samples of buffer 5 in the first window
            hot = (ts < ends[0]) & (rng.random(n) < 0.5)
            b[hot] = 5
            assert int(hot.sum()) > 65535
        hi = rng.random(n) < 0.8
        lvl = np.where(hi, cap[b], (rng.random(n) * cap[b]).astype(np.int64)).astype(np.uint16)
        s_ = np.zeros(n, gen.SAMPLE_DTYPE)
        s_["ts"], s_["buffer_id"], s_["level"], s_["capacity"] = ts, b, lvl, cap[b]
        ref = orc.reduce(s_, event_array([]), ends)
        assert ref["rc"] == 0
        mon.ingest(_dev(s_), None)
        assert_same(mon.window_reduce(ends), ref, mon)
        t = int(ends[-1])


def test_order_error_then_reset_then_multiwindow_lookback():
    """A multi-window call that fails with RTM_E_ORDER has already run its fold (which publishes
    look-back flags); after rtm_reset the next multi-window call must not read those flags as
    published (every call takes a fresh look-back epoch): its results equal the oracle's."""
    wl = gen.C1.scaled("C1-epoch", n_samples=400_000, n_events=40_000, n_windows=8)
    owner, cap, tot = gen.registry(wl)
    s, e = gen.samples(wl), gen.events(wl)
    kw = dict(t0=wl.t0, hang_windows=2, k=wl.k)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    bad = s.copy()
    j = len(bad) - 10  # one inversion near the end: every window's fold still runs
    bad[j], bad[j + 1] = bad[j + 1].copy(), bad[j].copy()
    bad["ts"][j] += 3
    mon.ingest(_dev(bad), _dev(e))
    with pytest.raises(RTMError) as ei:
        mon.window_reduce(wl.t_end())
    assert ei.value.code == N.RTM_E_ORDER
    mon.reset()
    for _ in range(2):  # the same multi-window call twice from a reset state
        ref = orc.reduce(s, e, wl.t_end())
        mon.ingest(_dev(s), _dev(e))
        assert_same(mon.window_reduce(wl.t_end()), ref, mon)
        mon.reset()
        orc.reset()


def test_merge_pending_state_and_world_k_limit():
    """rtm_window_reduce_local leaves the context merge-pending: a second reduce and rtm_watch
    return RTM_E_STATE (no state change) until rtm_merge; rtm_reset clears it.  rtm_create
    rejects world * k above what the merge holds in shared memory."""
    import ctypes

    from paper_conf_micro_mosallaeii024_b200 import _copy_from_ptr

    wl = gen.C1.scaled("C1-pending", n_samples=50_000, n_events=5_000, n_windows=3)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=2, k=wl.k)
    with pytest.raises(RTMError) as ei:
        Monitor(owner, cap, tot, n_components=wl.n_components, rank=0, world=16, k=1024,
                owned_components=np.ones(wl.n_components, np.uint8), t0=wl.t0)
    assert ei.value.code == N.RTM_E_INVALID
    orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, **kw)
    ref = orc.reduce(gen.samples(wl), gen.events(wl), wl.t_end())
    m = Monitor(owner, cap, tot, n_components=wl.n_components, rank=0, world=1, **kw)
    ends = np.ascontiguousarray(wl.t_end())
    for attempt in range(2):
        m.ingest(_dev(gen.samples(wl)), _dev(gen.events(wl)))
        pack, nbytes = ctypes.c_void_p(), ctypes.c_uint64()
        N.check(N.lib().rtm_window_reduce_local(m._h, ends.ctypes.data, len(ends), ctypes.byref(pack),
                                                ctypes.byref(nbytes)), "local")
        rc = N.lib().rtm_window_reduce_local(m._h, ends.ctypes.data, len(ends), ctypes.byref(pack),
                                             ctypes.byref(nbytes))
        assert rc == N.RTM_E_STATE
        with pytest.raises(RTMError) as ei:
            m.watch([1])
        assert ei.value.code == N.RTM_E_STATE
        if attempt == 0:  # abandon the exchange: reset clears the pending merge
            m.reset()
            continue
        t = torch.empty(int(nbytes.value), dtype=torch.uint8, device="cuda")
        _copy_from_ptr(t, pack.value, int(nbytes.value))
        torch.cuda.synchronize()
        summ = np.zeros(wl.n_windows, N.SUMMARY_DTYPE)
        N.check(N.lib().rtm_merge(m._h, t.data_ptr(), 1, summ.ctypes.data), "merge")
        m.W = wl.n_windows
        assert_same(m.results(), ref, m)
    assert N.lib().rtm_merge(m._h, t.data_ptr(), 1, summ.ctypes.data) == N.RTM_E_STATE


@pytest.mark.parametrize("hang_mode", [0, 1])
def test_very_sparse_calls_sequential_fold(hang_mode):
    """Calls with fewer than one kept sample per 8 buffer-windows (C5's shape: ~1 in 45) take the
    sequential fold (one warp per bin walks the call's windows, only touched buffers finalized).
    40 000 buffers, 900 windows in calls of 1, 299 and 600 windows, 0.02-0.05 samples per
    buffer-window, H small enough to flag components, watched buffers: every window's summary,
    top-k, progress, hang list, the last window's table and the value-monitor rings equal the
    oracle's."""
    wl = gen.C5.scaled("C5-seq", n_samples=1_200_000, n_events=120_000, n_buffers=40_000, n_windows=900,
                       hang_windows=6)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=6, k=wl.k, hang_mode=hang_mode)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    watched = [0, 12345, 39999]
    mon.watch(watched)
    s, e = gen.samples(wl), gen.events(wl)
    t_end = wl.t_end()
    rows, w0, flagged = [], 0, 0
    for m in (1, 299, 600):
        w1 = w0 + m
        sl = slice(wl.index_at("samples", wl.t_begin(w0)), wl.index_at("samples", wl.t_begin(w1)))
        el = slice(wl.index_at("events", wl.t_begin(w0)), wl.index_at("events", wl.t_begin(w1)))
        assert (sl.stop - sl.start) * 8 < wl.n_buffers * m or m == 1  # the sequential path (W > 1)
        ref = orc.reduce(s[sl], e[el], t_end[w0:w1], want_all_stats=True)
        rows.append(ref["all_stats"])
        mon.ingest(_dev(s[sl]), _dev(e[el]))
        got = mon.window_reduce(t_end[w0:w1])
        assert_same(got, ref, mon)
        flagged += int(ref["summary"]["n_hung"].sum())
        w0 = w1
    assert flagged > 0
    A = np.concatenate(rows)
    for q, b in enumerate(watched):
        ser = mon.watch_series(q)
        for f in ("integral", "last", "max", "min", "capacity", "n_samples", "mean_occ"):
            assert np.array_equal(ser[f], A[-300:, b][f]), (b, f)


@pytest.mark.parametrize("hang_mode,rank_mode", [(0, 0), (1, 0), (0, 2)])
def test_windowed_fold_compacted_finalize(hang_mode, rank_mode):
    """Calls with 1/8 .. 1 kept samples per buffer-window (C4's density) take the windowed fold with
    the compacted finalize (untouched cells resolved in one pass, touched buffers finalized 32 at a
    time): 20 000 buffers, 0.5 samples per buffer-window, calls of 40 and 23 windows, watched
    buffers, both hang criteria and the MEAN ranking - summaries, top-k, progress, hang lists, the
    last window's table and the value-monitor rings equal the oracle's."""
    wl = gen.C1.scaled("C1-cf", n_samples=630_000, n_events=63_000, n_buffers=20_000, n_windows=63, k=32,
                       hang_windows=3)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=3, k=wl.k, hang_mode=hang_mode, rank_mode=rank_mode)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    watched = [0, 777, 19999]
    mon.watch(watched)
    s, e = gen.samples(wl), gen.events(wl)
    t_end = wl.t_end()
    rows, w0 = [], 0
    for m in (40, 23):
        w1 = w0 + m
        sl = slice(wl.index_at("samples", wl.t_begin(w0)), wl.index_at("samples", wl.t_begin(w1)))
        el = slice(wl.index_at("events", wl.t_begin(w0)), wl.index_at("events", wl.t_begin(w1)))
        n = sl.stop - sl.start
        assert wl.n_buffers * m / 8 < n < wl.n_buffers * m  # windowed fold, compacted finalize
        ref = orc.reduce(s[sl], e[el], t_end[w0:w1], want_all_stats=True)
        rows.append(ref["all_stats"])
        mon.ingest(_dev(s[sl]), _dev(e[el]))
        assert_same(mon.window_reduce(t_end[w0:w1]), ref, mon)
        w0 = w1
    A = np.concatenate(rows)
    for q, b in enumerate(watched):
        ser = mon.watch_series(q)
        for f in ("integral", "last", "max", "min", "capacity", "n_samples", "mean_occ"):
            assert np.array_equal(ser[f], A[-len(ser):, b][f]), (b, f)


@pytest.mark.parametrize("hang_mode", [0, 1])
def test_range_parallel_sequential_fold(hang_mode):
    """Very sparse calls of >= 128 windows on the two-pass path (C5's shape: 327 680 buffers, ~0.02
    samples per buffer-window) fold each bin's windows in several ranges at once: a range starts
    from every buffer's latest kept sample in the earlier ranges (k_subpart's end keys), else the
    call's carry-in.  Two calls of 260 windows, H small enough to flag components, watched buffers:
    every window's summary, top-k, progress, hang list, the last window's table and the rings."""
    wl = gen.C5.scaled("C5-ranges", n_samples=1_800_000, n_events=180_000, n_windows=520, hang_windows=6)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=6, k=wl.k, hang_mode=hang_mode)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    watched = [3, 100_000, wl.n_buffers - 1]
    mon.watch(watched)
    s, e = gen.samples(wl), gen.events(wl)
    t_end = wl.t_end()
    rows, w0, flagged = [], 0, 0
    for m in (260, 260):
        w1 = w0 + m
        sl = slice(wl.index_at("samples", wl.t_begin(w0)), wl.index_at("samples", wl.t_begin(w1)))
        el = slice(wl.index_at("events", wl.t_begin(w0)), wl.index_at("events", wl.t_begin(w1)))
        assert (sl.stop - sl.start) * 8 < wl.n_buffers * m  # sequential fold, ranges (W >= 128)
        ref = orc.reduce(s[sl], e[el], t_end[w0:w1], want_all_stats=True)
        rows.append(ref["all_stats"])
        mon.ingest(_dev(s[sl]), _dev(e[el]))
        assert_same(mon.window_reduce(t_end[w0:w1]), ref, mon)
        flagged += int(ref["summary"]["n_hung"].sum())
        w0 = w1
    assert flagged > 0
    A = np.concatenate(rows)
    for q, b in enumerate(watched):
        ser = mon.watch_series(q)
        for f in ("integral", "last", "max", "min", "capacity", "n_samples", "mean_occ"):
            assert np.array_equal(ser[f], A[-300:, b][f]), (b, f)


def test_large_registry_bins_of_128_dense_and_sparse_calls():
    """Registries of 131073 .. 524288 buffers use bins of 128 buffers (C5's 327680): the fallback
    partition with 128-buffer bins and every fold path on them - a dense call (>= 2 samples per
    buffer-window: windowed chain fold), a sparse one (look-back over 3 windows per step) and a
    very sparse one (sequential fold) - against the oracle."""
    wl = gen.C1.scaled("C1-bl7", n_samples=3_600_000, n_events=360_000, n_buffers=140_000, n_windows=40)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=2, k=wl.k)
    orc, mon = _pair(owner, cap, tot, wl.n_components, **kw)
    s, e = gen.samples(wl), gen.events(wl)
    t_end = wl.t_end()
    calls = ([int(t_end[3])], [int(x) for x in t_end[4:8]])  # 2.6 and 0.64 samples per buffer-window
    w0 = 0
    for ends in calls:
        w1 = w0 + (4 if len(ends) == 1 else len(ends))
        sl = slice(wl.index_at("samples", wl.t_begin(w0)), wl.index_at("samples", wl.t_begin(w1)))
        el = slice(wl.index_at("events", wl.t_begin(w0)), wl.index_at("events", wl.t_begin(w1)))
        ref = orc.reduce(s[sl], e[el], ends)
        mon.ingest(_dev(s[sl]), _dev(e[el]))
        assert_same(mon.window_reduce(ends), ref, mon)
        w0 = w1
    t_end = t_end[:8]
    # a very sparse call: few records over many windows
    ends = [int(t_end[-1]) + 1000 * (i + 1) for i in range(40)]
    few = sample_array([(int(t_end[-1]) + 37 * i, (i * 7919) % wl.n_buffers, 1, int(cap[(i * 7919) % wl.n_buffers]))
                        for i in range(500)])
    ref = orc.reduce(few, event_array([]), ends)
    mon.ingest(_dev(few), None)
    assert_same(mon.window_reduce(ends), ref, mon)


@pytest.mark.parametrize("on_stream", [0, 1])
def test_c_abi_allgather_callback_two_ranks(on_stream):
    """The C-level multi-rank path: two contexts (world 2, owner sharding) on cuda:0, each driven
    by its own thread through rtm_window_reduce with an `allgather` callback (host-synchronised, or
    stream-ordered with allgather_on_stream), then rtm_sync_tables through the same callback; both
    ranks' merged results and tables equal the whole-trace oracle."""
    import ctypes
    import threading

    wl = gen.C1.scaled("C1-cb", n_samples=150_000, n_events=15_000, n_windows=5)
    owner, cap, tot = gen.registry(wl)
    kw = dict(t0=wl.t0, hang_windows=2, k=wl.k)
    orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, **kw)
    ref = orc.reduce(gen.samples(wl), gen.events(wl), wl.t_end())
    G = 2
    cudart = ctypes.CDLL("libcudart.so.12")
    cudart.cudaMemcpy.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int]
    cudart.cudaStreamSynchronize.argtypes = [ctypes.c_void_p]
    barrier = threading.Barrier(G)
    sends = [None] * G
    streams = [torch.cuda.Stream() for _ in range(G)]

    def make_cb(r):
        def cb(user, send, recv, nbytes):
            if on_stream:  # the callback must order itself: finish this rank's pack first
                cudart.cudaStreamSynchronize(ctypes.c_void_p(streams[r].cuda_stream))
            sends[r] = send
            barrier.wait()
            for q in range(G):
                if cudart.cudaMemcpy(ctypes.c_void_p(recv + q * nbytes), ctypes.c_void_p(sends[q]), nbytes, 3):
                    return 1
            barrier.wait()
            return 0
        return N.ALLGATHER_FN(cb)

    cbs = [make_cb(r) for r in range(G)]
    mons, keep = [], []
    for r in range(G):
        owned = (np.arange(wl.n_components) % G == r).astype(np.uint8)
        m = Monitor(owner, cap, tot, n_components=wl.n_components, rank=r, world=G, owned_components=owned,
                    stream=streams[r], **kw)
        # swap in a context whose config carries the callback (the binding's own uses the two-phase API)
        cfg = N.Config()
        cfg.n_buffers, cfg.n_components, cfg.n_kernels = len(owner), wl.n_components, len(tot)
        cfg.buffer_owner, cfg.buffer_capacity, cfg.kernel_total = m._owner.ctypes.data, m._cap.ctypes.data, m._tot.ctypes.data
        cfg.t0, cfg.hang_windows, cfg.k, cfg.rank_mode = wl.t0, 2, wl.k, 0
        cfg.device, cfg.rank, cfg.world = 0, r, G
        cfg.owned_components = owned.ctypes.data
        cfg.allgather = cbs[r]
        cfg.stream = streams[r].cuda_stream
        cfg.allgather_on_stream = on_stream
        h = ctypes.c_void_p()
        N.check(N.lib().rtm_create(ctypes.byref(cfg), ctypes.byref(h)), "rtm_create")
        N.lib().rtm_destroy(m._h)
        m._h = h
        keep.append(owned)
        s, e = gen.samples(wl, shard=(G, r)), gen.events(wl, shard=(G, r))
        keep += [s, e]
        N.check(N.lib().rtm_ingest(m._h, s.ctypes.data, len(s), e.ctypes.data, len(e), N.RTM_MEM_HOST), "ingest")
        mons.append(m)
    ends = np.ascontiguousarray(wl.t_end())
    rcs = [None] * G
    summs = [np.zeros(wl.n_windows, N.SUMMARY_DTYPE) for _ in range(G)]

    def run(r):
        rcs[r] = N.lib().rtm_window_reduce(mons[r]._h, ends.ctypes.data, len(ends), summs[r].ctypes.data)
        if rcs[r] == 0:
            rcs[r] = N.lib().rtm_sync_tables(mons[r]._h)

    th = [threading.Thread(target=run, args=(r,)) for r in range(G)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=120)
    assert rcs == [0, 0], rcs
    for r, m in enumerate(mons):
        m.W = wl.n_windows
        m._synced = True
        got = m.results()
        assert np.array_equal(got["summary"], summs[r])
        assert_same(got, ref, m)
        assert np.array_equal(m.topk_persistence(), orc.persistence())
