"""Pins for the CPU oracle (oracle/oracle.c) against things other than itself (CPU only).

Each pin is chosen so that a plausible mistake in the oracle (dropped carry-in term, wrong
window boundary, transposed ratio, wrong tie direction, off-by-one in the hang run) fails:
  - values the paper prints (Fig. 3 buffer table),
  - hand-worked closed forms (tests/golden/worked_examples.json),
  - the paper's case studies turned into constructed traces (L197-L199, L217-L229),
  - a structurally different brute force (oracle/brute.py) on random tiny traces,
  - invariants of the definition on a C1-shaped synthetic trace,
  - known splitmix64 output for the digest mixer.
"""
from __future__ import annotations

import json
import os
from fractions import Fraction

import numpy as np
import pytest

import gen
import oracle
from oracle import brute
from tests.helpers import event_array, pack_meta, random_tiny_case, sample_array

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ---------------------------------------------------------------------------------------------
def test_splitmix64_known_vector():
    # splitmix64 from state 0: first output is 0xE220A8397B1DCDAF (Steele et al. 2014 reference)
    assert gen.splitmix64(0) == 0xE220A8397B1DCDAF
    assert brute.fmix64(0x9E3779B97F4A7C15) == 0xE220A8397B1DCDAF


def test_digest_term_detects_any_single_field_change():
    """DESIGN.md reading R17: odd-constant products are bijections and fmix64 is a bijection, so
    changing exactly one field (buffer, last, max, min, cap, n, integral) always changes the term."""
    rng = np.random.default_rng(9)
    for _ in range(300):
        f = [int(rng.integers(0, 2**31)), *(int(x) for x in rng.integers(0, 65536, 4)), int(rng.integers(0, 2**32)),
             int(rng.integers(-(2**62), 2**62))]
        base = oracle.digest_term(*f)
        for i in range(7):
            g = list(f)
            g[i] = g[i] + 1 if i != 6 else g[i] - 12345
            if i in (1, 2, 3, 4):
                g[i] &= 0xFFFF
            assert oracle.digest_term(*g) != base, i


def test_digest_term_matches_spec_retyped():
    rng = np.random.default_rng(7)
    for _ in range(200):
        b, last, mx, mn, cap = (int(x) for x in rng.integers(0, 65536, 5))
        n = int(rng.integers(0, 2**32))
        integral = int(rng.integers(-(2**62), 2**62))
        assert oracle.digest_term(b, last, mx, mn, cap, n, integral) == brute.digest_term(b, last, mx, mn, cap, n,
                                                                                        integral)


# ---------------------------------------------------------------------------------------------
def _single_buffer(cap, t0):
    return oracle.Oracle(np.array([0], np.uint32), np.array([cap], np.uint16), np.array([5], np.int64),
                         n_components=1, t0=t0, hang_windows=1, k=1)


@pytest.mark.parametrize("case", json.load(open(os.path.join(GOLDEN, "worked_examples.json")))["cases"],
                         ids=lambda c: c["name"])
def test_worked_examples(case):
    cap, lin = case["cap"], case["L_in"]
    tb, te = case["window"]
    orc = _single_buffer(cap, tb - 10)
    # establish the carry-in level L_in with a first window [tb-10, tb)
    pre = orc.reduce(sample_array([(tb - 5, 0, lin, cap)]), event_array([]), [tb])
    assert pre["rc"] == 0
    out = orc.reduce(sample_array([(ts, 0, lvl, cap) for ts, lvl in case["samples"]]), event_array([]), [te])
    assert out["rc"] == 0
    st = out["stats"][0]
    assert int(st["integral"]) == case["integral"]
    assert (int(st["last"]), int(st["max"]), int(st["min"])) == (case["last"], case["max"], case["min"])
    assert int(st["n_samples"]) == case["n"]
    assert float(st["mean_occ"]) == case["mean_occ"]
    assert (int(st["min"]) == cap) == case["full"]


# ---------------------------------------------------------------------------------------------
def _fig3():
    rows = [ln.split() for ln in open(os.path.join(GOLDEN, "fig3_buffers.txt")) if not ln.startswith("#")]
    ids = [int(r[0]) for r in rows]
    size = [int(r[1]) for r in rows]
    cap = [int(r[2]) for r in rows]
    assert ids == list(range(12))
    return size, cap


@pytest.mark.parametrize("mode,expected", [(1, list(range(12))), (0, [0, 1, 2, 3, 4, 5, 7, 8, 9, 10, 11, 6])])
def test_fig3_bottleneck_analyzer_order(mode, expected):
    size, cap = _fig3()
    orc = oracle.Oracle(np.arange(12, dtype=np.uint32), np.array(cap, np.uint16), np.array([1], np.int64),
                        n_components=12, t0=0, hang_windows=1, k=12, rank_mode=mode)
    s = sample_array([(i, i, size[i], cap[i]) for i in range(12)])
    out = orc.reduce(s, event_array([]), [100])
    assert out["rc"] == 0 and out["topk_n"][0] == 12
    assert [int(x) for x in out["topk"][0]["buffer_id"]] == expected
    assert [int(x) for x in out["topk"][0]["level"]] == [size[i] for i in expected]


def test_fig4_chain_top1_is_C():
    # chain A->B->C->D, only C's buffer is full => C is the bottleneck.
    caps = [8, 8, 8, 8]
    levels = {"A": 5, "B": 3, "C": 8, "D": 2}
    orc = oracle.Oracle(np.arange(4, dtype=np.uint32), np.array(caps, np.uint16), np.array([1], np.int64),
                        n_components=4, t0=0, hang_windows=1, k=1)
    s = sample_array([(1, i, levels[n], 8) for i, n in enumerate("ABCD")])
    out = orc.reduce(s, event_array([]), [10])
    assert int(out["topk"][0][0]["buffer_id"]) == 2


# ---------------------------------------------------------------------------------------------
def _deadlock_trace():
    """Case study 2 as a constructed trace.
    comps: 0 L1, 1 L2 local storage, 2 L2 write buffer, 3 DRAM ctrl, 4 CU (buffer b owned by comp b)."""
    caps = [4, 4, 4, 4, 8]
    S, E = [], []
    task = 0

    def act(c, tp):
        nonlocal task
        E.append((tp + 10, task, pack_meta(c, 0, 0)))
        E.append((tp + 20, task, pack_meta(c, 0, 1)))
        task += 1

    S.append((0, 4, 8, 8))  # CU buffer constantly full (case study 1's 8/8 ROB port, L197-L199)
    for w in range(6):
        tp = 100 * w
        if w < 3:
            S.append((tp + 5, 0, 1, 4))
        elif w == 3:
            S.append((tp + 1, 0, 2, 4))
        if w < 3:
            for b in (1, 2, 3):
                S.append((tp + 5, b, 2, 4))
        if w == 2:
            S.append((250, 1, 4, 4))
            S.append((250, 2, 4, 4))
        if w == 3:
            S.append((320, 0, 4, 4))
            S.append((320, 3, 4, 4))
        evs = []
        for c in range(5):
            if (c in (1, 2) and w >= 3) or (c in (0, 3) and w >= 4):
                continue
            evs.append(c)
        for c in evs:
            act(c, tp)
    S.sort(key=lambda r: r[0])
    E.sort(key=lambda r: r[0])
    # a 320-level sample of buffer 0 must come after its tp+1 sample of window 3: sorted by ts keeps that
    return caps, S, E


def test_case_study2_deadlock_flags_and_case_study1_negative():
    caps, S, E = _deadlock_trace()
    orc = oracle.Oracle(np.arange(5, dtype=np.uint32), np.array(caps, np.uint16), np.array([100], np.int64),
                        n_components=5, t0=0, hang_windows=2, k=5)
    out = orc.reduce(sample_array(S), event_array(E), [100 * (w + 1) for w in range(6)], want_all_stats=True)
    assert out["rc"] == 0
    flagged = [list(np.nonzero(out["hung"][w])[0]) for w in range(6)]
    assert flagged == [[], [], [], [], [1, 2], [0, 1, 2, 3]]
    assert list(out["summary"]["n_hung"]) == [0, 0, 0, 0, 2, 4]
    # component 4: constantly 8/8 but active -> bottleneck, never a hang; mean occupancy exactly 1
    assert all(out["hung"][w][4] == 0 for w in range(6))
    assert all(float(out["all_stats"][w][4]["mean_occ"]) == 1.0 for w in range(6))
    # a completed run drains every buffer: no component is flagged afterwards (L229)
    drain = sample_array([(601, b, 0, caps[b]) for b in range(5)])
    out2 = orc.reduce(drain, event_array([]), [700, 800, 900])
    assert out2["rc"] == 0 and int(out2["summary"]["n_hung"].sum()) == 0


# ---------------------------------------------------------------------------------------------
def _run_both(case):
    kw = dict(t0=case["t0"], hang_windows=case["H"], k=case["k"], rank_mode=case["mode"])
    orc = oracle.Oracle(case["owner"], case["caps"], case["totals"], n_components=case["nc"], **kw)
    br = brute.Brute(case["owner"], case["caps"], case["totals"], case["nc"], **kw)
    results = []
    for srows, erows, ends in case["calls"]:
        o = orc.reduce(sample_array(srows), event_array(erows), ends, want_all_stats=True)
        try:
            b = br.reduce(srows, erows, ends)
        except brute.OrderError:
            b = "order"
        results.append((o, b))
        if b == "order":
            break
    return results


def _compare(o, b, nb, nk, nc):
    assert o["rc"] == 0
    for w, bw in enumerate(b):
        s = o["summary"][w]
        for f in ("t_begin", "t_end", "n_samples", "n_events", "n_dropped", "digest", "n_touched", "n_hung"):
            assert int(s[f]) == bw[f], (w, f)
        n = int(o["topk_n"][w])
        assert [(int(x["buffer_id"]), int(x["level"]), int(x["capacity"])) for x in o["topk"][w][:n]] == bw["topk"]
        for k in range(nk):
            for f in ("total", "started", "finished", "in_flight", "not_started"):
                assert int(o["progress"][w][k][f]) == bw["progress"][k][f]
        assert [c for c in range(nc) if o["hung"][w][c]] == bw["hung"]
        for bb in range(nb):
            st, bs = o["all_stats"][w][bb], bw["stats"][bb]
            for f in ("integral", "last", "max", "min", "capacity", "n_samples"):
                assert int(st[f]) == bs[f], (w, bb, f)
            assert float(st["mean_occ"]) == pytest.approx(bs["mean_occ"], rel=1e-15, abs=0)


@pytest.mark.parametrize("seed", range(60))
def test_oracle_matches_brute_force(seed):
    rng = np.random.default_rng(1000 + seed)
    case = random_tiny_case(rng, allow_disorder=(seed % 4 == 3))
    for o, b in _run_both(case):
        if b == "order":
            assert o["rc"] == -4
        else:
            _compare(o, b, case["nb"], case["nk"], case["nc"])


def test_order_violation_is_sticky():
    orc = _single_buffer(8, 0)
    bad = sample_array([(5, 0, 1, 8), (3, 0, 2, 8)])
    assert orc.reduce(bad, event_array([]), [10])["rc"] == -4
    assert orc.reduce(sample_array([]), event_array([]), [20])["rc"] == -4
    orc.reset()
    assert orc.reduce(sample_array([]), event_array([]), [20])["rc"] == 0


def test_invalid_arguments_leave_state():
    orc = _single_buffer(8, 0)
    assert orc.reduce(sample_array([]), event_array([]), [10, 5])["rc"] == -1  # t_end decreasing
    assert orc.reduce(sample_array([]), event_array([]), [-1])["rc"] == -1     # before t_prev
    out = orc.reduce(sample_array([(1, 0, 3, 8)]), event_array([]), [10])
    assert out["rc"] == 0 and out["summary"][0]["t_begin"] == 0


# ---------------------------------------------------------------------------------------------
def test_percent_key_is_exactly_order_preserving():
    """The CUDA path ranks by key32 = floor(l*2^32/c) (l<c), 2^32-1 (l==c); exact vs Fraction."""
    rng = np.random.default_rng(3)

    def key(l, c):
        return 0xFFFFFFFF if l == c else (l << 32) // c

    pairs = []
    for _ in range(20000):
        c1, c2 = (int(x) for x in rng.integers(1, 65536, 2))
        l1, l2 = int(rng.integers(0, c1 + 1)), int(rng.integers(0, c2 + 1))
        pairs.append((l1, c1, l2, c2))
    # near-Farey neighbours: a/b vs (a*q+1)/(b*q) style adjacent ratios with large denominators
    for c in (65535, 65534, 65521, 40000):
        for l in (1, 2, c // 2, c - 2, c - 1):
            pairs.append((l, c, l + 1, c + 1) if l + 1 <= c + 1 <= 65535 else (l, c, l, c))
            pairs.append((l, c, l * 2 + 1, min(65535, c * 2)))
    for l1, c1, l2, c2 in pairs:
        if l2 > c2:
            continue
        f = (Fraction(l1, c1) > Fraction(l2, c2)) - (Fraction(l1, c1) < Fraction(l2, c2))
        k = (key(l1, c1) > key(l2, c2)) - (key(l1, c1) < key(l2, c2))
        assert f == k, (l1, c1, l2, c2)


# ---------------------------------------------------------------------------------------------
@pytest.fixture(scope="module")
def c1_run():
    wl = gen.C1_INVALID
    owner, cap, tot = gen.registry(wl)
    s, e = gen.samples(wl), gen.events(wl)
    orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, t0=wl.t0, hang_windows=wl.hang_windows,
                        k=wl.k)
    out = orc.reduce(s, e, wl.t_end(), want_all_stats=True)
    assert out["rc"] == 0
    return wl, owner, cap, tot, s, e, out


def test_c1_progress_invariants(c1_run):
    wl, owner, cap, tot, s, e, out = c1_run
    p = out["progress"]
    assert np.all(p["finished"] + p["in_flight"] + p["not_started"] == p["total"])  # L131
    assert np.all(p["in_flight"] == p["started"] - p["finished"])
    assert np.all(np.diff(p["started"], axis=0) >= 0) and np.all(np.diff(p["finished"], axis=0) >= 0)
    comps = out["comps"]
    assert int(comps["in_flight"].sum()) == int(p["in_flight"][-1].sum())  # one comp + one kernel per task
    assert int(comps["started"].sum()) == int(p["started"][-1].sum())


def test_c1_counts_and_drops(c1_run):
    wl, owner, cap, tot, s, e, out = c1_run
    S = out["summary"]
    # every record is either kept in exactly one window or dropped exactly once
    assert int(S["n_samples"].sum() + S["n_events"].sum() + S["n_dropped"].sum()) == len(s) + len(e)
    valid = (s["buffer_id"] < wl.n_buffers)
    valid &= s["capacity"] == cap[np.minimum(s["buffer_id"], wl.n_buffers - 1)]
    valid &= s["level"] <= s["capacity"]
    ends = wl.t_end()
    inrange = (s["ts"] >= wl.t0) & (s["ts"] < ends[-1])
    assert int(S["n_samples"].sum()) == int((valid & inrange).sum())
    assert int(S["n_dropped"].sum()) > 0


def test_c1_carry_and_untouched_invariants(c1_run):
    wl, owner, cap, tot, s, e, out = c1_run
    A = out["all_stats"]
    ends = wl.t_end()
    W = np.diff(np.concatenate([[wl.t0], ends]))
    for w in range(1, wl.n_windows):
        untouched = A[w]["n_samples"] == 0
        lin = A[w - 1]["last"]
        assert np.all(A[w]["last"][untouched] == lin[untouched])
        assert np.all(A[w]["max"][untouched] == lin[untouched]) and np.all(A[w]["min"][untouched] == lin[untouched])
        assert np.all(A[w]["integral"][untouched] == lin[untouched].astype(np.int64) * W[w])
        assert np.all(A[w]["max"] >= lin) and np.all(A[w]["min"] <= lin)  # carry-in counts toward max/min


def test_c1_integral_sums_to_whole_run(c1_run):
    """sum_w I_b(w) equals the whole-run integral computed by an independent vectorised method."""
    wl, owner, cap, tot, s, e, out = c1_run
    ends = wl.t_end()
    valid = (s["buffer_id"] < wl.n_buffers)
    valid &= s["capacity"] == cap[np.minimum(s["buffer_id"], wl.n_buffers - 1)]
    valid &= s["level"] <= s["capacity"]
    valid &= (s["ts"] >= wl.t0) & (s["ts"] < ends[-1])
    k = s[valid]
    order = np.argsort(k["buffer_id"], kind="stable")
    b, ts, lv = k["buffer_id"][order], k["ts"][order], k["level"][order].astype(np.int64)
    nxt = np.empty_like(ts)
    nxt[:-1] = ts[1:]
    last_of_b = np.ones(len(b), bool)
    last_of_b[:-1] = b[1:] != b[:-1]
    nxt[last_of_b] = ends[-1]
    whole = np.zeros(wl.n_buffers, np.int64)
    np.add.at(whole, b, lv * (nxt - ts))  # level 0 before the first sample contributes 0
    assert np.array_equal(out["all_stats"]["integral"].sum(axis=0), whole)


def test_c1_topk_matches_fraction_sort(c1_run):
    wl, owner, cap, tot, s, e, out = c1_run
    A = out["all_stats"]
    for w in (0, wl.n_windows // 2, wl.n_windows - 1):
        order = sorted(range(wl.n_buffers), key=lambda b: (-Fraction(int(A[w][b]["last"]), int(cap[b])), b))
        assert [int(x) for x in out["topk"][w]["buffer_id"]] == order[: wl.k]


def test_c1_batch_invariance(c1_run):
    wl, owner, cap, tot, s, e, out = c1_run
    ends = wl.t_end()
    orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, t0=wl.t0, hang_windows=wl.hang_windows,
                        k=wl.k)
    # windows delivered in three calls; each call gets exactly the records inside its windows
    parts = [(0, 3), (3, 4), (4, 10)]
    for a, bnd in parts:
        lo = wl.t0 if a == 0 else ends[a - 1]
        hi = ends[bnd - 1]
        # field-invalid records travel with the call that holds the next valid record (drop attribution)
        valid = (s["buffer_id"] < wl.n_buffers)
        valid &= s["capacity"] == cap[np.minimum(s["buffer_id"], wl.n_buffers - 1)]
        valid &= s["level"] <= s["capacity"]
        idx_valid = np.nonzero(valid)[0]
        first = np.searchsorted(s["ts"][idx_valid], lo) if a else 0
        last = np.searchsorted(s["ts"][idx_valid], hi)
        i0 = 0 if first == 0 else idx_valid[first - 1] + 1
        i1 = len(s) if last >= len(idx_valid) or bnd == 10 else idx_valid[last - 1] + 1
        ev = e[(e["ts"] >= lo) & (e["ts"] < hi)]
        part = orc.reduce(s[i0:i1], ev, ends[a:bnd])
        assert part["rc"] == 0
        for f in ("n_samples", "digest", "n_touched", "n_hung"):
            assert np.array_equal(part["summary"][f], out["summary"][f][a:bnd]), f
        assert np.array_equal(part["topk"], out["topk"][a:bnd])
        assert np.array_equal(part["progress"], out["progress"][a:bnd])


def test_shard_merge_equals_whole():
    """Owner-component sharding: per-shard oracle + merge == whole-trace oracle."""
    wl = gen.C1.scaled("C1-shard", n_samples=200_000, n_events=20_000, n_windows=6)
    owner, cap, tot = gen.registry(wl)
    kw = dict(n_components=wl.n_components, t0=wl.t0, hang_windows=2, k=wl.k)
    whole = oracle.Oracle(owner, cap, tot, **kw).reduce(gen.samples(wl), gen.events(wl), wl.t_end())
    shards = []
    for r in range(3):
        owned = (np.arange(wl.n_components) % 3 == r).astype(np.uint8)
        o = oracle.Oracle(owner, cap, tot, owned=owned, **kw)
        shards.append(o.reduce(gen.samples(wl, shard=(3, r)), gen.events(wl, shard=(3, r)), wl.t_end()))
    top, top_n = oracle.merge_topk(shards, wl.k)
    assert np.array_equal(top, whole["topk"]) and np.array_equal(top_n, whole["topk_n"])
    for f in ("n_samples", "n_events", "n_dropped", "n_touched", "n_hung"):
        assert np.array_equal(sum(sh["summary"][f].astype(np.uint64) for sh in shards), whole["summary"][f])
    dig = np.zeros(wl.n_windows, np.uint64)
    for sh in shards:
        dig += sh["summary"]["digest"]
    assert np.array_equal(dig, whole["summary"]["digest"])
    for f in ("started", "finished"):
        assert np.array_equal(sum(sh["progress"][f] for sh in shards), whole["progress"][f])
    hung = np.zeros_like(whole["hung"])
    for sh in shards:
        hung |= sh["hung"]
    assert np.array_equal(hung, whole["hung"])


def test_shard_topk_mean_decomposes():
    """Rank mode MEAN at world > 1: the merge ranks the union of the shards' lists by
    their exchanged order keys, which is exact iff, in every window, each shard's list is the prefix
    of the whole-trace ranking restricted to that shard's owned buffers (then the whole top-k lies
    in the union, in the same relative order).  Checked on the oracle alone, no keys needed."""
    wl = gen.C1.scaled("C1-shard-mean", n_samples=200_000, n_events=20_000, n_windows=6)
    owner, cap, tot = gen.registry(wl)
    for k in (wl.k, 512):
        kw = dict(n_components=wl.n_components, t0=wl.t0, hang_windows=2, k=k, rank_mode=2)
        whole = oracle.Oracle(owner, cap, tot, **kw).reduce(gen.samples(wl), gen.events(wl), wl.t_end())
        for r in range(3):
            owned = (np.arange(wl.n_components) % 3 == r).astype(np.uint8)
            sh = oracle.Oracle(owner, cap, tot, owned=owned, **kw).reduce(gen.samples(wl, shard=(3, r)),
                                                                           gen.events(wl, shard=(3, r)), wl.t_end())
            n_owned = int(owned[owner].sum())
            for w in range(wl.n_windows):
                ids = [int(x) for x in sh["topk"][w]["buffer_id"][: sh["topk_n"][w]]]
                assert len(ids) == min(k, n_owned) and all(owned[owner[b]] for b in ids)
                mine = [int(b) for b in whole["topk"][w]["buffer_id"][: whole["topk_n"][w]] if owned[owner[b]]]
                assert ids[: len(mine)] == mine  # the whole list's owned part is this shard's prefix


def test_gpu_fullness_key_reciprocal_formula_is_exact():
    """The CUDA top-k computes floor(l*2^32/c) as q0 = (l*m)>>16, m = floor(2^48/c), plus one
    remainder fix-up (DESIGN.md §4 K5).  Emulated here exhaustively for small caps and on random
    pairs for large ones; it must equal the exact floor."""
    def gpu_key(l, c):
        if l >= c:
            return 0xFFFFFFFF
        m = (1 << 48) // c if c >= 2 else 0
        q = (l * m) >> 16
        r = (l << 32) - q * c
        if r >= c:
            q += 1
        return q

    for c in range(1, 300):
        for l in range(0, c):
            assert gpu_key(l, c) == (l << 32) // c
    rng = np.random.default_rng(11)
    for _ in range(50000):
        c = int(rng.integers(2, 65535))
        l = int(rng.integers(0, c))
        assert gpu_key(l, c) == (l << 32) // c
    for c in (65533, 65534, 40961, 32768, 32769):
        for l in (0, 1, c // 2, c - 2, c - 1):
            assert gpu_key(l, c) == (l << 32) // c


# ---------------------------------------------------------------------------------------------
# C3 (injected circular wait) and C4 (Zipf skew) shapes, oracle side
def _oracle_for(wl, **kw):
    owner, cap, tot = gen.registry(wl)
    args = dict(t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k)
    args.update(kw)
    return oracle.Oracle(owner, cap, tot, n_components=wl.n_components, **args)


def test_c3_small_injected_deadlock_is_flagged_and_nothing_else():
    """Case study 2 (L217, L229) at C3's shape: the injected pair is flagged from w_d + H - 1 on
    (at most `deadlock_lead` windows earlier if it happened to fall silent while its buffers were
    already held full), the upstream pair it backs up 5 windows later; the same trace without the
    injection flags nothing at this H (the calibration of H)."""
    wl = gen.C3_SMALL
    s, e = gen.samples(wl), gen.events(wl)
    r = _oracle_for(wl).reduce(s, e, wl.t_end(), want_topk=False)
    assert r["rc"] == 0
    hung = [set(np.nonzero(h)[0].tolist()) for h in r["hung"]]
    H, lead = wl.hang_windows, wl.deadlock_lead
    injected = set()
    for w_d, cs in wl.deadlock:
        for c in cs:
            injected.add(c)
            first = next(w for w in range(wl.n_windows) if c in hung[w])
            assert w_d + H - 1 - lead <= first <= w_d + H - 1
            assert all(c in hung[w] for w in range(w_d + H - 1, wl.n_windows))
    assert set().union(*hung) == injected
    clean = wl.scaled("C3-small-clean", deadlock=())
    rc = _oracle_for(clean).reduce(gen.samples(clean), gen.events(clean), clean.t_end(), want_topk=False)
    assert rc["hung"].sum() == 0
    # the injected components' stuck tasks stay in flight: no START / END after w_d
    w_d, (a, b) = wl.deadlock[0]
    comp = e["meta"] & 0xFFFFF
    assert not np.any(np.isin(comp[e["ts"] >= wl.t_begin(w_d)], [a, b]))


def test_c3_small_streamed_batches_equal_one_call():
    """The oracle context carries state across calls: streaming the trace in window batches (the
    way the large GPU parity tests drive it) gives the one-call results."""
    wl = gen.C3_SMALL.scaled("C3-batch", n_samples=2_000_000, n_events=200_000, n_windows=40,
                             deadlock=((20, (11240, 11243)),), hang_windows=4)
    s, e = gen.samples(wl), gen.events(wl)
    one = _oracle_for(wl).reduce(s, e, wl.t_end())
    orc = _oracle_for(wl)
    for w0 in range(0, wl.n_windows, 7):
        w1 = min(wl.n_windows, w0 + 7)
        sl = slice(wl.index_at("samples", wl.t_begin(w0)), wl.index_at("samples", wl.t_begin(w1)))
        el = slice(wl.index_at("events", wl.t_begin(w0)), wl.index_at("events", wl.t_begin(w1)))
        r = orc.reduce(s[sl], e[el], wl.t_end()[w0:w1])
        assert np.array_equal(r["summary"], one["summary"][w0:w1])
        assert np.array_equal(r["topk"], one["topk"][w0:w1])
        assert np.array_equal(r["progress"], one["progress"][w0:w1])
        assert np.array_equal(r["hung"], one["hung"][w0:w1])
    assert np.array_equal(r["stats"], one["stats"])


def test_zipf_generator_shape():
    """C4's buffer ids: Zipf(0.99) rank frequencies (top-1 share = 1 / H_{n,s}), scattered by a
    bijection over the id space."""
    wl = gen.C4_SMALL
    s = gen.samples(wl, 0, 1_000_000)
    cnt = np.bincount(s["buffer_id"], minlength=wl.n_buffers)
    r = np.arange(1, wl.n_buffers + 1, dtype=np.float64)
    p1 = 1.0 / np.sum(r ** -wl.zipf_s)
    top = np.sort(cnt)[::-1]
    assert abs(top[0] / len(s) - p1) < 5 * np.sqrt(p1 / len(s))
    assert abs(top[1] / len(s) - p1 / 2 ** wl.zipf_s) < 5 * np.sqrt(p1 / len(s))
    t = wl.zipf_table()
    assert np.all(np.diff(t.astype(np.float64)) >= 0) and t[-1] == np.uint64(2**64 - 1)
    p = wl.params()
    ids = (np.arange(wl.n_buffers, dtype=np.uint64) * p.zipf_a + p.zipf_b) % wl.n_buffers
    assert len(np.unique(ids)) == wl.n_buffers


def test_c4_small_oracle_topk_matches_fraction_sort():
    """k = 1024 under skew: the oracle's top-k of the last window equals an exact Fraction sort."""
    wl = gen.C4_SMALL.scaled("C4-tiny", n_samples=2_000_000, n_events=200_000, n_windows=3,
                             n_buffers=1 << 16)
    s, e = gen.samples(wl), gen.events(wl)
    r = _oracle_for(wl).reduce(s, e, wl.t_end())
    st = r["stats"]
    order = sorted(range(wl.n_buffers), key=lambda b: (-Fraction(int(st["last"][b]), int(st["capacity"][b])), b))
    assert r["topk"][-1]["buffer_id"].tolist() == order[:wl.k]


# ---------------------------------------------------------------------------------------------
# Persistence ranking: rank mode 2 = the window's time-weighted mean
# occupancy; windows-in-top-k counter
@pytest.mark.parametrize("seed", range(40))
def test_mean_occupancy_ranking_and_persistence_match_brute_force(seed):
    """Against brute.py's tick-loop integral ranked with exact Fractions I / (cap * W), and the
    persistence counter against counting the brute force's top-k lists."""
    rng = np.random.default_rng(5000 + seed)
    case = random_tiny_case(rng)
    case["mode"] = 2
    kw = dict(t0=case["t0"], hang_windows=case["H"], k=case["k"], rank_mode=2)
    orc = oracle.Oracle(case["owner"], case["caps"], case["totals"], n_components=case["nc"], **kw)
    br = brute.Brute(case["owner"], case["caps"], case["totals"], case["nc"], **kw)
    counts = np.zeros(case["nb"], np.uint32)
    for srows, erows, ends in case["calls"]:
        o = orc.reduce(sample_array(srows), event_array(erows), ends, want_all_stats=True)
        b = br.reduce(srows, erows, ends)
        _compare(o, b, case["nb"], case["nk"], case["nc"])
        for bw in b:
            for bid, _, _ in bw["topk"]:
                counts[bid] += 1
    assert np.array_equal(orc.persistence(), counts)


def test_mean_ranking_closed_forms():
    """(i) A window without samples holds every level constant, so mean occupancy = level / cap
    exactly and the mean ranking equals the Percent ranking (Fig. 3 table as levels).
    (ii) Worked example E1 (integral 46 of 80 -> 0.575) ranks below a buffer full the whole
    window (1.0) and above one at 1/4 all window (0.25), ties by id."""
    rows = [ln.split() for ln in open(os.path.join(GOLDEN, "fig3_buffers.txt")) if ln.strip() and not ln.startswith("#")]
    lvls = [int(r[1]) for r in rows]
    caps = np.array([int(r[2]) for r in rows], np.uint16)
    n = len(rows)
    owner = np.arange(n, dtype=np.uint32)
    fill = sample_array([(0, b, lvls[b], int(caps[b])) for b in range(n)])
    tops = {}
    for mode in (0, 2):
        orc = oracle.Oracle(owner, caps, np.ones(1, np.int64), n_components=n, t0=0, hang_windows=4, k=n,
                            rank_mode=mode)
        orc.reduce(fill, event_array([]), [1])
        r = orc.reduce(sample_array([]), event_array([]), [11])  # no samples: levels constant
        tops[mode] = r["topk"][0]["buffer_id"].tolist()
    assert tops[2] == tops[0]
    # (ii): buffers 0 (E1), 1 (full all window), 2 (2 of 8 all window), 3 (same as 1, higher id)
    caps = np.array([8, 4, 8, 4], np.uint16)
    orc = oracle.Oracle(np.arange(4, dtype=np.uint32), caps, np.ones(1, np.int64), n_components=4, t0=-10,
                        hang_windows=4, k=4, rank_mode=2)
    orc.reduce(sample_array([(-1, 0, 2, 8), (-1, 1, 4, 4), (-1, 2, 2, 8), (-1, 3, 4, 4)]), event_array([]), [0])
    r = orc.reduce(sample_array([(3, 0, 5, 8), (3, 0, 4, 8), (7, 0, 8, 8)]), event_array([]), [10],
                   want_all_stats=True)
    assert int(r["all_stats"][0][0]["integral"]) == 46
    assert r["topk"][0]["buffer_id"].tolist() == [1, 3, 0, 2]
    assert orc.persistence().tolist() == [2, 2, 2, 2]


# ---------------------------------------------------------------------------------------------
# Dynamic progress bars (Create/Update/DestroyProgressBar, L99, L131)
def _bar_ops(rng, nk):
    """A random sequence of registry operations (as (op, arg) tuples) applied between calls."""
    ops = []
    for _ in range(int(rng.integers(0, 4))):
        u = rng.random()
        if u < 0.4:
            ops.append(("destroy", int(rng.integers(0, nk))))
        elif u < 0.7:
            ops.append(("create", int(rng.integers(0, 20))))
        else:
            ops.append(("update", (int(rng.integers(0, nk)), int(rng.integers(0, 20)))))
    return ops


def _apply(ctx, op, arg):
    """Apply one registry op; returns the result or 'err' (both sides must agree)."""
    try:
        if op == "create":
            return ctx.bar_create(arg)
        if op == "update":
            return ctx.bar_update(*arg)
        return ctx.bar_destroy(arg)
    except Exception:
        return "err"


@pytest.mark.parametrize("seed", range(40))
def test_dynamic_progress_bars_match_brute_force(seed):
    """Bars created / updated / destroyed between calls: a destroyed id takes no events (they are
    dropped and counted), reads all-zero, and a re-created id starts from zero with its new total;
    the oracle equals brute.py on random tiny traces."""
    rng = np.random.default_rng(9000 + seed)
    case = random_tiny_case(rng)
    kw = dict(t0=case["t0"], hang_windows=case["H"], k=case["k"], rank_mode=case["mode"])
    orc = oracle.Oracle(case["owner"], case["caps"], case["totals"], n_components=case["nc"], **kw)
    br = brute.Brute(case["owner"], case["caps"], case["totals"], case["nc"], **kw)
    for srows, erows, ends in case["calls"]:
        for op, arg in _bar_ops(rng, case["nk"]):
            assert _apply(orc, op, arg) == _apply(br, op, arg)
        o = orc.reduce(sample_array(srows), event_array(erows), ends, want_all_stats=True)
        b = br.reduce(srows, erows, ends)
        _compare(o, b, case["nb"], case["nk"], case["nc"])


def test_dynamic_progress_bars_worked_example():
    """Bar 1 destroyed: its 2 events are dropped and it reads zero; re-created with total 5 it
    counts only later events (L131: finished / executing / not started)."""
    owner, cap = np.zeros(1, np.uint32), np.array([4], np.uint16)
    orc = oracle.Oracle(owner, cap, np.array([3, 4], np.int64), n_components=1, t0=0, k=1)
    ev = lambda rows: event_array([(t, i, pack_meta(0, kern, kind)) for t, i, kern, kind in rows])  # noqa: E731
    r = orc.reduce(sample_array([]), ev([(1, 0, 0, 0), (2, 1, 1, 0), (3, 1, 1, 1)]), [10])
    assert list(r["progress"][0][1].tolist()) == [4, 1, 1, 0, 3]
    orc.bar_destroy(1)
    r = orc.reduce(sample_array([]), ev([(11, 2, 1, 0), (12, 3, 1, 0), (13, 0, 0, 1)]), [20])
    assert int(r["summary"]["n_dropped"][0]) == 2 and int(r["summary"]["n_events"][0]) == 1
    assert list(r["progress"][0][1].tolist()) == [0, 0, 0, 0, 0]
    assert list(r["progress"][0][0].tolist()) == [3, 1, 1, 0, 2]
    assert orc.bar_create(5) == 1
    r = orc.reduce(sample_array([]), ev([(21, 4, 1, 0)]), [30])
    assert list(r["progress"][0][1].tolist()) == [5, 1, 0, 1, 4]
    with pytest.raises(ValueError):
        orc.bar_create(1)  # both ids live


# ---------------------------------------------------------------------------------------------
# Looser hang criterion and root causes
def test_hang_roots_case_study_2_and_chain():
    """Case study 2 (L217, L229, L235): L1 (0) and the DRAM controller (3) back up behind the L2
    write buffer (2) <-> local storage (1) circular wait: roots {1, 2}.  Fig. 4's chain A -> B ->
    C -> D (L161) with B and C stuck: C is the root (B waits on it); with D stuck too, D is."""
    src, dst = [0, 3, 2, 1, 0], [2, 1, 1, 2, 4]
    assert brute.hang_roots([0, 1, 2, 3], src, dst) == [1, 2]
    assert brute.hang_roots([0, 3], src, dst) == [0, 3]  # nothing flagged downstream of them
    chain_s, chain_d = [0, 1, 2], [1, 2, 3]
    assert brute.hang_roots([1, 2], chain_s, chain_d) == [2]
    assert brute.hang_roots([1, 2, 3], chain_s, chain_d) == [3]
    assert brute.hang_roots([], chain_s, chain_d) == []


def test_nonempty_hang_mode_matches_brute_force_and_flags_back_pressure():
    """RTM_HANG_NONEMPTY ("any content in a buffer", L229) against brute.py on random tiny traces;
    and on the constructed deadlock it also flags the backed-up components earlier than the full
    criterion does (a non-empty buffer is enough)."""
    for seed in range(30):
        rng = np.random.default_rng(11000 + seed)
        case = random_tiny_case(rng)
        kw = dict(t0=case["t0"], hang_windows=case["H"], k=case["k"], rank_mode=case["mode"], hang_mode=1)
        orc = oracle.Oracle(case["owner"], case["caps"], case["totals"], n_components=case["nc"], **kw)
        br = brute.Brute(case["owner"], case["caps"], case["totals"], case["nc"], **kw)
        for srows, erows, ends in case["calls"]:
            o = orc.reduce(sample_array(srows), event_array(erows), ends, want_all_stats=True)
            _compare(o, br.reduce(srows, erows, ends), case["nb"], case["nk"], case["nc"])
    # one buffer at 1 of 4 (non-empty, not full) in a silent component: window 0 starts empty (the
    # carry-in 0 counts), windows 1 and 2 are non-empty throughout: flagged at window 2 (H = 2)
    orc = oracle.Oracle(np.zeros(1, np.uint32), np.array([4], np.uint16), np.ones(1, np.int64), n_components=1,
                        t0=0, hang_windows=2, k=1, hang_mode=1)
    r = orc.reduce(sample_array([(0, 0, 1, 4)]), event_array([]), [10, 20, 30])
    assert r["hung"][:, 0].tolist() == [0, 0, 1]
    full = oracle.Oracle(np.zeros(1, np.uint32), np.array([4], np.uint16), np.ones(1, np.int64), n_components=1,
                         t0=0, hang_windows=2, k=1, hang_mode=0)
    assert full.reduce(sample_array([(0, 0, 1, 4)]), event_array([]), [10, 20, 30])["hung"].sum() == 0
