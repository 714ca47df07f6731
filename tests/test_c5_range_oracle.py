"""The range-parallel oracle of tools/c5_full.py (prefix replayed as coarse windows, H warm-up
windows, then the range) gives exactly the sequential oracle's per-window results: summaries,
progress rows, sampled top-k and hang lists, final per-buffer table.  CPU only."""
from __future__ import annotations

import os
import sys

import numpy as np

import gen
import oracle

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
import c5_full as T  # noqa: E402


def test_range_parallel_oracle_equals_sequential():
    wl = gen.C5.scaled("C5-mini", n_samples=360_000, n_events=40_000, n_buffers=4096, n_windows=500,
                       hang_windows=6, k=16)
    W, batch = 240, 40
    sampled = [0, 1, 39, 40, 100, 238, 239]
    cps = set(range(batch - 1, W, batch)) | set(sampled) | {W - 1}
    owner, cap, tot = gen.registry(wl)
    orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, t0=wl.t0, hang_windows=wl.hang_windows,
                        k=wl.k)
    s_lo, s_hi, e_lo, e_hi = T.ranges(wl, 0, W)
    ref = orc.reduce(gen.samples(wl, s_lo, s_hi - s_lo), gen.events(wl, e_lo, e_hi - e_lo), wl.t_end(0, W))
    assert ref["rc"] == 0
    assert ref["summary"]["n_hung"].sum() > 0  # the hang-run warm-up is exercised
    prog = {w: ref["progress"][w] for w in cps}
    tops = {w: ref["topk"][w][:ref["topk_n"][w]] for w in sampled}
    hung = {w: np.nonzero(ref["hung"][w])[0].astype(np.uint32) for w in sampled}
    r = T.oracle_pass(wl, W, batch, sampled, cps, ref["summary"], prog, tops, hung, ref["stats"], 3)
    assert r["oracle_ok"], r["mismatches"]
    assert r["summary_windows_checked"] == W and r["topk_windows_checked"] == len(sampled)
    # a corrupted GPU-side value is caught
    bad = ref["summary"].copy()
    bad["digest"][123] ^= 1
    r = T.oracle_pass(wl, W, batch, sampled, cps, bad, prog, tops, hung, ref["stats"], 3)
    assert not r["oracle_ok"] and r["mismatches"][0][:3] == ["summary", "digest", "123"]
