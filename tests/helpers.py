"""Shared test helpers: tiny hand-built traces and comparisons (no method arithmetic here)."""
from __future__ import annotations

import numpy as np

from gen import EVENT_DTYPE, SAMPLE_DTYPE, pack_meta  # noqa: F401


def sample_array(rows):
    a = np.zeros(len(rows), SAMPLE_DTYPE)
    for i, (ts, b, lvl, cap) in enumerate(rows):
        a[i] = (ts, b, lvl, cap)
    return a


def event_array(rows):
    a = np.zeros(len(rows), EVENT_DTYPE)
    for i, (ts, task, meta) in enumerate(rows):
        a[i] = (ts, task, meta)
    return a


def random_tiny_case(rng, *, allow_disorder=False):
    """A small random trace exercising ties, carry-in, drops, zero-length windows."""
    nb = int(rng.integers(1, 7))
    nc = int(rng.integers(1, 4))
    nk = int(rng.integers(1, 4))
    caps = rng.choice([1, 2, 3, 4, 8], size=nb).astype(np.uint16)
    owner = rng.integers(0, nc, size=nb).astype(np.uint32)
    totals = rng.integers(0, 12, size=nk).astype(np.int64)
    t0 = int(rng.integers(-20, 20))
    calls = []
    t = t0
    for _ in range(int(rng.integers(1, 4))):
        W = int(rng.integers(1, 5))
        ends = []
        cur = t
        for _w in range(W):
            cur += int(rng.choice([0, 1, 3, 7, 12]))
            ends.append(cur)
        lo, hi = t - 5, ends[-1] + 5
        ns = int(rng.integers(0, 30))
        ts = np.sort(rng.integers(lo, hi + 1, size=ns))
        srows = []
        for x in ts:
            b = int(rng.integers(0, nb))
            cap = int(caps[b])
            lvl = int(rng.integers(0, cap + 1))
            r = [int(x), b, lvl, cap]
            u = rng.random()
            if u < 0.06:
                r[1] = nb + int(rng.integers(0, 3))
                r[0] = int(rng.integers(lo - 10, hi + 10))  # invalid: ts unconstrained
            elif u < 0.10:
                r[2] = cap + 1
                r[0] = int(rng.integers(lo - 10, hi + 10))
            elif u < 0.13:
                r[3] = cap + 1
            srows.append(tuple(r))
        ne = int(rng.integers(0, 15))
        ets = np.sort(rng.integers(lo, hi + 1, size=ne))
        erows = []
        for x in ets:
            c = int(rng.integers(0, nc))
            k = int(rng.integers(0, nk))
            kind = int(rng.integers(0, 2))
            if rng.random() < 0.08:
                c = nc + 1
            erows.append((int(x), int(rng.integers(0, 100)), pack_meta(c, k, kind)))
        if allow_disorder and len(srows) > 2 and rng.random() < 0.5:
            i = int(rng.integers(0, len(srows) - 1))
            srows[i], srows[i + 1] = srows[i + 1], srows[i]
        calls.append((srows, erows, ends))
        t = ends[-1]
    return dict(nb=nb, nc=nc, nk=nk, caps=caps, owner=owner, totals=totals, t0=t0,
                H=int(rng.integers(1, 3)), k=int(rng.integers(1, nb + 2)), mode=int(rng.integers(0, 2)), calls=calls)
