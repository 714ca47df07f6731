"""Brute-force statement of the window snapshot (TEST INFRASTRUCTURE ONLY, tiny traces).

A second, structurally different reading of DESIGN.md §2 used to pin ``oracle.c``:
  - the occupancy integral is a literal tick loop  sum_{t=t_prev}^{t_end-1} L(t),  where L(t)
    is the level of the latest kept sample (ingest order) with ts <= t, else the carry-in
    ("fullness of a buffer over time");
  - the Bottleneck Analyzer list is a full ``sorted`` with exact ``fractions.Fraction``
    fullness keys (Fig. 3);
  - drop attribution searches forward for the next field-valid record;
  - the ts-order contract is checked over all pairs;
  - the digest mixer is re-typed from the specification in pure Python integers.
Pure-Python loops: only for traces of a few hundred records and ticks.
"""
from __future__ import annotations

from fractions import Fraction

M64 = (1 << 64) - 1


def fmix64(z: int) -> int:
    z &= M64
    z ^= z >> 30
    z = (z * 0xBF58476D1CE4E5B9) & M64
    z ^= z >> 27
    z = (z * 0x94D049BB133111EB) & M64
    z ^= z >> 31
    return z


def digest_term(b, last, mx, mn, cap, n, integral) -> int:
    levels = last | (mx << 16) | (mn << 32) | (cap << 48)
    ident = (n << 32) | b
    x = ((integral & M64) * 0x9E3779B97F4A7C15) & M64
    x ^= (ident * 0xC2B2AE3D27D4EB4F) & M64
    x ^= (levels * 0x165667B19E3779F9) & M64
    return fmix64(x)


class OrderError(Exception):
    pass


class Brute:
    def __init__(self, owner, capacity, kernel_total, n_components, *, t0=0, hang_windows=8, k=16, rank_mode=0,
                 owned=None, hang_mode=0):
        self.owner = [int(x) for x in owner]
        self.cap = [int(x) for x in capacity]
        self.total = [int(x) for x in kernel_total]
        self.nb, self.nc, self.nk = len(self.owner), int(n_components), len(self.total)
        self.H, self.k, self.mode, self.hang_mode = hang_windows, k, rank_mode, hang_mode
        self.owned = [1] * self.nc if owned is None else [int(x) for x in owned]
        self.t_prev = t0
        self.lvl = [0] * self.nb
        self.cs, self.ce = [0] * self.nc, [0] * self.nc
        self.ks, self.ke = [0] * self.nk, [0] * self.nk
        self.run = [0] * self.nc
        self.live = [1] * self.nk

    # progress bar registry (Create / Update / DestroyProgressBar)
    def bar_create(self, total):
        k = self.live.index(0)  # lowest free id (ValueError if none)
        self.live[k], self.total[k], self.ks[k], self.ke[k] = 1, int(total), 0, 0
        return k

    def bar_update(self, k, total):
        if not self.live[k]:
            raise ValueError("not live")
        self.total[k] = int(total)

    def bar_destroy(self, k):
        if not self.live[k]:
            raise ValueError("not live")
        self.live[k] = 0

    # field validity (DESIGN.md §2 "ingest")
    def _sample_valid(self, r):
        ts, b, lvl, cap = r
        return b < self.nb and cap == self.cap[b] and lvl <= cap

    def _event_valid(self, r):
        ts, task, meta = r
        kern = (meta >> 20) & 0x7FF
        return (meta & 0xFFFFF) < self.nc and kern < self.nk and self.live[kern] == 1

    def reduce(self, samples, events, t_end):
        """samples: list of (ts, buffer_id, level, capacity); events: list of (ts, task_id, meta)."""
        t_end = [int(x) for x in t_end]
        W = len(t_end)
        t_begin = self.t_prev
        bounds = [t_begin] + t_end

        def window_of(ts):
            for w in range(W):
                if bounds[w] <= ts < bounds[w + 1]:
                    return w
            return None

        def classify(recs, valid_fn):
            valid = [valid_fn(r) for r in recs]
            vts = [r[0] for r, v in zip(recs, valid) if v]
            for i in range(len(vts)):
                for j in range(i + 1, len(vts)):
                    if vts[j] < vts[i]:
                        raise OrderError()
            kept = [[] for _ in range(W)]
            dropped = [0] * W
            for i, r in enumerate(recs):
                if valid[i]:
                    ts = r[0]
                    if ts < t_begin:
                        dropped[0] += 1
                    elif ts >= t_end[-1]:
                        dropped[W - 1] += 1
                    else:
                        kept[window_of(ts)].append(r)
                else:
                    charge = W - 1
                    for j in range(i + 1, len(recs)):
                        if valid[j]:
                            ts = recs[j][0]
                            charge = 0 if ts < t_begin else (W - 1 if ts >= t_end[-1] else window_of(ts))
                            break
                    dropped[charge] += 1
            return kept, dropped

        skept, sdrop = classify(samples, self._sample_valid)
        ekept, edrop = classify(events, self._event_valid)

        out = []
        for w in range(W):
            tp, te = bounds[w], bounds[w + 1]
            ks = skept[w]
            stats = []
            digest, touched = 0, 0
            for b in range(self.nb):
                mine = [r for r in ks if r[1] == b]
                lin = self.lvl[b]
                integral = 0
                for t in range(tp, te):
                    level = lin
                    for r in mine:
                        if r[0] <= t:
                            level = r[2]
                    integral += level
                levels = [lin] + [r[2] for r in mine]
                last = mine[-1][2] if mine else lin
                st = dict(integral=integral, last=last, max=max(levels), min=min(levels), capacity=self.cap[b],
                          n_samples=len(mine),
                          mean_occ=(integral / (self.cap[b] * (te - tp)) if te > tp else 0.0))
                stats.append(st)
                if mine:
                    touched += 1
                    digest = (digest + digest_term(b, last, st["max"], st["min"], self.cap[b], len(mine),
                                                   integral)) & M64
            for b in range(self.nb):
                self.lvl[b] = stats[b]["last"]
            active = [0] * self.nc
            for ts, task, meta in ekept[w]:
                c, kk, kind = meta & 0xFFFFF, (meta >> 20) & 0x7FF, meta >> 31
                if kind == 0:
                    self.cs[c] += 1
                    self.ks[kk] += 1
                else:
                    self.ce[c] += 1
                    self.ke[kk] += 1
                active[c] = 1
            progress = [dict(total=self.total[k], started=self.ks[k], finished=self.ke[k],
                             in_flight=self.ks[k] - self.ke[k], not_started=self.total[k] - self.ks[k])
                        if self.live[k] else dict(total=0, started=0, finished=0, in_flight=0, not_started=0)
                        for k in range(self.nk)]
            elig = [b for b in range(self.nb) if self.owned[self.owner[b]]]
            if self.mode == 0:
                order = sorted(elig, key=lambda b: (-Fraction(self.lvl[b], self.cap[b]), b))
            elif self.mode == 2:  # the window's mean occupancy: tick-loop integral / (cap * W)
                order = sorted(elig, key=lambda b: (-(Fraction(stats[b]["integral"], self.cap[b] * (te - tp))
                                                      if te > tp else Fraction(0)), b))
            else:
                order = sorted(elig, key=lambda b: (-self.lvl[b], b))
            top = [(b, self.lvl[b], self.cap[b]) for b in order[: self.k]]
            hung = []
            for c in range(self.nc):
                held = (lambda b: stats[b]["min"] >= 1) if self.hang_mode == 1 else \
                    (lambda b: stats[b]["min"] == self.cap[b])
                anyfull = any(held(b) for b in range(self.nb) if self.owner[b] == c)
                cond = anyfull and not active[c]
                self.run[c] = self.run[c] + 1 if cond else 0
                if self.run[c] >= self.H:
                    hung.append(c)
            out.append(dict(t_begin=tp, t_end=te, n_samples=len(ks), n_events=len(ekept[w]),
                            n_dropped=sdrop[w] + edrop[w], digest=digest, n_touched=touched, n_hung=len(hung),
                            topk=top, progress=progress, hung=hung, stats=stats))
        self.t_prev = t_end[-1]
        return out


def hang_roots(flagged, src, dst):
    """Root causes among hang-flagged components:
    with the links restricted to flagged components ("c sends to d"), c is a root iff every
    flagged component reachable from c can reach c back (c lies in a sink strongly-connected
    component: a circular wait, or a stuck component with no flagged successor).  Brute-force
    reachability, ascending ids."""
    F = set(int(x) for x in flagged)
    succ = {c: [] for c in F}
    for a, b in zip(src, dst):
        a, b = int(a), int(b)
        if a in F and b in F:
            succ[a].append(b)

    def reach(c):
        seen, todo = {c}, [c]
        while todo:
            x = todo.pop()
            for y in succ[x]:
                if y not in seen:
                    seen.add(y)
                    todo.append(y)
        return seen

    R = {c: reach(c) for c in F}
    return sorted(c for c in F if all(c in R[d] for d in R[c]))
