"""CPU oracle for the monitoring-snapshot reduction — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` leg may import this package.  The product package
(``paper_conf_micro_mosallaeii024_b200``) never imports it, and it never imports the product.

``liboracle.so`` is ``oracle/oracle.c`` (plain single-threaded C);
``oracle/brute.py`` is a second, structurally different pure-Python statement of the same
definition used to pin the C oracle on tiny traces.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))

SUMMARY_DTYPE = np.dtype([("t_begin", "<i8"), ("t_end", "<i8"), ("n_samples", "<u8"), ("n_events", "<u8"),
                          ("n_dropped", "<u8"), ("digest", "<u8"), ("n_touched", "<u4"), ("n_hung", "<u4")])
TOPK_DTYPE = np.dtype([("buffer_id", "<u4"), ("level", "<u2"), ("capacity", "<u2")])
PROGRESS_DTYPE = np.dtype([("total", "<i8"), ("started", "<i8"), ("finished", "<i8"), ("in_flight", "<i8"),
                           ("not_started", "<i8")])
BSTAT_DTYPE = np.dtype([("integral", "<i8"), ("last", "<u2"), ("max", "<u2"), ("min", "<u2"), ("capacity", "<u2"),
                        ("n_samples", "<u4"), ("pad", "<u4"), ("mean_occ", "<f8")])
COMP_DTYPE = np.dtype([("started", "<i8"), ("finished", "<i8"), ("in_flight", "<i8")])
assert SUMMARY_DTYPE.itemsize == 56 and BSTAT_DTYPE.itemsize == 32


class _Config(ctypes.Structure):
    _fields_ = [("n_buffers", ctypes.c_uint32), ("n_components", ctypes.c_uint32), ("n_kernels", ctypes.c_uint32),
                ("buffer_owner", ctypes.c_void_p), ("buffer_capacity", ctypes.c_void_p),
                ("kernel_total", ctypes.c_void_p), ("t0", ctypes.c_int64), ("hang_windows", ctypes.c_uint32),
                ("k", ctypes.c_uint32), ("rank_mode", ctypes.c_int32), ("owned", ctypes.c_void_p),
                ("hang_mode", ctypes.c_int32)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        path = os.path.join(HERE, "liboracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `python __graft_entry__.py build`")
        L = ctypes.CDLL(path)
        vp, u32, u64 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64
        L.orc_create.argtypes = [ctypes.POINTER(_Config)]
        L.orc_create.restype = vp
        L.orc_destroy.argtypes = [vp]
        L.orc_reset.argtypes = [vp]
        L.orc_reduce.argtypes = [vp, vp, u64, vp, u64, vp, u32, vp, vp, vp, vp, vp, vp, vp, vp]
        L.orc_reduce.restype = ctypes.c_int
        L.orc_digest_term.argtypes = [u32, ctypes.c_uint16, ctypes.c_uint16, ctypes.c_uint16, ctypes.c_uint16, u32,
                                      ctypes.c_int64]
        L.orc_digest_term.restype = u64
        L.orc_merge_topk.argtypes = [vp, vp, u32, u32, u32, ctypes.c_int32, vp, vp]
        L.orc_merge_topk.restype = ctypes.c_int
        L.orc_persistence.argtypes = [vp, vp]
        L.orc_persistence.restype = None
        L.orc_bar_create.argtypes = [vp, ctypes.c_int64, ctypes.POINTER(u32)]
        L.orc_bar_update.argtypes = [vp, u32, ctypes.c_int64]
        L.orc_bar_destroy.argtypes = [vp, u32]
        for fn in ("orc_bar_create", "orc_bar_update", "orc_bar_destroy"):
            getattr(L, fn).restype = ctypes.c_int
        _lib = L
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data


class Oracle:
    """Stateful oracle context (mirrors rtm_create / rtm_window_reduce semantics)."""

    def __init__(self, owner, capacity, kernel_total, *, n_components=None, t0=0, hang_windows=8, k=16, rank_mode=0,
                 owned=None, hang_mode=0):
        self.owner = np.ascontiguousarray(owner, dtype=np.uint32)
        self.capacity = np.ascontiguousarray(capacity, dtype=np.uint16)
        self.kernel_total = np.ascontiguousarray(kernel_total, dtype=np.int64)
        self.n_buffers = len(self.owner)
        if n_components is None:
            n_components = len(owned) if owned is not None else int(self.owner.max()) + 1
        self.n_components = int(n_components)
        self.n_kernels = len(self.kernel_total)
        self.k = k
        self.owned = None if owned is None else np.ascontiguousarray(owned, dtype=np.uint8)
        cfg = _Config(self.n_buffers, self.n_components, self.n_kernels, _ptr(self.owner), _ptr(self.capacity),
                      _ptr(self.kernel_total), t0, hang_windows, k, rank_mode, _ptr(self.owned), hang_mode)
        self._h = lib().orc_create(ctypes.byref(cfg))
        if not self._h:
            raise ValueError("orc_create rejected the configuration")

    def close(self):
        if self._h:
            lib().orc_destroy(self._h)
            self._h = None

    __del__ = close

    def reset(self):
        lib().orc_reset(self._h)

    def bar_create(self, total):
        i = ctypes.c_uint32()
        if lib().orc_bar_create(self._h, int(total), ctypes.byref(i)) != 0:
            raise ValueError("no free progress bar id")
        return i.value

    def bar_update(self, bar, total):
        if lib().orc_bar_update(self._h, int(bar), int(total)) != 0:
            raise ValueError("progress bar not live")

    def bar_destroy(self, bar):
        if lib().orc_bar_destroy(self._h, int(bar)) != 0:
            raise ValueError("progress bar not live")

    def persistence(self):
        """Per buffer: windows (since create / reset) in which it was in the top-k list."""
        out = np.zeros(self.n_buffers, np.uint32)
        lib().orc_persistence(self._h, out.ctypes.data)
        return out

    def reduce(self, samples, events, t_end, *, want_hung=True, want_all_stats=False, want_topk=True):
        samples = np.ascontiguousarray(samples)
        events = np.ascontiguousarray(events)
        t_end = np.ascontiguousarray(t_end, dtype=np.int64)
        W = len(t_end)
        out = {
            "summary": np.zeros(W, SUMMARY_DTYPE),
            "topk": np.zeros(W * self.k, TOPK_DTYPE).reshape(W, self.k),
            "topk_n": np.zeros(W, np.uint32),
            "progress": np.zeros(W * self.n_kernels, PROGRESS_DTYPE).reshape(W, self.n_kernels),
            "hung": np.zeros((W, self.n_components), np.uint8) if want_hung else None,
            "stats": np.zeros(self.n_buffers, BSTAT_DTYPE),
            "comps": np.zeros(self.n_components, COMP_DTYPE),
            "all_stats": np.zeros((W, self.n_buffers), BSTAT_DTYPE) if want_all_stats else None,
        }
        rc = lib().orc_reduce(self._h, _ptr(samples), len(samples), _ptr(events), len(events), _ptr(t_end), W,
                              _ptr(out["summary"]), _ptr(out["topk"]) if want_topk else None,
                              _ptr(out["topk_n"]) if want_topk else None, _ptr(out["progress"]),
                              _ptr(out["hung"]), _ptr(out["stats"]), _ptr(out["comps"]), _ptr(out["all_stats"]))
        out["rc"] = rc
        return out


def digest_term(b, last, mx, mn, cap, n, integral) -> int:
    return int(lib().orc_digest_term(b, last, mx, mn, cap, n, integral))


def merge_topk(shard_outs, k, rank_mode=0):
    """Whole-trace top-k from per-shard top-k lists."""
    W = len(shard_outs[0]["topk_n"])
    tops = [np.ascontiguousarray(o["topk"]) for o in shard_outs]
    ns = [np.ascontiguousarray(o["topk_n"]) for o in shard_outs]
    tp = (ctypes.c_void_p * len(tops))(*[t.ctypes.data for t in tops])
    npp = (ctypes.c_void_p * len(ns))(*[n.ctypes.data for n in ns])
    out = np.zeros((W, k), TOPK_DTYPE)
    out_n = np.zeros(W, np.uint32)
    lib().orc_merge_topk(tp, npp, len(tops), W, k, rank_mode, out.ctypes.data, out_n.ctypes.data)
    return out, out_n
