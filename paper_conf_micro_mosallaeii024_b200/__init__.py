"""B200-native monitoring-snapshot reducer (AkitaRTM's dashboard state, §IV-C).

Thin Python binding over the C ABI in ``include/rtm.h`` (``librtm.so``, sm_100a CUDA).  Every
step of the reduction runs in the library's kernels; this module only marshals arguments and
uses PyTorch for device memory, streams and ``torch.distributed`` plumbing.

    mon = Monitor(owner, capacity, kernel_total, n_components=C, t0=0, hang_windows=8, k=64)
    mon.ingest(samples_dev, events_dev)          # torch uint8/structured tensors on cuda, or numpy
    res = mon.window_reduce(t_end)               # per-window summaries, top-k, progress bars
    mon.hang_check(w); mon.buffer_stats(); mon.progress(w, comps=True)
"""
from __future__ import annotations

import ctypes
from collections.abc import Mapping

import numpy as np

from . import _native as N
from ._native import (BSTAT_DTYPE, COMP_DTYPE, EVENT_DTYPE, PROGRESS_DTYPE, RTM_RANK_MEAN, RTM_RANK_PERCENT,
                      RTM_RANK_SIZE,
                      SAMPLE_DTYPE, SUMMARY_DTYPE, TOPK_DTYPE, RTMError)

__all__ = ["Monitor", "RTMError", "SAMPLE_DTYPE", "EVENT_DTYPE", "SUMMARY_DTYPE", "TOPK_DTYPE", "PROGRESS_DTYPE",
           "COMP_DTYPE", "BSTAT_DTYPE", "RTM_RANK_PERCENT", "RTM_RANK_SIZE", "RTM_RANK_MEAN", "version"]

N.lib()  # fail at import time if the native library is missing


def version() -> str:
    return N.lib().rtm_version().decode()


def _records(x, dtype):
    """(pointer, count, mem, keepalive) for a torch tensor (cuda/cpu) or a numpy array of 16-B records."""
    if x is None:
        return None, 0, N.RTM_MEM_DEVICE, None
    if isinstance(x, np.ndarray):
        a = np.ascontiguousarray(x)
        nbytes = a.nbytes
        if nbytes % 16:
            raise ValueError("record arrays must hold whole 16-byte records")
        return a.ctypes.data, nbytes // 16, N.RTM_MEM_HOST, a
    import torch

    if not isinstance(x, torch.Tensor):
        raise TypeError("records must be a numpy array or a torch tensor")
    if not x.is_contiguous():
        raise ValueError("record tensor must be contiguous")
    nbytes = x.numel() * x.element_size()
    if nbytes % 16:
        raise ValueError("record tensors must hold whole 16-byte records")
    mem = N.RTM_MEM_DEVICE if x.is_cuda else N.RTM_MEM_HOST
    return x.data_ptr(), nbytes // 16, mem, x


class Monitor:
    """One reducer context (rtm_create).  Not thread-safe; bound to one device and stream."""

    def __init__(self, buffer_owner, buffer_capacity, kernel_total, *, n_components: int, t0: int = 0,
                 hang_windows: int = 8, k: int = 64, rank_mode: int = RTM_RANK_PERCENT, device: int = 0,
                 rank: int = 0, world: int = 1, owned_components=None, stream=None, process_group=None,
                 buffer_global_id=None, n_global_buffers: int = 0, pack_buffers: int = 0, hang_mode: int = 0):
        import torch

        if not torch.cuda.is_available():
            raise RuntimeError("Monitor needs a CUDA device (sm_100a); there is no CPU fallback")
        self._owner = np.ascontiguousarray(buffer_owner, dtype=np.uint32)
        self._cap = np.ascontiguousarray(buffer_capacity, dtype=np.uint16)
        self._tot = np.ascontiguousarray(kernel_total, dtype=np.int64)
        self._owned = None if owned_components is None else np.ascontiguousarray(owned_components, dtype=np.uint8)
        self.n_buffers, self.n_components, self.n_kernels = len(self._owner), int(n_components), len(self._tot)
        self.k, self.device, self.rank, self.world = int(k), int(device), int(rank), int(world)
        self._pg = process_group
        with torch.cuda.device(device):
            self._stream = stream if stream is not None else torch.cuda.current_stream(device)
        cfg = N.Config()
        cfg.n_buffers, cfg.n_components, cfg.n_kernels = self.n_buffers, self.n_components, self.n_kernels
        cfg.buffer_owner, cfg.buffer_capacity = self._owner.ctypes.data, self._cap.ctypes.data
        cfg.kernel_total = self._tot.ctypes.data
        cfg.t0, cfg.hang_windows, cfg.k, cfg.rank_mode = int(t0), int(hang_windows), self.k, int(rank_mode)
        cfg.device, cfg.rank, cfg.world = self.device, self.rank, self.world
        cfg.owned_components = None if self._owned is None else self._owned.ctypes.data
        cfg.allgather = N.ALLGATHER_FN()  # the binding runs the exchange itself (two-phase API)
        cfg.stream = self._stream.cuda_stream
        # rank-local buffer numbering (include/rtm.h): records carry local ids, results global ids
        self._gid = None if buffer_global_id is None else np.ascontiguousarray(buffer_global_id, dtype=np.uint32)
        cfg.buffer_global_id = None if self._gid is None else self._gid.ctypes.data
        cfg.n_global_buffers = int(n_global_buffers)
        cfg.pack_buffers = int(pack_buffers)
        cfg.hang_mode = int(hang_mode)
        self.n_table = int(n_global_buffers) if self._gid is not None else self.n_buffers
        h = ctypes.c_void_p()
        N.check(N.lib().rtm_create(ctypes.byref(cfg), ctypes.byref(h)), "rtm_create")
        self._h = h
        self._keep = []
        self.W = 0
        self._synced = True
        self._n_hung = np.zeros(0, np.uint32)

    # ------------------------------------------------------------------------------------------
    def close(self):
        if getattr(self, "_h", None):
            N.lib().rtm_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def reset(self):
        N.check(N.lib().rtm_reset(self._h), "rtm_reset")
        self._keep = []

    def ingest(self, samples=None, events=None):
        sp, sn, sm, ska = _records(samples, SAMPLE_DTYPE)
        ep, en, em, eka = _records(events, EVENT_DTYPE)
        if sn and en and sm != em:
            self.ingest(samples, None)
            self.ingest(None, events)
            return
        mem = sm if sn else em
        N.check(N.lib().rtm_ingest(self._h, sp, sn, ep, en, mem), "rtm_ingest")
        self._keep.extend([ska, eka])  # zero-copy device chunks must outlive the next reduce

    def window_reduce(self, t_end):
        """THE hot path: reduce all pending records over len(t_end) windows (blocking)."""
        t_end = np.ascontiguousarray(t_end, dtype=np.int64)
        W = len(t_end)
        summ = np.zeros(W, SUMMARY_DTYPE)
        if self.world > 1:
            self._reduce_distributed(t_end, summ)
            self._synced = False
        else:
            N.check(N.lib().rtm_window_reduce(self._h, t_end.ctypes.data, W, summ.ctypes.data), "rtm_window_reduce")
        self._keep = []
        self.W = W
        return LazyResults(self, W, summ)

    def results(self, W=None):
        """All per-window results of the last batch (one rtm_window_results call)."""
        W = self.W if W is None else W
        summ = np.zeros(W, SUMMARY_DTYPE)
        topk = np.zeros((W, self.k), TOPK_DTYPE)
        topk_n = np.zeros(W, np.uint32)
        bars = np.zeros((W, self.n_kernels), PROGRESS_DTYPE)
        N.check(N.lib().rtm_window_results(self._h, 0, W, summ.ctypes.data, topk.ctypes.data, topk_n.ctypes.data,
                                           bars.ctypes.data), "rtm_window_results")
        return {"summary": summ, "topk": topk, "topk_n": topk_n, "progress": bars}

    def _reduce_distributed(self, t_end, summ):
        """world > 1: local reduce -> all-gather of the packed per-window results -> merge kernels."""
        import torch

        from .dist import allgather_packs

        pack = ctypes.c_void_p()
        nbytes = ctypes.c_uint64()
        N.check(N.lib().rtm_window_reduce_local(self._h, t_end.ctypes.data, len(t_end), ctypes.byref(pack),
                                                ctypes.byref(nbytes)), "rtm_window_reduce_local")
        recv = self._exchange(pack.value, int(nbytes.value))
        N.check(N.lib().rtm_merge(self._h, recv.data_ptr(), self.world, summ.ctypes.data), "rtm_merge")

    def _exchange(self, ptr: int, n: int):
        """All-gather a library pack (device, complete in the Monitor stream's order).  NCCL: the
        copy, the collective and the library's next kernels are ordered on that stream - no host
        synchronisation; gloo stages through host memory (synchronous)."""
        import torch

        from .dist import allgather_packs

        dev = torch.device("cuda", self.device)
        with torch.cuda.stream(self._stream):
            send = torch.empty(n, dtype=torch.uint8, device=dev)
            _copy_from_ptr(send, ptr, n)
            recv = allgather_packs(send, self.world, self._pg)
        return recv

    def sync_tables(self):
        """world > 1: exchange the last call's per-buffer table, per-component totals and hang
        lists (collective: every rank calls it after the same reduce).  The accessors that need
        them call it on first use after a reduce."""
        if self.world <= 1 or self._synced:
            return
        pack = ctypes.c_void_p()
        nbytes = ctypes.c_uint64()
        N.check(N.lib().rtm_tables_local(self._h, ctypes.byref(pack), ctypes.byref(nbytes)), "rtm_tables_local")
        recv = self._exchange(pack.value, int(nbytes.value))
        N.check(N.lib().rtm_tables_merge(self._h, recv.data_ptr(), self.world), "rtm_tables_merge")
        self._synced = True

    def _n_hung_at(self, window: int) -> int:
        """Merged flagged count of `window` of the last batch (identical on every rank)."""
        out = np.zeros(1, SUMMARY_DTYPE)
        N.check(N.lib().rtm_window_results(self._h, window, 1, out.ctypes.data, None, None, None),
                "rtm_window_results")
        return int(out["n_hung"][0])

    def topk(self, window: int):
        out = np.zeros(self.k, TOPK_DTYPE)
        n = ctypes.c_uint32()
        N.check(N.lib().rtm_topk_buffers(self._h, window, out.ctypes.data, ctypes.byref(n)), "rtm_topk_buffers")
        return out[: n.value]

    def progress(self, window: int, comps: bool = False):
        bars = np.zeros(self.n_kernels, PROGRESS_DTYPE)
        if comps:
            self.sync_tables()
        cs = np.zeros(self.n_components, COMP_DTYPE) if comps else None
        N.check(N.lib().rtm_progress(self._h, window, bars.ctypes.data, None if cs is None else cs.ctypes.data),
                "rtm_progress")
        return (bars, cs) if comps else bars

    def hang_check(self, window: int):
        if self.world > 1 and self._n_hung_at(window):
            self.sync_tables()
        n = ctypes.c_uint32()
        N.check(N.lib().rtm_hang_check(self._h, window, None, 0, ctypes.byref(n)), "rtm_hang_check")
        ids = np.zeros(max(1, n.value), np.uint32)
        N.check(N.lib().rtm_hang_check(self._h, window, ids.ctypes.data, len(ids), ctypes.byref(n)),
                "rtm_hang_check")
        return ids[: n.value]

    def set_links(self, src, dst):
        """Component connection graph (component src[i] sends to dst[i]) for hang_roots."""
        a = np.ascontiguousarray(src, dtype=np.uint32)
        b = np.ascontiguousarray(dst, dtype=np.uint32)
        if a.shape != b.shape:
            raise ValueError("src and dst must have the same length")
        N.check(N.lib().rtm_set_links(self._h, a.ctypes.data if len(a) else None, b.ctypes.data if len(b) else None,
                                      len(a)), "rtm_set_links")

    def hang_roots(self, window: int):
        """Root causes among the window's flagged components (sink SCCs of the flagged links)."""
        if self.world > 1 and self._n_hung_at(window):
            self.sync_tables()
        cap = self.n_components
        out = np.zeros(max(1, cap), np.uint32)
        n = ctypes.c_uint32()
        N.check(N.lib().rtm_hang_roots(self._h, window, out.ctypes.data, cap, ctypes.byref(n)), "rtm_hang_roots")
        return out[: n.value].copy()

    def buffer_stats(self, first: int = 0, count: int | None = None):
        if count is None:
            count = self.n_table - first  # global ids with a rank-local numbering
        self.sync_tables()
        out = np.zeros(count, BSTAT_DTYPE)
        N.check(N.lib().rtm_buffer_stats(self._h, first, count, out.ctypes.data), "rtm_buffer_stats")
        return out

    # progress bar registry (Create / Update / DestroyProgressBar)
    def bar_create(self, total: int) -> int:
        i = ctypes.c_uint32()
        N.check(N.lib().rtm_bar_create(self._h, int(total), ctypes.byref(i)), "rtm_bar_create")
        return i.value

    def bar_update(self, bar: int, total: int) -> None:
        N.check(N.lib().rtm_bar_update(self._h, int(bar), int(total)), "rtm_bar_update")

    def bar_destroy(self, bar: int) -> None:
        N.check(N.lib().rtm_bar_destroy(self._h, int(bar)), "rtm_bar_destroy")

    def topk_persistence(self, first: int = 0, count: int | None = None):
        """Windows-in-top-k counter per buffer since create / reset (persistence, L173, L197-L199)."""
        if count is None:
            count = self.n_table - first
        out = np.zeros(count, np.uint32)
        N.check(N.lib().rtm_topk_persistence(self._h, first, count, out.ctypes.data), "rtm_topk_persistence")
        return out

    def watch(self, buffer_ids):
        """Value monitor: watch up to 5 buffers; clears the rings."""
        ids = np.ascontiguousarray(buffer_ids, dtype=np.uint32)
        N.check(N.lib().rtm_watch(self._h, ids.ctypes.data if len(ids) else None, len(ids)), "rtm_watch")

    def watch_series(self, slot: int):
        """Points of watched slot `slot` (last <= 300 windows, oldest first): t_end + window stats."""
        out = np.zeros(N.RTM_WATCH_POINTS, N.WATCH_DTYPE)
        n = ctypes.c_uint32()
        N.check(N.lib().rtm_watch_series(self._h, slot, out.ctypes.data, ctypes.byref(n)), "rtm_watch_series")
        return out[: n.value]

    def use_graphs(self, mode: int = N.RTM_GRAPHS_AUTO):
        """Launch mechanism of window_reduce (include/rtm.h rtm_use_graphs): RTM_GRAPHS_OFF direct
        launches, RTM_GRAPHS_AUTO CUDA-graph replay for calls of <= 64 windows (default),
        RTM_GRAPHS_ALWAYS for every call.  Results are identical."""
        N.check(N.lib().rtm_use_graphs(self._h, int(mode)), "rtm_use_graphs")

    def graph_stats(self):
        """(calls launched from a newly captured CUDA graph, calls that replayed a cached one)."""
        a, b = ctypes.c_uint64(), ctypes.c_uint64()
        N.check(N.lib().rtm_graph_stats(self._h, ctypes.byref(a), ctypes.byref(b)), "rtm_graph_stats")
        return int(a.value), int(b.value)

    def profile(self, enable: bool = True):
        N.check(N.lib().rtm_profile(self._h, 1 if enable else 0), "rtm_profile")

    def profile_read(self):
        arr = (N.KernelTime * 32)()
        n = ctypes.c_uint32()
        N.check(N.lib().rtm_profile_read(self._h, arr, 32, ctypes.byref(n)), "rtm_profile_read")
        return {arr[i].name.decode(): dict(launches=arr[i].launches, total_ms=arr[i].total_ms,
                                           algo_bytes=arr[i].algo_bytes) for i in range(min(n.value, 32))}


_cudart = None


class LazyResults(Mapping):
    """The mapping Monitor.window_reduce returns: "summary" is filled by the call itself; the
    other per-window arrays ("topk", "topk_n", "progress") are copied out of the library on first
    access (one rtm_window_results call), so a caller that only needs the summaries pays no host
    copy of the top-k / progress tables.  Valid until the next window_reduce."""

    _KEYS = ("summary", "topk", "topk_n", "progress")

    def __init__(self, mon, W, summary):
        self._mon, self._W = mon, W
        self._d = {"summary": summary}

    def __getitem__(self, key):
        if key not in self._KEYS:
            raise KeyError(key)
        if key not in self._d:
            self._d.update(self._mon.results(self._W))
        return self._d[key]

    def __iter__(self):
        return iter(self._KEYS)

    def __len__(self):
        return len(self._KEYS)


def _copy_from_ptr(dst_tensor, src_ptr: int, nbytes: int):
    """Device-to-device copy from a raw library pointer into a torch tensor (exchange plumbing)."""
    global _cudart
    import torch

    if _cudart is None:
        _cudart = ctypes.CDLL("libcudart.so.12") if _try("libcudart.so.12") else ctypes.CDLL("libcudart.so")
        _cudart.cudaMemcpyAsync.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int,
                                            ctypes.c_void_p]
        _cudart.cudaMemcpyAsync.restype = ctypes.c_int
    st = torch.cuda.current_stream(dst_tensor.device)
    err = _cudart.cudaMemcpyAsync(dst_tensor.data_ptr(), src_ptr, nbytes, 3, st.cuda_stream)
    if err != 0:
        raise RuntimeError(f"cudaMemcpyAsync failed: {err}")


def _try(name):
    try:
        ctypes.CDLL(name)
        return True
    except OSError:
        return False
