"""ctypes declarations for librtm.so (include/rtm.h).  Argument marshalling only.

The library is built in-tree (``python __graft_entry__.py build``); importing this module
fails loudly if it is missing — there is no CPU fallback for the reduction.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("RTM_LIB_PATH") or os.path.join(HERE, "librtm.so")  # override: profiling builds

RTM_OK, RTM_E_INVALID, RTM_E_CUDA, RTM_E_COMM, RTM_E_ORDER, RTM_E_TOO_SMALL, RTM_E_STATE, RTM_E_NOMEM = (
    0, -1, -2, -3, -4, -5, -6, -7)
RTM_MEM_HOST, RTM_MEM_DEVICE = 0, 1
RTM_RANK_PERCENT, RTM_RANK_SIZE, RTM_RANK_MEAN = 0, 1, 2
RTM_GRAPHS_OFF, RTM_GRAPHS_AUTO, RTM_GRAPHS_ALWAYS = 0, 1, 2

# record and result layouts (include/rtm.h)
SAMPLE_DTYPE = np.dtype([("ts", "<i8"), ("buffer_id", "<u4"), ("level", "<u2"), ("capacity", "<u2")])
EVENT_DTYPE = np.dtype([("ts", "<i8"), ("task_id", "<u4"), ("meta", "<u4")])
SUMMARY_DTYPE = np.dtype([("t_begin", "<i8"), ("t_end", "<i8"), ("n_samples", "<u8"), ("n_events", "<u8"),
                          ("n_dropped", "<u8"), ("digest", "<u8"), ("n_touched", "<u4"), ("n_hung", "<u4")])
TOPK_DTYPE = np.dtype([("buffer_id", "<u4"), ("level", "<u2"), ("capacity", "<u2")])
PROGRESS_DTYPE = np.dtype([("total", "<i8"), ("started", "<i8"), ("finished", "<i8"), ("in_flight", "<i8"),
                           ("not_started", "<i8")])
COMP_DTYPE = np.dtype([("started", "<i8"), ("finished", "<i8"), ("in_flight", "<i8")])
BSTAT_DTYPE = np.dtype([("integral", "<i8"), ("last", "<u2"), ("max", "<u2"), ("min", "<u2"), ("capacity", "<u2"),
                        ("n_samples", "<u4"), ("reserved", "<u4"), ("mean_occ", "<f8")])

WATCH_DTYPE = np.dtype([("t_end", "<i8"), ("integral", "<i8"), ("last", "<u2"), ("max", "<u2"), ("min", "<u2"),
                        ("capacity", "<u2"), ("n_samples", "<u4"), ("reserved", "<u4"), ("mean_occ", "<f8")])
assert WATCH_DTYPE.itemsize == 40
RTM_WATCH_MAX, RTM_WATCH_POINTS = 5, 300

ALLGATHER_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64)


class Config(ctypes.Structure):
    _fields_ = [
        ("n_buffers", ctypes.c_uint32), ("n_components", ctypes.c_uint32), ("n_kernels", ctypes.c_uint32),
        ("buffer_owner", ctypes.c_void_p), ("buffer_capacity", ctypes.c_void_p), ("kernel_total", ctypes.c_void_p),
        ("t0", ctypes.c_int64), ("hang_windows", ctypes.c_uint32), ("k", ctypes.c_uint32),
        ("rank_mode", ctypes.c_int32), ("device", ctypes.c_int32), ("rank", ctypes.c_int32),
        ("world", ctypes.c_int32), ("owned_components", ctypes.c_void_p), ("allgather", ALLGATHER_FN),
        ("allgather_user", ctypes.c_void_p), ("stream", ctypes.c_void_p),
        ("buffer_global_id", ctypes.c_void_p), ("n_global_buffers", ctypes.c_uint32),
        ("pack_buffers", ctypes.c_uint32), ("hang_mode", ctypes.c_int32),
        ("allgather_on_stream", ctypes.c_int32),
    ]


class KernelTime(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char_p), ("launches", ctypes.c_uint32), ("total_ms", ctypes.c_double),
                ("algo_bytes", ctypes.c_uint64)]


# every symbol include/rtm.h declares (checked by tests/test_abi.py)
EXPORTS = ("rtm_create", "rtm_destroy", "rtm_reset", "rtm_ingest", "rtm_window_reduce", "rtm_topk_buffers",
           "rtm_progress", "rtm_hang_check", "rtm_buffer_stats", "rtm_window_results", "rtm_window_reduce_local",
           "rtm_merge", "rtm_profile", "rtm_profile_read", "rtm_status_str", "rtm_version",
           "rtm_kernel_launches", "rtm_watch", "rtm_watch_series", "rtm_topk_persistence",
           "rtm_bar_create", "rtm_bar_update", "rtm_bar_destroy", "rtm_set_links", "rtm_hang_roots",
           "rtm_exchange_bytes", "rtm_sync_tables", "rtm_tables_local", "rtm_tables_merge", "rtm_use_graphs",
           "rtm_graph_stats")

_lib = None


def lib():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: build it with `python __graft_entry__.py build` "
                           "(the window-snapshot reduction has no CPU fallback)")
    L = ctypes.CDLL(LIB_PATH)
    vp, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int32
    P = ctypes.POINTER
    L.rtm_create.argtypes = [P(Config), P(vp)]
    L.rtm_destroy.argtypes = [vp]
    L.rtm_destroy.restype = None
    L.rtm_reset.argtypes = [vp]
    L.rtm_ingest.argtypes = [vp, vp, u64, vp, u64, i32]
    L.rtm_window_reduce.argtypes = [vp, vp, u32, vp]
    L.rtm_topk_buffers.argtypes = [vp, u32, vp, P(u32)]
    L.rtm_progress.argtypes = [vp, u32, vp, vp]
    L.rtm_hang_check.argtypes = [vp, u32, vp, u32, P(u32)]
    L.rtm_buffer_stats.argtypes = [vp, u32, u32, vp]
    L.rtm_window_results.argtypes = [vp, u32, u32, vp, vp, vp, vp]
    L.rtm_window_reduce_local.argtypes = [vp, vp, u32, P(vp), P(u64)]
    L.rtm_merge.argtypes = [vp, vp, u32, vp]
    L.rtm_profile.argtypes = [vp, i32]
    L.rtm_profile_read.argtypes = [vp, vp, u32, P(u32)]
    L.rtm_watch.argtypes = [vp, vp, u32]
    L.rtm_topk_persistence.argtypes = [vp, u32, u32, vp]
    L.rtm_bar_create.argtypes = [vp, ctypes.c_int64, P(u32)]
    L.rtm_bar_update.argtypes = [vp, u32, ctypes.c_int64]
    L.rtm_bar_destroy.argtypes = [vp, u32]
    L.rtm_set_links.argtypes = [vp, vp, vp, u32]
    L.rtm_hang_roots.argtypes = [vp, u32, vp, u32, P(u32)]
    L.rtm_watch_series.argtypes = [vp, u32, vp, P(u32)]
    L.rtm_sync_tables.argtypes = [vp]
    L.rtm_tables_local.argtypes = [vp, P(vp), P(u64)]
    L.rtm_tables_merge.argtypes = [vp, vp, u32]
    L.rtm_use_graphs.argtypes = [vp, i32]
    L.rtm_graph_stats.argtypes = [vp, P(u64), P(u64)]
    for fn in ("rtm_watch", "rtm_watch_series", "rtm_topk_persistence", "rtm_bar_create", "rtm_bar_update",
               "rtm_bar_destroy", "rtm_set_links", "rtm_hang_roots", "rtm_create", "rtm_reset", "rtm_ingest", "rtm_window_reduce", "rtm_topk_buffers", "rtm_progress",
               "rtm_hang_check", "rtm_buffer_stats", "rtm_window_reduce_local", "rtm_merge", "rtm_profile",
               "rtm_profile_read", "rtm_window_results", "rtm_sync_tables", "rtm_tables_local", "rtm_tables_merge",
               "rtm_use_graphs", "rtm_graph_stats"):
        getattr(L, fn).restype = ctypes.c_int
    L.rtm_status_str.argtypes = [ctypes.c_int]
    L.rtm_status_str.restype = ctypes.c_char_p
    L.rtm_version.argtypes = []
    L.rtm_version.restype = ctypes.c_char_p
    L.rtm_kernel_launches.argtypes = []
    L.rtm_kernel_launches.restype = ctypes.c_uint64
    L.rtm_exchange_bytes.argtypes = [u32, u32, u32, i32]
    L.rtm_exchange_bytes.restype = ctypes.c_uint64
    _lib = L
    return L


class RTMError(RuntimeError):
    def __init__(self, code: int, where: str):
        self.code = code
        msg = lib().rtm_status_str(code).decode()
        super().__init__(f"{where}: {msg} ({code})")


def check(code: int, where: str) -> None:
    if code != RTM_OK:
        raise RTMError(code, where)
