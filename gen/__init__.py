"""Seeded synthetic trace generator (input infrastructure shared by tests, oracle harness and bench).

Holds none of the monitored method's arithmetic: only record layouts, the workload
configurations (BASELINE.json configs C1-C5 as restated in SURVEY.md §8(d)) and a ctypes
wrapper over the counter-based generator in ``gen/rtm_gen.h`` (host build ``libgen.so``,
device build ``libgen_cuda.so``).
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))

# 16-byte records (include/rtm.h: rtm_level_sample / rtm_task_event)
SAMPLE_DTYPE = np.dtype([("ts", "<i8"), ("buffer_id", "<u4"), ("level", "<u2"), ("capacity", "<u2")])
EVENT_DTYPE = np.dtype([("ts", "<i8"), ("task_id", "<u4"), ("meta", "<u4")])
assert SAMPLE_DTYPE.itemsize == 16 and EVENT_DTYPE.itemsize == 16

START, END = 0, 1


def pack_meta(comp: int, kernel: int, kind: int) -> int:
    """meta = component (bits 0..19) | kernel (bits 20..30) | kind (bit 31)."""
    return (comp & 0xFFFFF) | ((kernel & 0x7FF) << 20) | ((kind & 1) << 31)


class GenParams(ctypes.Structure):
    _fields_ = [
        ("seed", ctypes.c_uint64),
        ("n_samples", ctypes.c_uint64),
        ("n_events", ctypes.c_uint64),
        ("t0", ctypes.c_int64),
        ("ts_mul_s", ctypes.c_uint64),
        ("ts_mul_e", ctypes.c_uint64),
        ("n_buffers", ctypes.c_uint32),
        ("n_components", ctypes.c_uint32),
        ("n_kernels", ctypes.c_uint32),
        ("buffers_per_comp", ctypes.c_uint32),
        ("lag", ctypes.c_uint32),
        ("tasks_per_kernel", ctypes.c_uint32),
        ("invalid_ppm", ctypes.c_uint32),
        ("shard_world", ctypes.c_uint32),
        ("shard_rank", ctypes.c_uint32),
        ("reserved", ctypes.c_uint32),
    ]


@dataclass
class Workload:
    """One benchmark / parity configuration (BASELINE.json configs)."""

    name: str
    n_samples: int
    n_events: int
    n_buffers: int
    n_kernels: int
    n_windows: int
    k: int
    hang_windows: int
    seed: int
    buffers_per_comp: int = 4
    samples_per_tick: int = 2
    t0: int = 1000
    invalid_ppm: int = 0
    rank_mode: int = 0  # 0 percent, 1 size
    description: str = ""

    @property
    def n_components(self) -> int:
        return (self.n_buffers + self.buffers_per_comp - 1) // self.buffers_per_comp

    @property
    def ticks(self) -> int:
        return max(1, self.n_samples // self.samples_per_tick)

    @property
    def lag(self) -> int:
        return min(4 * self.n_components, max(1, self.n_events // 4))

    @property
    def tasks_per_kernel(self) -> int:
        started = self.lag + max(0, self.n_events - self.lag) // 2 + 1
        # bars are planned 25% larger than the trace covers: not_started stays > 0
        return max(1, -(-(started * 5 // 4) // self.n_kernels))

    def params(self, shard_world: int = 1, shard_rank: int = 0) -> GenParams:
        p = GenParams()
        p.seed = self.seed
        p.n_samples = self.n_samples
        p.n_events = self.n_events
        p.t0 = self.t0
        p.ts_mul_s = (1 << 32) // self.samples_per_tick
        p.ts_mul_e = (self.ticks << 32) // max(1, self.n_events)
        p.n_buffers = self.n_buffers
        p.n_components = self.n_components
        p.n_kernels = self.n_kernels
        p.buffers_per_comp = self.buffers_per_comp
        p.lag = self.lag
        p.tasks_per_kernel = self.tasks_per_kernel
        p.invalid_ppm = self.invalid_ppm
        p.shard_world = shard_world
        p.shard_rank = shard_rank
        return p

    def t_end(self, first: int = 0, count: int | None = None) -> np.ndarray:
        """Window ends: t_end[w] = t0 + (w+1)*T // n_windows (half-open windows)."""
        if count is None:
            count = self.n_windows - first
        w = np.arange(first, first + count, dtype=np.int64)
        return (self.t0 + ((w + 1) * self.ticks) // self.n_windows).astype(np.int64)

    def scaled(self, name: str, **kw) -> "Workload":
        d = dict(self.__dict__)
        d.update(kw)
        d["name"] = name
        return Workload(**d)


# BASELINE.json configs[0..4]; C3-C5 shapes are recorded here for later rounds.
C1 = Workload("C1-tiny", 1_000_000, 100_000, 1000, 4, 10, 16, 8, seed=1,
              description="tiny synthetic trace: 1k buffers, 1M samples + 100k events, 10 windows, k=16")
C1_INVALID = C1.scaled("C1-invalid", invalid_ppm=10_000)
C2 = Workload("C2-1gpu", 90_000_000, 10_000_000, 20480, 8, 1000, 64, 8, seed=2,
              description="MGPUSim-shaped 1-GPU run: ~20k buffers, 100M records, 1k windows, k=64")
C3 = Workload("C3-4gpu", 900_000_000, 100_000_000, 81920, 32, 10000, 64, 16, seed=3,
              description="MGPUSim-shaped 4-GPU run: ~80k buffers, 1B records, 10k windows")
CONFIGS = {w.name: w for w in (C1, C1_INVALID, C2, C3)}


# ---------------------------------------------------------------------------------------
def _load(name: str):
    path = os.path.join(HERE, name)
    if not os.path.exists(path):
        raise RuntimeError(f"{path} missing: run `python __graft_entry__.py build` (or make -C gen)")
    return ctypes.CDLL(path)


_host = None


def host_lib():
    global _host
    if _host is None:
        lib = _load("libgen.so")
        P = ctypes.POINTER(GenParams)
        for fn in ("gen_fill_samples", "gen_fill_events"):
            getattr(lib, fn).argtypes = [P, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p]
            getattr(lib, fn).restype = ctypes.c_uint64
        lib.gen_fill_registry.argtypes = [P, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        lib.gen_fill_registry.restype = None
        lib.gen_splitmix64_c.argtypes = [ctypes.c_uint64]
        lib.gen_splitmix64_c.restype = ctypes.c_uint64
        _host = lib
    return _host


def samples(wl: Workload, start: int = 0, count: int | None = None, shard=(1, 0)) -> np.ndarray:
    if count is None:
        count = wl.n_samples - start
    out = np.empty(count, dtype=SAMPLE_DTYPE)
    p = wl.params(*shard)
    n = host_lib().gen_fill_samples(ctypes.byref(p), start, count, out.ctypes.data)
    return out[:n]


def events(wl: Workload, start: int = 0, count: int | None = None, shard=(1, 0)) -> np.ndarray:
    if count is None:
        count = wl.n_events - start
    out = np.empty(count, dtype=EVENT_DTYPE)
    p = wl.params(*shard)
    n = host_lib().gen_fill_events(ctypes.byref(p), start, count, out.ctypes.data)
    return out[:n]


def registry(wl: Workload):
    """(buffer_owner u32[n_buffers], buffer_capacity u16[n_buffers], kernel_total i64[n_kernels])."""
    owner = np.empty(wl.n_buffers, dtype=np.uint32)
    cap = np.empty(wl.n_buffers, dtype=np.uint16)
    tot = np.empty(wl.n_kernels, dtype=np.int64)
    p = wl.params()
    host_lib().gen_fill_registry(ctypes.byref(p), owner.ctypes.data, cap.ctypes.data, tot.ctypes.data)
    return owner, cap, tot


def splitmix64(x: int) -> int:
    return int(host_lib().gen_splitmix64_c(x))


_dev = None


def device_lib():
    global _dev
    if _dev is None:
        lib = _load("libgen_cuda.so")
        P = ctypes.POINTER(GenParams)
        for fn in ("gen_cuda_fill_samples", "gen_cuda_fill_events", "gen_cuda_flag_samples"):
            getattr(lib, fn).argtypes = [P, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p]
            getattr(lib, fn).restype = ctypes.c_int
        lib.gen_cuda_remap_weak.argtypes = [P, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint64,
                                            ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p]
        lib.gen_cuda_remap_weak.restype = ctypes.c_int
        _dev = lib
    return _dev


def fill_device(kind: str, wl: Workload, ptr: int, start: int, count: int, stream: int = 0) -> None:
    """Write records [start, start+count) of the (unsharded) trace into device memory at ptr."""
    p = wl.params()
    fn = device_lib().gen_cuda_fill_samples if kind == "samples" else device_lib().gen_cuda_fill_events
    err = fn(ctypes.byref(p), start, count, ctypes.c_void_p(ptr), ctypes.c_void_p(stream))
    if err != 0:
        raise RuntimeError(f"gen_cuda fill failed: cudaError {err}")


def remap_weak(wl: Workload, sptr: int, ns: int, eptr: int, ne: int, rank: int, world: int, stream: int = 0) -> None:
    """Map rank `rank`'s local device trace into the id space of a `world`-times larger system."""
    p = wl.params()
    err = device_lib().gen_cuda_remap_weak(ctypes.byref(p), ctypes.c_void_p(sptr), ns, ctypes.c_void_p(eptr), ne,
                                           rank, world, ctypes.c_void_p(stream))
    if err != 0:
        raise RuntimeError(f"gen_cuda_remap_weak failed: cudaError {err}")
