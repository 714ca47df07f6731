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
        ("zipf_n", ctypes.c_uint32),
        ("zipf_cdf", ctypes.c_uint64),
        ("zipf_a", ctypes.c_uint32),
        ("zipf_b", ctypes.c_uint32),
        ("dl_fill_ts", ctypes.c_int64 * 2),
        ("dl_quiet_ts", ctypes.c_int64 * 2),
        ("dl_comp", ctypes.c_uint32 * 4),
        ("dl_sink", ctypes.c_uint32),
        ("n_dl_stages", ctypes.c_uint32),
    ]


assert ctypes.sizeof(GenParams) == 160


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
    # C4: Zipf exponent over buffer ranks (0 = uniform ids); ranks scattered by an affine map
    zipf_s: float = 0.0
    zipf_a: int = 0x9E3779B1 % (1 << 20) | 1
    zipf_b: int = 12345
    # C3: injected circular wait, per stage (window where the components go quiet, components);
    # their buffers are held full from `deadlock_lead` windows earlier
    deadlock: tuple = ()
    deadlock_lead: int = 3

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
        if self.zipf_s > 0:
            import math
            a = self.zipf_a % self.n_buffers or 1
            while math.gcd(a, self.n_buffers) != 1:  # bijection on [0, n)
                a += 1
            p.zipf_n = self.n_buffers
            p.zipf_a = a
            p.zipf_b = self.zipf_b % self.n_buffers
        if self.deadlock:
            assert len(self.deadlock) <= 2
            p.n_dl_stages = len(self.deadlock)
            p.dl_sink = self.n_components - 1
            for s, (w_d, comps) in enumerate(self.deadlock):
                p.dl_quiet_ts[s] = self.t_begin(w_d)
                p.dl_fill_ts[s] = self.t_begin(max(0, w_d - self.deadlock_lead))
                p.dl_comp[2 * s] = comps[0]
                p.dl_comp[2 * s + 1] = comps[1]
        return p

    def t_begin(self, w: int) -> int:
        """Begin of window w (= end of window w-1; t0 for w = 0)."""
        return self.t0 + (w * self.ticks) // self.n_windows

    def index_at(self, kind: str, T: int) -> int:
        """First stream index whose ts >= T (ts_i = t0 + (i * mul) >> 32 is non-decreasing)."""
        p = self.params()
        mul = p.ts_mul_s if kind == "samples" else p.ts_mul_e
        n = self.n_samples if kind == "samples" else self.n_events
        d = T - self.t0
        if d <= 0:
            return 0
        return min(n, -(-(d << 32) // mul))

    def zipf_table(self) -> np.ndarray:
        """u64 inverse-CDF thresholds of Zipf(s) over ranks 0..n-1 (P(rank r) ~ (r+1)^-s): a draw
        u < 2^64 maps to the first r with u < cdf[r].  Built once on the host in fp64 (input data,
        identical for the host and device generators); last entry 2^64-1."""
        n = self.n_buffers
        w = np.arange(1, n + 1, dtype=np.float64) ** (-self.zipf_s)
        c = np.cumsum(w)
        c /= c[-1]
        t = np.minimum(np.floor(c * 2.0**64), 2.0**64 - 2048).astype(np.uint64)
        t = np.maximum.accumulate(t)
        t[-1] = np.uint64(0xFFFFFFFFFFFFFFFF)
        return t

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
# C3: 4 simulated GPUs x 20480 components; the injected circular wait sits on simulated GPU 2
# (components 10240..15359): an "L2 local storage" / "L2 write buffer" pair goes quiet at window
# 6000 and the upstream L1 / DRAM-controller pair it backs up at window 6005 (case study 2,
# PAPER.md L217, L229).  H = 40: the smallest of {32, 40, 48, 56, 64} at which the injection-free
# trace flags nothing (tools/calibrate_h.py: 6 components at H = 32, none from 40 on).
C3_DEADLOCK = ((6000, (11240, 11243)), (6005, (11236, 11250)))
C3 = Workload("C3-4gpu", 900_000_000, 100_000_000, 81920, 32, 10000, 64, 40, seed=3, deadlock=C3_DEADLOCK,
              description="MGPUSim-shaped 4-GPU run: ~80k buffers, 1B records, 10k windows, injected "
                          "circular-full-buffer deadlock")
C3_CLEAN = C3.scaled("C3-clean", deadlock=())
# C3 shape at 1/100 of the records (same buffers, components, deadlock pair): oracle in seconds
C3_SMALL = C3.scaled("C3-small", n_samples=9_000_000, n_events=1_000_000, n_windows=100,
                     deadlock=((40, (11240, 11243)), (45, (11236, 11250))))
# C4: 1M buffers, Zipf(0.99) hot spots (YCSB-style exponent; BASELINE.json gives none), k = 1024.
# H = 96: the smallest of {16, 32, 48, 64, 96} at which the trace flags nothing (cold buffers held
# full between rare samples in quiet components; tools/calibrate_h.py: 593 at 32, 1 at 64, 0 at 96)
C4 = Workload("C4-skewed", 1_800_000_000, 200_000_000, 1 << 20, 64, 2000, 1024, 96, seed=4, zipf_s=0.99,
              description="skewed trace: 1M buffers, Zipf-distributed buffer_id hot spots, 2B records, top-k=1024")
C4_SMALL = C4.scaled("C4-small", n_samples=18_000_000, n_events=2_000_000, n_windows=20)
# C5: streamed in batches of windows at full size (tools/c5_full.py).  H = 2048: a component sees
# ~0.01 task events per window (800 events over 81920 components), so quiet gaps of a few hundred
# windows are normal; P(gap >= H) = exp(-H/102) over ~8e8 gaps needs H ~ 2000 to flag nothing.
# Measured: H = 256 flags ~850 components per window; H = 2048 one component in 2282 of 1M windows.
C5 = Workload("C5-long", 7_200_000_000, 800_000_000, 327680, 128, 1_000_000, 64, 2048, seed=5,
              description="long run: 16 simulated GPUs, ~320k buffers, 8B records in 1M windows")
CONFIGS = {w.name: w for w in (C1, C1_INVALID, C2, C3, C3_CLEAN, C3_SMALL, C4, C4_SMALL, C5)}


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
    tab = None
    if p.zipf_n:
        tab = _zipf_host(wl)
        p.zipf_cdf = tab.ctypes.data
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
        lib.gen_cuda_upload.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.POINTER(ctypes.c_void_p)]
        lib.gen_cuda_upload.restype = ctypes.c_int
        _dev = lib
    return _dev


_ZIPF_HOST: dict = {}
_ZIPF_DEV: dict = {}


def _zipf_key(wl):
    return (wl.n_buffers, wl.zipf_s)


def _zipf_host(wl):
    k = _zipf_key(wl)
    if k not in _ZIPF_HOST:
        _ZIPF_HOST[k] = wl.zipf_table()
    return _ZIPF_HOST[k]


def _zipf_dev(wl):
    """Device copy of the Zipf table (process lifetime; input data for the device generator)."""
    k = _zipf_key(wl)
    if k not in _ZIPF_DEV:
        t = _zipf_host(wl)
        ptr = ctypes.c_void_p()
        err = device_lib().gen_cuda_upload(t.ctypes.data, t.nbytes, ctypes.byref(ptr))
        if err != 0:
            raise RuntimeError(f"gen_cuda_upload failed: cudaError {err}")
        _ZIPF_DEV[k] = ptr.value
    return _ZIPF_DEV[k]


def fill_device(kind: str, wl: Workload, ptr: int, start: int, count: int, stream: int = 0) -> None:
    """Write records [start, start+count) of the (unsharded) trace into device memory at ptr."""
    p = wl.params()
    if p.zipf_n and kind == "samples":
        p.zipf_cdf = _zipf_dev(wl)
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
