#!/usr/bin/env python
"""Benchmark: trace records/s reduced to window snapshots (BASELINE.json metric) on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]

One step = one rtm_window_reduce over the whole workload (all 1000 windows of C2, the
configuration BASELINE.json quotes the metric on: ~20k buffers, 90M level samples + 10M task
events, k=64), re-armed with rtm_reset.  Inputs are resident in HBM before the timed region
(1.6 GB > the 126 MB L2, so no flush is needed between steps).  `value` is whole-job records/s
(max-over-ranks device time); `e2e` repeats the metric through the same C-ABI with HOST
buffers (host->device copy of the trace and device->host read of the results inside the
timed region).  N > 1: weak scaling, every rank holds one C2-sized shard of an N-times larger
simulated system (owner-component sharding) and the per-window results are merged across
ranks with an all-gather + the library's merge kernels every step.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "trace records/sec reduced to snapshot (1/2/4/8 B200) + % HBM peak"
UNIT = "records/s"


def _peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


class ClockSampler:
    """SM clocks + throttle reasons sampled DURING the timed region (NVML every 2 ms; nvidia-smi
    fallback).  Reasons follow nvidia-smi's clocks_event_reasons names."""

    REASONS = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
               "hw_power_brake_slowdown": 0x80, "sw_power_cap": 0x4}

    def __init__(self, index: int, period: float = 0.002):
        self.index = index
        self.period = period
        self.rows = []  # (sm_mhz, max_mhz, reason_mask)
        self._stop = threading.Event()
        self._t = None
        self._nvml = None
        try:
            import pynvml

            pynvml.nvmlInit()
            self._nvml = pynvml
            self._h = pynvml.nvmlDeviceGetHandleByIndex(index)
            # the max clock is constant and its query slow (~3 ms): once, before the timed region;
            # one warm-up sample too (the first NVML queries of a process take several ms, which
            # left a 30 ms region with a single sample)
            self._max = float(pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM))
            self._sample()
        except Exception:
            self._nvml = None

    def _sample(self):
        if self._nvml is not None:
            n = self._nvml
            sm = n.nvmlDeviceGetClockInfo(self._h, n.NVML_CLOCK_SM)
            rs = n.nvmlDeviceGetCurrentClocksEventReasons(self._h)
            return float(sm), self._max, int(rs)
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.sw_power_cap,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.hw_thermal_slowdown")
        out = subprocess.run(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}", "--format=csv,noheader,nounits"],
                             capture_output=True, text=True, timeout=5).stdout
        p = [x.strip() for x in out.strip().split(",")]
        bits = (0x8, 0x4, 0x20, 0x40)
        mask = sum(b for b, v in zip(bits, p[2:6]) if v == "Active")
        return float(p[0]), float(p[1]), mask

    def _run(self):
        while not self._stop.is_set():
            try:
                self.rows.append(self._sample())
            except Exception:
                pass
            self._stop.wait(self.period)

    def __enter__(self):
        # the timed loop holds the GIL between its (GIL-releasing) library calls: a short switch
        # interval lets the sampler thread run every period instead of every 5 ms or less often
        self._switch = sys.getswitchinterval()
        sys.setswitchinterval(2e-4)
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join(timeout=10)
        sys.setswitchinterval(self._switch)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        sm = [r[0] for r in self.rows]
        reasons = sorted({k for r in self.rows for k, bit in self.REASONS.items() if r[2] & bit})
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": max(r[1] for r in self.rows), "reasons": reasons,
                "samples": len(self.rows), "source": "nvml" if self._nvml is not None else "nvidia-smi"}


# ---------------------------------------------------------------------------------------------
def cpu_reference_step(wl, n_windows_sample: int):
    """Oracle (as it stands, one host core) over the first `n_windows_sample` windows."""
    import gen
    import oracle

    ends = wl.t_end()[:n_windows_sample]
    t_hi = int(ends[-1])
    # bounded sample: the records with ts < t_hi (ts = t0 + (i*mul) >> 32 is monotone in i), plus a few
    # beyond it that the reduction drops as early records
    ns = min(wl.n_samples, int((t_hi - wl.t0) * wl.samples_per_tick) + 4)
    ne = min(wl.n_events, int((t_hi - wl.t0) * wl.n_events // max(1, wl.ticks)) + 4)
    s, e = gen.samples(wl, 0, ns), gen.events(wl, 0, ne)
    owner, cap, tot = gen.registry(wl)
    orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, t0=wl.t0, hang_windows=wl.hang_windows,
                        k=wl.k)
    t0 = time.perf_counter()
    out = orc.reduce(s, e, ends, want_hung=False)
    dt = time.perf_counter() - t0
    assert out["rc"] == 0
    recs = int(out["summary"]["n_samples"].sum() + out["summary"]["n_events"].sum() + out["summary"]["n_dropped"].sum())
    return recs, dt


def host_info():
    """nproc, CPU model and RAM of the box the baseline ran on."""
    model = None
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    ram = None
    try:
        for ln in open("/proc/meminfo"):
            if ln.startswith("MemTotal"):
                ram = round(int(ln.split()[1]) / 1024 / 1024, 1)
                break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model, "ram_gib": ram}


def _shard_worker(args):
    """One shard of the sharded oracle baseline: owner components c % P == r."""
    wl_name, n_win, P, r, barrier = args
    import gen
    import oracle

    wl = gen.CONFIGS[wl_name]
    ends = wl.t_end()[:n_win]
    t_hi = int(ends[-1])
    ns = min(wl.n_samples, int((t_hi - wl.t0) * wl.samples_per_tick) + 4)
    ne = min(wl.n_events, int((t_hi - wl.t0) * wl.n_events // max(1, wl.ticks)) + 4)
    s, e = gen.samples(wl, 0, ns, shard=(P, r)), gen.events(wl, 0, ne, shard=(P, r))
    owner, cap, tot = gen.registry(wl)
    owned = (np.arange(wl.n_components) % P == r).astype(np.uint8)
    orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, t0=wl.t0, hang_windows=wl.hang_windows,
                        k=wl.k, owned=owned)
    barrier.wait()  # every shard starts together: the parallel run shares the host's memory system
    t0 = time.perf_counter()
    out = orc.reduce(s, e, ends, want_hung=False)
    dt = time.perf_counter() - t0
    assert out["rc"] == 0
    return dt, out


def cpu_sharded_step(wl, n_win, P):
    """The oracle as it stands on P = nproc host processes, one component shard each (owner
    sharding), plus the merge of their per-window results (top-k lists, counters):
    SURVEY.md §8(d)(ii).  Time = the slowest shard's reduce + the merge."""
    import multiprocessing as mp

    import oracle

    ctx = mp.get_context("fork")
    with ctx.Manager() as m:
        barrier = m.Barrier(P)
        with ctx.Pool(P) as pool:
            res = pool.map(_shard_worker, [(wl.name, n_win, P, r, barrier) for r in range(P)])
    dts = [r[0] for r in res]
    outs = [r[1] for r in res]
    t0 = time.perf_counter()
    top, top_n = oracle.merge_topk(outs, wl.k)
    tot = {f: sum(o["summary"][f].astype(np.uint64) for o in outs)
           for f in ("n_samples", "n_events", "n_dropped", "digest", "n_touched")}
    prog = {f: sum(o["progress"][f] for o in outs) for f in ("started", "finished")}
    dt_merge = time.perf_counter() - t0
    del top, top_n, prog
    recs = int(tot["n_samples"].sum() + tot["n_events"].sum() + tot["n_dropped"].sum())
    return recs, max(dts) + dt_merge


def run_reference(args):
    """--impl reference: the CPU oracle as it stands, timed on the box's host cores (rank 0 only):
    `nproc` processes, one owner-component shard each, + the merge of their results (the
    single-core run when the host has one core or RTM_REF_CORES=1); same metric and config."""
    import gen

    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    wl = gen.C2
    info = host_info()
    P = int(os.environ.get("RTM_REF_CORES", str(info["nproc"] or 1)))
    n_win = int(os.environ.get("RTM_REF_WINDOWS", str(25 if P <= 1 else max(25, min(wl.n_windows, 2500 // P)))))

    def one():
        return cpu_reference_step(wl, n_win) if P <= 1 else cpu_sharded_step(wl, n_win, P)

    for _ in range(args.warmup):
        one()
    tot_recs, tot_t = 0, 0.0
    for _ in range(args.steps):
        r, dt = one()
        tot_recs += r
        tot_t += dt
    v = tot_recs / tot_t
    how = ("single-threaded C oracle" if P <= 1 else
           f"{P} processes, one owner-component shard each, + the merge (slowest shard's reduce + merge time)")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot_t / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
            "config": {"workload": wl.description, "sample": f"first {n_win} of {wl.n_windows} windows"},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": P, "kind": "oracle", "host": info,
                             "sample": f"first {n_win} windows of C2 ({tot_recs // args.steps} records/step), {how}"},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------------------------
def weak_registry(wl, rank, world):
    """Rank `rank`'s shard of the N-times larger system, as a RANK-LOCAL registry: its own
    C2-sized buffer set (dense local ids, include/rtm.h buffer_global_id) with the global id of
    every local buffer and the global owning component.  Global layout: component-major, global
    component = local component * N + rank (owner-component sharding)."""
    import gen

    wr = wl.scaled(wl.name, seed=wl.seed + 1000 * rank) if world > 1 else wl
    owner, cap, tot = gen.registry(wr)
    if world == 1:
        return wr, owner, cap, tot, None
    bpc = wl.buffers_per_comp
    lb = np.arange(wl.n_buffers, dtype=np.int64)
    gcomp = (lb // bpc) * world + rank
    gid = (gcomp * bpc + lb % bpc).astype(np.uint32)
    return wr, gcomp.astype(np.uint32), cap, tot * world, gid


def run_native(args):
    import torch

    import gen
    from paper_conf_micro_mosallaeii024_b200 import Monitor

    world = args.gpus
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("RTM_BENCH_BACKEND", "nccl") != "nccl":  # plumbing checks: ranks may share a GPU
        local %= torch.cuda.device_count()
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist

        backend = os.environ.get("RTM_BENCH_BACKEND", "nccl")  # gloo: ranks sharing one GPU (plumbing checks)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    wl = gen.CONFIGS[args.config]
    wr, owner, cap, tot, gid = weak_registry(wl, rank, world)
    nc = wl.n_components * world
    dev = torch.device("cuda", local)
    ds = torch.empty(wl.n_samples * 16, dtype=torch.uint8, device=dev)
    de = torch.empty(wl.n_events * 16, dtype=torch.uint8, device=dev)
    st = torch.cuda.current_stream(dev).cuda_stream
    gen.fill_device("samples", wr, ds.data_ptr(), 0, wl.n_samples, st)
    gen.fill_device("events", wr, de.data_ptr(), 0, wl.n_events, st)
    if world > 1:  # samples keep their rank-local buffer ids; events name global components
        gen.remap_weak(wr, ds.data_ptr(), 0, de.data_ptr(), wl.n_events, rank, world, st)
    torch.cuda.synchronize()
    extra = {} if gid is None else dict(buffer_global_id=gid, n_global_buffers=wl.n_buffers * world,
                                        pack_buffers=wl.n_buffers)
    mon = Monitor(owner, cap, tot, n_components=nc, t0=wl.t0, hang_windows=wl.hang_windows, k=wl.k, device=local,
                  rank=rank, world=world, rank_mode=args.rank_mode, **extra)
    t_end = wl.t_end()
    n_rec = wl.n_samples + wl.n_events

    def step():
        mon.reset()
        mon.ingest(ds, de)
        return mon.window_reduce(t_end)

    for _ in range(max(3, args.warmup)):
        res = step()
    # correctness guard on the timed configuration: every record accounted for
    S = res["summary"]
    assert int(S["n_samples"].sum() + S["n_events"].sum() + S["n_dropped"].sum()) == n_rec * world
    from paper_conf_micro_mosallaeii024_b200 import _native

    n_launch0 = _native.lib().rtm_kernel_launches()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        if dist:
            dist.barrier()
        torch.cuda.synchronize()
        t_wall = time.perf_counter()
        ev0.record()
        for _ in range(args.steps):
            step()
        ev1.record()
        torch.cuda.synchronize()
        t_wall = time.perf_counter() - t_wall
        if dist:
            dist.barrier()
    ms = ev0.elapsed_time(ev1)
    n_launches = int(_native.lib().rtm_kernel_launches() - n_launch0)
    # per-kernel CUDA-event times: a separate pass of the same K steps (not the timed region)
    mon.profile(True)
    ev0.record()
    for _ in range(args.steps):
        step()
    ev1.record()
    torch.cuda.synchronize()
    prof_ms = ev0.elapsed_time(ev1)
    prof = mon.profile_read()
    mon.profile(False)
    if dist:
        t = torch.tensor([ms], device=dev if dist.get_backend() == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    value = n_rec * world * args.steps / (ms / 1e3)

    # ---- e2e through the same C-ABI with HOST buffers (pinned), results read back each step
    e2e_value, e2e_steps = None, 0
    if 16 * n_rec <= (8 << 30) and not args.no_e2e:
        e2e_value, e2e_steps = run_e2e(args, mon, ds, de, wl, t_end, n_rec, world, dist, dev)
    streaming = None
    if world == 1 and not args.no_streaming:
        streaming = run_streaming(mon, ds, de, wl, t_end)
    W = wl.n_windows
    d2h = W * (8 * 6 + wl.k * 8 + 4 + wl.n_kernels * 40 + 4)
    rank_done = rank != 0
    if rank_done:
        if dist:
            dist.destroy_process_group()
        return
    return finish(args, wl, world, ms, prof, prof_ms, n_rec, value, e2e_value, e2e_steps, d2h, n_launches, clk,
                  t_wall, dist, streaming)


def run_streaming(mon, ds, de, wl, t_end, n_windows: int = 300, warmup: int = 20):
    """Per-window snapshot latency in streaming mode: one window per
    rtm_window_reduce call, the window's records already in HBM (slices of the resident trace),
    host wall clock from the ingest to the results on the host (the call blocks on its D2H)."""
    mon.reset()
    lat, recs = [], 0
    for w in range(warmup + n_windows):
        s0, s1 = wl.index_at("samples", wl.t_begin(w)), wl.index_at("samples", wl.t_begin(w + 1))
        e0, e1 = wl.index_at("events", wl.t_begin(w)), wl.index_at("events", wl.t_begin(w + 1))
        sv, ev, te = ds[s0 * 16:s1 * 16], de[e0 * 16:e1 * 16], t_end[w:w + 1]  # views made before the clock
        t = time.perf_counter()
        mon.ingest(sv, ev)
        mon.window_reduce(te)
        dt = time.perf_counter() - t
        if w >= warmup:
            lat.append(dt * 1e6)
            recs += (s1 - s0) + (e1 - e0)
    lat = np.array(lat)
    return {"what": "one window per rtm_window_reduce call, records resident in HBM, host wall clock per call",
            "windows": n_windows, "records_per_window": recs / n_windows,
            "p50_us": float(np.percentile(lat, 50)), "p99_us": float(np.percentile(lat, 99)),
            "tool": "tools/latency.py (per-kernel breakdown, C5)"}


def run_e2e(args, mon, ds, de, wl, t_end, n_rec, world, dist, dev):
    import torch

    hs = torch.empty(wl.n_samples * 16, dtype=torch.uint8, pin_memory=True)
    he = torch.empty(wl.n_events * 16, dtype=torch.uint8, pin_memory=True)
    hs.copy_(ds)
    he.copy_(de)
    torch.cuda.synchronize()
    e2e_steps = max(1, min(10, args.steps))  # ~30 ms per step (the H2D of 1.6 GB)

    def step_host():
        mon.reset()
        mon.ingest(hs, he)
        return mon.window_reduce(t_end)

    step_host()
    if dist:
        dist.barrier()
    torch.cuda.synchronize()
    te = time.perf_counter()
    for _ in range(e2e_steps):
        step_host()
    torch.cuda.synchronize()
    te = time.perf_counter() - te
    if dist:
        t = torch.tensor([te], device=dev if dist.get_backend() == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        te = float(t.item())
    return n_rec * world * e2e_steps / te, e2e_steps


NOMINAL_HBM_GBS = 8000.0  # B200 HBM3e nominal (SURVEY.md §8(d) reports both denominators)


def finish(args, wl, world, ms, prof, prof_ms, n_rec, value, e2e_value, e2e_steps, d2h, n_launches, clk, t_wall,
           dist, streaming=None):
    W = wl.n_windows
    # ---- roofline: algorithmic bytes = 16 B per record, read once.  They are
    # charged to the kernel that reads the records (k_partition; it also runs the task-event tiles
    # on the lane-major path); the fold reads only the 8-B staging entries (not algorithmic: they
    # show up in `traffic`).  The per-kernel numbers come from a separate profiled pass of the same
    # K steps (CUDA events around every launch, rtm_profile), so the timed region above carries no
    # profiling events.
    peaks = _peaks()
    hbm = float(peaks.get("hbm_gbs", 6650.0))
    step_ms = ms / args.steps
    pstep_ms = prof_ms / args.steps
    shares = {k: round(prof[k]["total_ms"] / args.steps / pstep_ms, 4) for k in prof if prof[k]["launches"]}
    algo = [k for k in prof if prof[k]["launches"] and prof[k]["algo_bytes"]]
    dom = max(algo, key=lambda k: prof[k]["total_ms"])
    dk = prof[dom]
    achieved_gbs = (dk["algo_bytes"] / dk["launches"]) / (dk["total_ms"] / dk["launches"] / 1e3) / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp) and args.config == "C2-1gpu":  # traffic.json holds the C2 capture
        try:
            allt = json.load(open(tp)).get("all", {})
            traffic = next((v for k, v in allt.items() if k == dom or k.startswith((dom + "_", dom + "<"))), None)
        except Exception:
            traffic = None
    per_kernel = {k: {"ms_per_step": round(prof[k]["total_ms"] / args.steps, 4), "share": shares[k],
                      "algo_bytes_per_launch": prof[k]["algo_bytes"] / prof[k]["launches"],
                      "achieved_gbs": (round((prof[k]["algo_bytes"] / prof[k]["launches"]) /
                                             (prof[k]["total_ms"] / prof[k]["launches"] / 1e3) / 1e9, 1)
                                       if prof[k]["algo_bytes"] else None)}
                  for k in prof if prof[k]["launches"]}
    path_gbs = 16.0 * n_rec / (step_ms / 1e3) / 1e9
    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        n_win = int(os.environ.get("RTM_CPU_WINDOWS", "40"))
        recs, dt = cpu_reference_step(wl, n_win)
        info = host_info()
        cpu = {"value": recs / dt, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"first {n_win} of {W} {wl.name} windows ({recs} records), single-threaded C oracle",
               "host": info}
        P = info["nproc"] or 1
        if P > 1 and not args.no_cpu_sharded:
            # every shard process generates the sample's records and keeps its own (~1.6 MB of
            # records per C2 window per process): bound the host memory to ~8 GB in total
            n_win_p = int(os.environ.get("RTM_CPU_WINDOWS_SHARDED", str(max(5, min(W, 10 * n_win, 5000 // P)))))
            recs_p, dt_p = cpu_sharded_step(wl, n_win_p, P)
            cpu["sharded"] = {"value": recs_p / dt_p, "unit": UNIT, "cores": P, "kind": "oracle",
                              "sample": f"first {n_win_p} of {W} {wl.name} windows ({recs_p} records) on {P} "
                                        "processes, one owner-component shard each, + the merge "
                                        "(slowest shard's reduce + merge time)"}
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": step_ms, "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int64",
        "data": "synthetic",
        "config": {"workload": wl.description + (f" (x{world} shards, weak scaling)" if world > 1 else ""),
                   "n_buffers": int(wl.n_buffers * world), "records_per_gpu": n_rec, "windows": W, "k": wl.k,
                   "hang_windows": wl.hang_windows, "rank_mode": args.rank_mode,
                   "l2": f"inputs ({16 * n_rec / 1e9:.1f} GB/GPU) larger than L2; no flush",
                   "parallelism": f"owner-component shards x{world}" if world > 1 else "single GPU"},
        "roofline": {"bound": "hbm", "kernel": dom, "achieved": achieved_gbs, "peak": hbm, "unit": "GB/s",
                     "frac": achieved_gbs / hbm, "frac_nominal": achieved_gbs / NOMINAL_HBM_GBS, "traffic": traffic,
                     "algo_bytes_per_launch": dk["algo_bytes"] / dk["launches"],
                     "algo_bytes_rule": "16 B per record read (SURVEY.md §8(d)); staging entries are not algorithmic",
                     "peak_source": "MEASURED_PEAKS.json hbm_gbs (burst copy)", "nominal_peak": NOMINAL_HBM_GBS,
                     "share": shares.get(dom),
                     "path_achieved": path_gbs, "path_frac": path_gbs / hbm,
                     "path_frac_nominal": path_gbs / NOMINAL_HBM_GBS},
        "kernels": per_kernel,
        "kernel_share": shares,
        "kernel_timing": f"separate profiled pass of {args.steps} steps ({pstep_ms:.4f} ms/step with events); "
                         "the timed region carries no profiling events",
        # side-stream kernels: their event interval runs from the partition's end until they get SM
        # slots beside the persistent fold (k_order_check, k_progress), or overlaps the partition
        "side_stream": [k for k in ("k_events", "k_order_check", "k_progress", "k_hang") if k in shares],
        "cpu_baseline": cpu,
        "e2e": ({"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": 16 * n_rec, "d2h_bytes_per_step": d2h,
                 "steps": e2e_steps,
                 "note": "pinned host trace -> device inside every step: bound by the host link "
                         "(16 B/record over PCIe/C2C), not by the kernels"}
                if e2e_value is not None else None),
        "streaming": streaming,
        "gpu_launches": n_launches,
        "clocks": clk.summary(),
        "wall_s_timed": t_wall,
    }
    print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="native", choices=["native", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-sharded", action="store_true", help="skip the nproc-process oracle baseline")
    ap.add_argument("--no-streaming", action="store_true", help="skip the one-window-per-call latency")
    ap.add_argument("--rank-mode", type=int, default=0, help="0 percent (bench line), 1 size, 2 mean occupancy")
    ap.add_argument("--config", default="C2-1gpu",
                    help="workload (gen.CONFIGS); the bench line is C2-1gpu, the others are parity configs "
                         "measured for profiles/")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    else:
        run_native(args)


if __name__ == "__main__":
    main()
