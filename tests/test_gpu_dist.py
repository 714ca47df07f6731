"""GPU: the binding's world > 1 path end to end — two processes, a torch.distributed process group
(gloo: the one-GPU box has no second device for NCCL, both ranks share cuda:0), owner-component
sharding, `Monitor.window_reduce` = rtm_window_reduce_local -> all_gather of the packs -> rtm_merge.
Every rank's merged results must equal the whole-trace oracle, in rank modes
PERCENT and MEAN (the pack carries MEAN's 64-bit order keys), across two calls with a progress bar
destroyed and another updated in between; the windows-in-top-k counter and the value monitor's
rings (filled on the owning rank only) are compared too."""
from __future__ import annotations

import os
import socket
import sys
import traceback

import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, mode, result_path):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    sys.path.insert(0, ROOT)
    try:
        import numpy as np
        import torch
        import torch.distributed as dist

        import gen
        import oracle
        from paper_conf_micro_mosallaeii024_b200 import Monitor
        from tests.test_gpu_parity import _dev, assert_same

        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        wl = gen.C1.scaled("C1-dist", n_samples=200_000, n_events=20_000, n_windows=6)
        owner, cap, tot = gen.registry(wl)
        kw = dict(t0=wl.t0, hang_windows=2, k=wl.k, rank_mode=mode)
        orc = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, **kw)
        owned = (np.arange(wl.n_components) % world == rank).astype(np.uint8)
        mon = Monitor(owner, cap, tot, n_components=wl.n_components, rank=rank, world=world,
                      owned_components=owned, **kw)
        watched = [0, 5, 17, 998]  # owners 0, 1, 4, 249: both ranks own some
        mon.watch(watched)
        s_all, e_all = gen.samples(wl), gen.events(wl)
        s_sh, e_sh = gen.samples(wl, shard=(world, rank)), gen.events(wl, shard=(world, rank))
        t_end = wl.t_end()
        rows = []
        for lo, hi in ((0, 2), (2, 6)):
            if lo == 2:  # dynamic progress bars between calls, the same on every rank
                for x in (orc, mon):
                    x.bar_destroy(0)
                    x.bar_update(1, 4321)
            sl = slice(wl.index_at("samples", wl.t_begin(lo)), wl.index_at("samples", wl.t_begin(hi)))
            el = slice(wl.index_at("events", wl.t_begin(lo)), wl.index_at("events", wl.t_begin(hi)))
            ref = orc.reduce(s_all[sl], e_all[el], t_end[lo:hi], want_all_stats=True)
            rows.append(ref["all_stats"])
            ss = s_sh[(s_sh["ts"] >= wl.t_begin(lo)) & (s_sh["ts"] < wl.t_begin(hi))]
            es = e_sh[(e_sh["ts"] >= wl.t_begin(lo)) & (e_sh["ts"] < wl.t_begin(hi))]
            mon.ingest(_dev(ss), _dev(es))
            mon.window_reduce(t_end[lo:hi])
            assert_same(mon.results(), ref, mon)
        # windows-in-top-k counter, counted from the merged lists
        assert np.array_equal(mon.topk_persistence(), orc.persistence())
        # value monitor: the owner's ring equals the oracle's per-window table, others stay empty
        A = np.concatenate(rows)
        for q, b in enumerate(watched):
            ser = mon.watch_series(q)
            if owned[owner[b]]:
                assert np.array_equal(ser["t_end"], t_end), b
                for f in ("integral", "last", "max", "min", "capacity", "n_samples", "mean_occ"):
                    assert np.array_equal(ser[f], A[:, b][f]), (b, f)
            else:
                assert len(ser) == 0, b
        msg = "ok"
        dist.destroy_process_group()
    except Exception:  # noqa: BLE001 - reported through the result file
        msg = traceback.format_exc()
    with open(f"{result_path}.{rank}", "w") as f:
        f.write(msg)


@pytest.mark.parametrize("mode", [0, 2])
def test_monitor_world2_gloo_merge_equals_whole(tmp_path, mode):
    import torch.multiprocessing as mp

    path = str(tmp_path / "res")
    mp.start_processes(_worker, args=(2, _free_port(), mode, path), nprocs=2, start_method="spawn", join=True)
    for r in range(2):
        assert open(f"{path}.{r}").read() == "ok"
