"""GPU: the binding's world > 1 path end to end — two processes, a torch.distributed process group
(gloo: the one-GPU box has no second device for NCCL, both ranks share cuda:0), owner-component
sharding, `Monitor.window_reduce` = rtm_window_reduce_local -> all_gather of the packs -> rtm_merge.
Every rank's merged results must equal the whole-trace oracle, in rank modes
PERCENT and MEAN (the pack carries MEAN's 64-bit order keys)."""
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
        ref = oracle.Oracle(owner, cap, tot, n_components=wl.n_components, **kw).reduce(
            gen.samples(wl), gen.events(wl), wl.t_end())
        owned = (np.arange(wl.n_components) % world == rank).astype(np.uint8)
        mon = Monitor(owner, cap, tot, n_components=wl.n_components, rank=rank, world=world,
                      owned_components=owned, **kw)
        mon.ingest(_dev(gen.samples(wl, shard=(world, rank))), _dev(gen.events(wl, shard=(world, rank))))
        mon.window_reduce(wl.t_end())
        assert_same(mon.results(), ref, mon)
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
