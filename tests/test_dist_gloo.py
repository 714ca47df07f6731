"""World-size-2 gloo test of the N>1 path on CPU.

Each rank reduces its owner-component shard with the oracle (the library needs a GPU), packs its
per-window results, exchanges them with the product's all-gather plumbing
(paper_conf_micro_mosallaeii024_b200.dist.allgather_packs over gloo), merges, and checks the
merged snapshot against the whole-trace oracle.  Also pins the LPT shard planner.
"""
from __future__ import annotations

import os
import socket
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _pack(out):
    """Fixed little-endian byte layout of the fields the merge needs (test-side packer)."""
    parts = [out["summary"].view(np.uint8).ravel(), out["topk"].view(np.uint8).ravel(),
             out["topk_n"].view(np.uint8).ravel(), out["progress"].view(np.uint8).ravel(),
             np.packbits(out["hung"], axis=1, bitorder="little").ravel()]
    return np.concatenate(parts)


def _unpack(buf, W, k, nk, nc):
    from oracle import PROGRESS_DTYPE, SUMMARY_DTYPE, TOPK_DTYPE

    o = 0
    res = {}
    n = W * SUMMARY_DTYPE.itemsize
    res["summary"] = buf[o:o + n].copy().view(SUMMARY_DTYPE); o += n
    n = W * k * TOPK_DTYPE.itemsize
    res["topk"] = buf[o:o + n].copy().view(TOPK_DTYPE).reshape(W, k); o += n
    n = W * 4
    res["topk_n"] = buf[o:o + n].copy().view(np.uint32); o += n
    n = W * nk * PROGRESS_DTYPE.itemsize
    res["progress"] = buf[o:o + n].copy().view(PROGRESS_DTYPE).reshape(W, nk); o += n
    nb = (nc + 7) // 8
    res["hung"] = np.unpackbits(buf[o:o + W * nb].reshape(W, nb), axis=1, bitorder="little")[:, :nc]
    return res


def _worker(rank, world, port, result_path):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    sys.path.insert(0, ROOT)
    import torch
    import torch.distributed as dist

    import gen
    import oracle
    from paper_conf_micro_mosallaeii024_b200.dist import allgather_packs, owned_mask, plan_components_lpt

    dist.init_process_group("gloo", rank=rank, world_size=world)
    wl = gen.C1.scaled("C1-gloo", n_samples=120_000, n_events=12_000, n_windows=5)
    owner, cap, tot = gen.registry(wl)
    s, e = gen.samples(wl), gen.events(wl)
    # shard plan from per-component record counts (LPT), then route records to their owner rank
    load = np.bincount(owner[np.minimum(s["buffer_id"], wl.n_buffers - 1)], minlength=wl.n_components)
    plan = plan_components_lpt(load, world)
    kw = dict(n_components=wl.n_components, t0=wl.t0, hang_windows=2, k=wl.k)
    mine_s = plan[owner[np.minimum(s["buffer_id"], wl.n_buffers - 1)]] == rank
    ecomp = np.minimum(e["meta"] & 0xFFFFF, wl.n_components - 1)
    mine_e = plan[ecomp] == rank
    orc = oracle.Oracle(owner, cap, tot, owned=owned_mask(plan, rank), **kw)
    local = orc.reduce(s[mine_s], e[mine_e], wl.t_end())
    assert local["rc"] == 0
    send = torch.from_numpy(_pack(local))
    recv = allgather_packs(send, world).numpy()
    per = len(send)
    shards = [_unpack(recv[r * per:(r + 1) * per], wl.n_windows, wl.k, wl.n_kernels, wl.n_components)
              for r in range(world)]
    top, top_n = oracle.merge_topk(shards, wl.k)
    whole = oracle.Oracle(owner, cap, tot, **kw).reduce(s, e, wl.t_end())
    ok = np.array_equal(top, whole["topk"]) and np.array_equal(top_n, whole["topk_n"])
    for f in ("n_samples", "n_events", "n_dropped", "n_touched", "n_hung"):
        ok &= np.array_equal(sum(x["summary"][f].astype(np.uint64) for x in shards), whole["summary"][f])
    dig = np.zeros(wl.n_windows, np.uint64)
    for x in shards:
        dig += x["summary"]["digest"]
    ok &= np.array_equal(dig, whole["summary"]["digest"])
    for f in ("started", "finished"):
        ok &= np.array_equal(sum(x["progress"][f] for x in shards), whole["progress"][f])
    hung = np.zeros_like(whole["hung"])
    for x in shards:
        hung |= x["hung"].astype(np.uint8)
    ok &= np.array_equal(hung, whole["hung"])
    with open(f"{result_path}.{rank}", "w") as f:
        f.write("ok" if ok else "mismatch")
    dist.destroy_process_group()


def test_gloo_world2_exchange_and_merge(tmp_path):
    import torch.multiprocessing as mp

    port = _free_port()
    path = str(tmp_path / "res")
    mp.start_processes(_worker, args=(2, port, path), nprocs=2, start_method="spawn", join=True)
    for r in range(2):
        assert open(f"{path}.{r}").read() == "ok"


def test_lpt_plan_balances_and_is_deterministic():
    from paper_conf_micro_mosallaeii024_b200.dist import plan_components_lpt

    rng = np.random.default_rng(4)
    load = (rng.zipf(1.3, size=5000) % 100000).astype(np.int64)
    for world in (2, 4, 8):
        plan = plan_components_lpt(load, world)
        per = np.bincount(plan, weights=load, minlength=world)
        # LPT bound: max load <= mean + max single item
        assert per.max() <= load.sum() / world + load.max()
        assert np.array_equal(plan, plan_components_lpt(load, world))
    assert list(plan_components_lpt([5, 5, 5, 5], 2)) == [0, 1, 0, 1]
