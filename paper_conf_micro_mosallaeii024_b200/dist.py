"""Multi-rank plumbing for owner-component sharding.

Host-side only: the shard plan and the all-gather of the per-rank result packs.  The merge itself
runs in the library's kernels (``rtm_merge``).  Works with the NCCL backend on GPUs and with gloo on
CPU (tests/test_dist_gloo.py).
"""
from __future__ import annotations

import heapq

import numpy as np


def plan_components_lpt(component_load, world: int) -> np.ndarray:
    """Longest-processing-time assignment of components to ranks.

    component_load[c] = records of component c (e.g. from a histogram pre-pass).  Returns
    rank[c].  LPT places each component, heaviest first, on the currently lightest rank; ties go
    to the lowest rank id, so the plan is deterministic.
    """
    load = np.asarray(component_load, dtype=np.int64)
    order = np.lexsort((np.arange(len(load)), -load))  # heaviest first, then id
    heap = [(0, r) for r in range(world)]
    rank = np.empty(len(load), dtype=np.int32)
    for c in order:
        tot, r = heapq.heappop(heap)
        rank[c] = r
        heapq.heappush(heap, (tot + int(load[c]), r))
    return rank


def owned_mask(rank_of_component, rank: int) -> np.ndarray:
    return (np.asarray(rank_of_component) == rank).astype(np.uint8)


def allgather_packs(send, world: int, group=None):
    """Gather every rank's packed per-window results (rank-major) — the one exchange step."""
    import torch
    import torch.distributed as dist

    if send.is_cuda and dist.get_backend(group) == "gloo":  # gloo: stage through host memory
        return allgather_packs(send.cpu(), world, group).to(send.device)
    recv = torch.empty(world * send.numel(), dtype=send.dtype, device=send.device)
    try:
        dist.all_gather_into_tensor(recv, send, group=group)
    except (RuntimeError, NotImplementedError):  # backends without the fused collective
        parts = [torch.empty_like(send) for _ in range(world)]
        dist.all_gather(parts, send, group=group)
        recv = torch.cat(parts)
    return recv
