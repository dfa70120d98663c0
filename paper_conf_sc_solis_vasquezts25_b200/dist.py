"""Multi-GPU plumbing: shard independent (ligand, run) units over ranks, gather best poses.

Every LGA run is independent (Alg 1 coarse level), so the
only inter-GPU step is the final gather of fixed-size best-pose records
[energy, genes...].  Units are packed by LPT (longest processing
time first) on a cost model of one run's ADADELTA work.
"""
from __future__ import annotations

import heapq
import os


def unit_cost(n_atoms: int, n_tors: int, n_pairs: int, pop: int, iters: int) -> float:
    """Relative cost of one run: pop * iters * (pair + atom + rotation work), SURVEY §8(e)."""
    return float(pop) * iters * (75.0 * n_pairs + 200.0 * n_atoms + 30.0 * (n_atoms + 2 * n_tors) + 100.0)


def lpt_shard(costs, n_ranks: int):
    """Greedy LPT: assign units (by descending cost) to the least-loaded rank.
    Returns per-rank lists of unit indices, each sorted ascending (deterministic)."""
    if n_ranks < 1:
        raise ValueError("n_ranks >= 1")
    heap = [(0.0, r) for r in range(n_ranks)]
    heapq.heapify(heap)
    out = [[] for _ in range(n_ranks)]
    for u in sorted(range(len(costs)), key=lambda k: (-costs[k], k)):
        load, r = heapq.heappop(heap)
        out[r].append(u)
        heapq.heappush(heap, (load + costs[u], r))
    return [sorted(x) for x in out]


def gather_records(records, group=None):
    """all_gather_into_tensor of equally shaped per-rank record tensors [n, width]
    -> [world * n, width] (NCCL over NVLink on GPU, gloo on CPU)."""
    import torch
    import torch.distributed as dist
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size(group) == 1:
        return records
    ws = dist.get_world_size(group)
    src = records.contiguous()
    if records.is_cuda and dist.get_backend(group) == "gloo":
        src = src.cpu()  # gloo gathers host tensors (CPU tests of the multi-rank path on one GPU)
    out = torch.empty((ws * src.shape[0],) + tuple(src.shape[1:]), dtype=src.dtype, device=src.device)
    dist.all_gather_into_tensor(out, src, group=group)
    return out.to(records.device)


def init_process_group(backend: str, device=None):
    """torch.distributed.init_process_group from the launcher's environment (RANK,
    WORLD_SIZE, MASTER_ADDR/PORT) with a bounded collective timeout: a rank that dies
    or hangs turns the one gather into an error after AD_DIST_TIMEOUT_S seconds
    (default 600) instead of a silent hang (SURVEY §5 failure detection)."""
    import datetime

    import torch.distributed as dist
    timeout = datetime.timedelta(seconds=float(os.environ.get("AD_DIST_TIMEOUT_S", "600")))
    kw = {"timeout": timeout}
    if device is not None and backend == "nccl":
        kw["device_id"] = device
    dist.init_process_group(backend, **kw)
