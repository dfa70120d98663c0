"""Virtual screen (config 5): many ligands x runs, sharded over ranks, one gather.

Units = (ligand, run) pairs, each `pop` poses of ADADELTA local search
(Alg 3) against one receptor.  Units are LPT-packed over ranks
(dist.lpt_shard); every rank uploads only its ligands, buckets them by shared-
memory footprint (one ad_local_search launch per bucket, pose_ligand selects the
ligand of every pose), and the best pose of every unit is gathered with one
all_gather_into_tensor (NCCL over NVLink on GPUs).  Record layout (float32):
[ligand id, run id, best energy, genes (stride)].
"""
from __future__ import annotations

import numpy as np

from . import dist as addist


def plan(ligands, runs, pop, iters, world):
    costs, units = [], []
    for k, L in enumerate(ligands):
        c = addist.unit_cost(L.n_atoms, L.n_tors, L.n_pairs, pop, iters)
        for r in range(runs):
            units.append((k, r))
            costs.append(c)
    return units, addist.lpt_shard(costs, world)


def run_screen(ctx, grid, ff, ligands, start_genes, runs, pop, iters, rank=0, world=1, engine="simt",
               n_buckets=4, stream_sync=True):
    """start_genes: [n_ligands * runs * pop, stride] host array (ligand-major, run, pop).
    Returns (records [n_units_total_padded, 3 + stride] torch tensor on rank's device, units list)."""
    import torch

    from . import ad
    stride = start_genes.shape[1]
    units, shards = plan(ligands, runs, pop, iters, world)
    mine = [units[u] for u in shards[rank]]
    ctx.upload_grid(grid)
    # bucket units by ligand footprint (pairs ~ blob size), one launch per bucket;
    # only the bucket's ligands are live during its launch (the library sizes
    # shared memory for the largest live ligand)
    order = sorted(mine, key=lambda kr: (ligands[kr[0]].n_pairs, kr))
    buckets = [b for b in np.array_split(np.arange(len(order)), max(1, min(n_buckets, len(order)))) if len(b)]
    dev = torch.device("cuda", torch.cuda.current_device())
    n_max = max(len(s) for s in shards)
    rec = torch.full((n_max, 3 + stride), float("nan"), device=dev)
    row = 0
    for b in buckets:
        us = [order[i] for i in b]
        lig_ids = {k: ctx.upload_ligand(ligands[k], ff) for k in sorted({k for k, _ in us})}
        genes = np.concatenate([start_genes[(k * runs + r) * pop:(k * runs + r + 1) * pop] for k, r in us])
        pl = np.repeat(np.array([lig_ids[k] for k, _ in us], np.int32), pop)
        g = torch.from_numpy(genes).to(dev)
        bE = torch.empty(len(genes), device=dev)
        rb = torch.empty(len(us), 1 + stride, device=dev)
        big = max(us, key=lambda kr: ligands[kr[0]].n_pairs)[0]
        ad.ad_local_search(ctx.h, lig_ids[big], torch.from_numpy(pl).to(dev), g, bE, rb, None, max_iters=iters,
                           pop_per_run=pop, engine=ad.ENGINES[engine], warps_per_cta=(8 if pop % 8 == 0 else 1))
        ids = torch.tensor([[k, r] for k, r in us], dtype=torch.float32, device=dev)
        rec[row:row + len(us), :2] = ids
        rec[row:row + len(us), 2:] = rb
        row += len(us)
        for lid in lig_ids.values():  # synchronises the device
            ad.ad_free_ligand(ctx.h, lid)
    if stream_sync:
        torch.cuda.synchronize()
    return addist.gather_records(rec), units
