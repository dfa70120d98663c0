"""Virtual screen (config 5): many ligands x runs, sharded over ranks, one gather.

Units = (ligand, run) pairs, each `pop` poses of ADADELTA local search
(Alg 3) against one receptor.  Units are LPT-packed over ranks
(dist.lpt_shard); every rank uploads only its ligands (all resident, uploads
from a pool of host threads), buckets its units by shared-memory footprint
(one ad_local_search launch per bucket; ad_set_launch_ligands sizes the launch
for the bucket's ligands, pose_ligand selects the ligand of every pose), and
the best pose of every unit is gathered with one all_gather_into_tensor (NCCL
over NVLink on GPUs).  Record layout (float32): [ligand id, run id, best
energy, genes (stride)].
"""
from __future__ import annotations

import os

import numpy as np

from . import dist as addist


def plan(spec, world):
    """LPT shard of the (ligand, run) units; unit cost from the ligand's size (its
    pair count when the ligand exists, else the spec's estimate)."""
    costs, units = [], []
    for k in range(spec.n_ligands):
        n, t = spec.sizes[k]
        c = addist.unit_cost(n, t, spec.n_pairs(k), spec.pop, spec.iters)
        for r in range(spec.runs):
            units.append((k, r))
            costs.append(c)
    return units, addist.lpt_shard(costs, world)


class ListSpec:
    """A screen over explicit ligands and start genotypes ([n_ligands * runs * pop,
    stride], ligand-major) with the interface of synth.ScreenSpec."""

    def __init__(self, grid, ligands, start_genes, runs, pop, iters):
        self.grid, self.ligands, self.start = grid, ligands, start_genes
        self.n_ligands, self.runs, self.pop, self.iters = len(ligands), runs, pop, iters
        self.stride = start_genes.shape[1]
        self.sizes = [(L.n_atoms, L.n_tors) for L in ligands]

    def ligand(self, k):
        return self.ligands[k]

    def genes(self, k):
        n = self.runs * self.pop
        return self.start[k * n:(k + 1) * n]

    def n_pairs(self, k):
        return self.ligands[k].n_pairs


_GEN_SPEC = None


def _gen(k):
    return _GEN_SPEC.ligand(k), _GEN_SPEC.genes(k)


def generate(spec, ks, processes=0):
    """Ligands and start genotypes of ligands ks (a fork pool over the host cores
    for a lazy spec: input synthesis is ~30 ms of NumPy per ligand)."""
    global _GEN_SPEC
    if processes <= 1 or len(ks) < 64 or isinstance(spec, ListSpec):
        return {k: (spec.ligand(k), spec.genes(k)) for k in ks}
    import multiprocessing as mp
    _GEN_SPEC = spec
    with mp.get_context("fork").Pool(processes) as pool:
        out = pool.map(_gen, ks, chunksize=max(1, len(ks) // (8 * processes)))
    _GEN_SPEC = None
    return dict(zip(ks, out))


def make_buckets(mine, ligands, n_buckets, kind=None):
    """Split this rank's units into launch buckets: grouped by (wide ligand, pair-loop
    kind) -- a bucket never mixes >32-gene ligands with narrow ones (the wide kernel
    variant would then run for all) nor pair-loop kinds (a launch runs the specialised
    kernel twins only when all its ligands share the kind; kind: ligand -> ad
    .pair_loop_kind) -- ordered by pair count so the footprint bound stays tight, and
    cut at equal unit counts."""
    kind = kind or {}
    key = lambda k: (6 + ligands[k].n_tors > 32, kind.get(k, 0))  # noqa: E731
    order = sorted(mine, key=lambda kr: (key(kr[0]), ligands[kr[0]].n_pairs, kr))
    out = []
    for grp in sorted({key(k) for k, _ in mine}):
        part = [u for u in order if key(u[0]) == grp]
        nb = max(1, round(n_buckets * len(part) / len(order)))
        out += [[part[i] for i in b] for b in np.array_split(np.arange(len(part)), min(nb, len(part))) if len(b)]
    return out


class Screen:
    """One rank's share of a screen, set up once (grid + its ligands uploaded,
    buckets and device buffers built) and run any number of times (`step`).
    spec: synth.ScreenSpec or ListSpec."""

    def __init__(self, ctx, spec, ff, rank=0, world=1, engine="simt", n_buckets=8, effort=None,
                 upload_threads=0, gen_processes=0):
        import time

        import torch

        from . import ad
        t0 = time.perf_counter()
        self.ctx, self.spec, self.engine = ctx, spec, engine
        runs, pop = spec.runs, spec.pop
        self.runs, self.pop, self.iters, self.stride = runs, pop, spec.iters, spec.stride
        self.units, shards = plan(spec, world)
        mine = [self.units[u] for u in shards[rank]]
        self.n_rec = max(len(s) for s in shards)  # equal record count on every rank (gather)
        need = sorted({k for k, _ in mine})
        made = generate(spec, need, gen_processes)
        ligands = {k: made[k][0] for k in need}
        t1 = time.perf_counter()
        ctx.upload_grid(spec.grid)
        if effort is not None:
            ctx.set_schedule_effort(effort)
        ids = ctx.upload_ligands([ligands[k] for k in need], ff, threads=upload_threads)
        self.lig_id = dict(zip(need, ids))
        t2 = time.perf_counter()
        dev = torch.device("cuda", torch.cuda.current_device())
        self.buckets = []
        kind = {k: ad.pair_loop_kind(ctx.h, self.lig_id[k]) for k in need}
        for us in make_buckets(mine, ligands, n_buckets, kind):
            genes = np.concatenate([made[k][1][r * pop:(r + 1) * pop] for k, r in us])
            pl = np.repeat(np.array([self.lig_id[k] for k, _ in us], np.int32), pop)
            self.buckets.append({
                "units": us,
                "lig_ids": sorted({self.lig_id[k] for k, _ in us}),
                "bound": self.lig_id[max(us, key=lambda kr: ligands[kr[0]].n_pairs)[0]],
                "start": torch.from_numpy(np.ascontiguousarray(genes)).to(dev),
                "genes": torch.empty((len(genes), self.stride), dtype=torch.float32, device=dev),
                "pl": torch.from_numpy(pl).to(dev),
                "bE": torch.empty(len(genes), dtype=torch.float32, device=dev),
                "rb": torch.empty(len(us), 1 + self.stride, dtype=torch.float32, device=dev),
                "ids": torch.tensor([[k, r] for k, r in us], dtype=torch.float32, device=dev),
            })
        self.rec = torch.full((self.n_rec, 3 + self.stride), float("nan"), device=dev)
        self.n_units = len(mine)
        self.n_poses = self.n_units * pop
        self.ligands = ligands  # this rank's ligands, by screen index
        self.setup_s = {"generate": t1 - t0, "upload": t2 - t1}
        self.ad = ad

    def pin_host_inputs(self):
        """Pinned host copies of every bucket's start genotypes (for end-to-end
        steps that copy the inputs host -> device inside the timed region)."""
        for b in self.buckets:
            b["host"] = b["start"].cpu().pin_memory()
        return sum(b["host"].numel() * 4 for b in self.buckets)

    def step(self, n_evals=None, gather=True, from_host=False, ckpt_dir=None, rank=0):
        """Restore the start genotypes (device copy, or from the pinned host copies
        with from_host), run every bucket's LS launch, write the unit records; then
        (world > 1) gather them.  Enqueued on the current stream; returns the
        (gathered) record tensor.

        ckpt_dir (screen resilience): every finished bucket's records are
        written to ckpt_dir/rank<rank>_bucket<i>.npy (synchronously, atomic rename), and
        a bucket whose file exists is not launched again but read back -- a screen
        restarted after a crash or preemption resumes at its first unfinished bucket."""
        import torch
        ad = self.ad
        row = 0
        for i, b in enumerate(self.buckets):
            n = len(b["units"])
            path = os.path.join(ckpt_dir, f"rank{rank}_bucket{i}.npy") if ckpt_dir else None
            if path and os.path.exists(path):
                saved = torch.from_numpy(np.load(path)).to(self.rec.device)
                if tuple(saved.shape) == (n, self.rec.shape[1]) and torch.equal(saved[:, :2], b["ids"]):
                    self.rec[row:row + n] = saved
                    row += n
                    continue
            b["genes"].copy_(b["host"] if from_host else b["start"], non_blocking=True)
            ad.ad_set_launch_ligands(self.ctx.h, b["lig_ids"])
            ad.ad_local_search(self.ctx.h, b["bound"], b["pl"], b["genes"], b["bE"], b["rb"], n_evals,
                               max_iters=self.iters, pop_per_run=self.pop, engine=ad.ENGINES[self.engine])
            self.rec[row:row + n, :2] = b["ids"]
            self.rec[row:row + n, 2:] = b["rb"]
            if path:
                os.makedirs(ckpt_dir, exist_ok=True)
                np.save(path + ".tmp.npy", self.rec[row:row + n].cpu().numpy())  # (synchronises the stream)
                os.replace(path + ".tmp.npy", path)
            row += n
        ad.ad_set_launch_ligands(self.ctx.h, None)
        return addist.gather_records(self.rec) if gather else self.rec

    def close(self):
        for lid in self.lig_id.values():
            self.ctx.free_ligand(lid)
        self.lig_id = {}


def run_screen(ctx, grid, ff, ligands, start_genes, runs, pop, iters, rank=0, world=1, engine="simt",
               n_buckets=4, stream_sync=True, ckpt_dir=None):
    """One screen: start_genes [n_ligands * runs * pop, stride] host array
    (ligand-major, run, pop).  Returns (records [world * n_rec, 3 + stride] torch
    tensor on the rank's device, units list).  ckpt_dir: per-bucket result files,
    resume (Screen.step)."""
    import torch
    s = Screen(ctx, ListSpec(grid, ligands, start_genes, runs, pop, iters), ff, rank=rank, world=world,
               engine=engine, n_buckets=n_buckets)
    try:
        rec = s.step(ckpt_dir=ckpt_dir, rank=rank)
        if stream_sync:
            ctx.sync()  # device-side argument errors (pose_ligand, footprint, stride) raise here
        return rec, s.units
    finally:
        s.close()
