"""Command-line docking on real inputs (the artifact command of
P:L520-521: ``autodock_gpu -ffile protein.maps.fld -lfile ligand.pdbqt -nrun N``).

    python -m paper_conf_sc_solis_vasquezts25_b200.dock --ffile protein.maps.fld \\
        --lfile ligand.pdbqt --nrun 20 [--lga] [--pop 150] [--lsit 300] [--seed 0] [--out res.json]

Reads the AutoGrid maps and the PDBQT ligand (io.py), uploads them through the C
ABI, and runs either ADADELTA local search from random starts (the north_star hot
path: nrun x pop poses, lsit iterations, Alg 3) or the Lamarckian GA
(--lga, Alg 1, ad_lga_run).  Prints one line per run (best energy,
genotype) and writes them as JSON.  Every step runs in libad on the GPU; there
is no CPU fallback.
"""
from __future__ import annotations

import argparse
import json
import sys

import numpy as np


def random_starts(rng, n, n_tors, grid, around):
    """Start genotypes: translation uniform within 2 A of `around` (grid units),
    uniform random orientation (axis on the sphere, alpha U[0, 360)), torsions
    U[-180, 180) -- the synthetic generator's recipe centred on the
    ligand's input position."""
    g = np.zeros((n, 6 + n_tors), np.float32)
    h = float(grid.spacing)
    g[:, :3] = around[None, :] + rng.uniform(-2.0, 2.0, (n, 3)) / h
    g[:, 3] = rng.uniform(0.0, 360.0, n)
    g[:, 4] = np.degrees(np.arccos(1.0 - 2.0 * rng.uniform(0.0, 1.0, n)))
    g[:, 5] = rng.uniform(0.0, 360.0, n)
    g[:, 6:] = rng.uniform(-180.0, 180.0, (n, n_tors))
    return g


def main(argv=None):
    ap = argparse.ArgumentParser(description=__doc__.split("\n\n")[0])
    ap.add_argument("--ffile", required=True, help="AutoGrid field file (protein.maps.fld)")
    ap.add_argument("--lfile", required=True, help="ligand PDBQT")
    ap.add_argument("--nrun", type=int, default=20)
    ap.add_argument("--pop", type=int, default=150)
    ap.add_argument("--lsit", type=int, default=300, help="ADADELTA iterations per local search")
    ap.add_argument("--lga", action="store_true", help="Lamarckian GA (Alg 1) instead of LS from random starts")
    ap.add_argument("--ngen", type=int, default=27000, help="--lga: generation budget")
    ap.add_argument("--nev", type=int, default=2_500_000, help="--lga: evaluation budget per run")
    ap.add_argument("--engine", default="simt", choices=["simt", "tc", "tc_fp16", "paper", "paper_tcec"])
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--device", type=int, default=0)
    ap.add_argument("--out", default=None, help="write the per-run results as JSON")
    a = ap.parse_args(argv)

    import torch

    from . import ad
    from . import io as adio
    from .synth import FFParams

    grid, names = adio.read_fld(a.ffile)
    lig, centroid = adio.read_pdbqt(a.lfile, names)
    ff = FFParams()
    ctx = ad.Context(a.device)
    try:
        ctx.upload_grid(grid)
        lid = ctx.upload_ligand(lig, ff)
        rng = np.random.default_rng(a.seed)
        around = adio.input_genes(centroid, grid, lig.n_tors)[:3]
        starts = random_starts(rng, a.nrun * a.pop, lig.n_tors, grid, around)
        g = torch.from_numpy(starts).to(f"cuda:{a.device}")
        if a.lga:
            out = ctx.lga(lid, g, a.nrun, pop_size=a.pop, max_gens=a.ngen, max_evals=a.nev, ls_iters=a.lsit,
                          seed=a.seed, engine=a.engine)
            rb = out["run_best"]
        else:
            out = ctx.local_search(lid, g, max_iters=a.lsit, engine=a.engine, pop_per_run=a.pop,
                                   warps_per_cta=(64 if a.engine.startswith("paper") else 0))
            rb = out["run_best"]
        torch.cuda.synchronize()
        ctx.sync()
        rb = rb.cpu().numpy()
    finally:
        ctx.close()
    runs = [{"run": r, "energy": float(rb[r, 0]), "genes": [float(v) for v in rb[r, 1:1 + 6 + lig.n_tors]]}
            for r in range(a.nrun)]
    for rr in sorted(runs, key=lambda x: x["energy"]):
        print(f"run {rr['run']:4d}  E = {rr['energy']:12.4f} kcal/mol")
    if a.out:
        with open(a.out, "w") as f:
            json.dump({"ffile": a.ffile, "lfile": a.lfile, "n_atoms": lig.n_atoms, "n_tors": lig.n_tors,
                       "n_pairs": lig.n_pairs, "mode": "lga" if a.lga else "ls", "runs": runs}, f, indent=1)
    return runs


if __name__ == "__main__":
    main(sys.argv[1:])
