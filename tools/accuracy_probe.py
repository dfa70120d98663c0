"""GPU side of the accuracy probe (run under gpurun): relaxed / start poses of
configs 1-3 through every engine, saved for the oracle comparison that
tools/accuracy_report.py runs on the host (no oracle on the GPU side).

Output: gpurun_out/<tag>.npz with, per case, the genes, the GPU energies and
gradients per engine, and free-running LS traces (Z19 ii)."""
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_solis_vasquezts25_b200 import ad, synth  # noqa: E402


def at_start(ctx, lid, genes, engine):
    """E and gradient of `genes` from engine `engine` (step 0 of a 1-iteration LS trace)."""
    g = torch.from_numpy(genes).cuda()
    wpc = 64 if engine.startswith("paper") else 0
    o = ctx.local_search(lid, g, max_iters=1, engine=engine, trace=True, warps_per_cta=wpc)
    torch.cuda.synchronize()
    tr = o["trace"][:, 0].cpu().numpy()
    stride = genes.shape[1]
    return tr[:, 0].copy(), tr[:, 1 + stride:].copy()


def main(tag):
    out = {}
    ctx = ad.Context(0)
    for cfg, n_relax, n_eng in ((1, 256, 256), (2, 3000, 1024), (3, 300, 192)):
        w = synth.make_config(cfg)
        ctx.upload_grid(w.grid)
        lid = ctx.upload_ligand(w.ligands[0], w.ff)
        starts = w.genes[:n_relax].copy()
        g = torch.from_numpy(starts).cuda()
        t0 = time.time()
        o = ctx.local_search(lid, g, max_iters=w.iters if cfg != 1 else 300, engine="simt")
        torch.cuda.synchronize()
        relaxed = g.cpu().numpy()
        out[f"c{cfg}_relaxed"] = relaxed
        out[f"c{cfg}_relaxed_bE"] = o["best_energy"].cpu().numpy()
        for kind, genes in (("relaxed", relaxed[:n_eng]), ("start", starts[:n_eng])):
            gd = torch.from_numpy(genes).cuda()
            E, G, A = ctx.score(lid, gd, grad=True, aux=True)
            torch.cuda.synchronize()
            out[f"c{cfg}_{kind}_score_E"] = E.cpu().numpy()
            out[f"c{cfg}_{kind}_score_G"] = G.cpu().numpy()
            for eng in ("simt", "tc", "paper", "paper_tcec"):
                E2, G2 = at_start(ctx, lid, genes, eng)
                out[f"c{cfg}_{kind}_{eng}_E"] = E2
                out[f"c{cfg}_{kind}_{eng}_G"] = G2
        # Z19 (ii): free-running traces from identical starts
        nt = 64 if cfg != 3 else 16
        for kind, genes in (("start", starts[:nt]), ("relaxed", relaxed[:nt])):
            gd = torch.from_numpy(genes).cuda()
            o = ctx.local_search(lid, gd, max_iters=300, engine="simt", trace=True)
            torch.cuda.synchronize()
            out[f"c{cfg}_{kind}_trace"] = o["trace"].cpu().numpy()
        print(f"config {cfg} done in {time.time() - t0:.1f} s", flush=True)
    ctx.close()
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    np.savez_compressed(os.path.join(ROOT, "gpurun_out", f"{tag}.npz"), **out)
    print("saved", tag)


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "probe")
