"""Are two library builds bit-identical on the LS path?  (A/B of code changes that
should not change arithmetic.)

usage: python tools/lib_equal.py LIB_A LIB_B [CFG ...]   (default configs 1 2 3)
Runs each library in its own subprocess (AD_LIB) on the first 256 poses of each
config, 30 SIMT LS iterations plus one scoring call, and compares best energies,
final genes and gradients bit for bit."""
import os
import subprocess
import sys
import tempfile

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r"""
import sys, numpy as np, torch
sys.path.insert(0, %r)
from paper_conf_sc_solis_vasquezts25_b200 import ad, synth
out = {}
for cfg in map(int, sys.argv[2:]):
    w = synth.make_config(cfg)
    ctx = ad.Context(0); ctx.upload_grid(w.grid); lid = ctx.upload_ligand(w.ligands[0], w.ff)
    n = min(256, w.n_poses)
    g = torch.from_numpy(w.genes[:n].copy()).cuda()
    E, G, _ = ctx.score(lid, g, grad=True)
    o = ctx.local_search(lid, g, max_iters=30, engine="simt")
    torch.cuda.synchronize()
    out[f"E{cfg}"] = E.cpu().numpy(); out[f"G{cfg}"] = G.cpu().numpy()
    out[f"best{cfg}"] = o["best_energy"].cpu().numpy(); out[f"genes{cfg}"] = g.cpu().numpy()
    ctx.close()
np.savez(sys.argv[1], **out)
""" % ROOT


def main():
    a, b = sys.argv[1], sys.argv[2]
    cfgs = sys.argv[3:] or ["1", "2", "3"]
    res = []
    with tempfile.TemporaryDirectory() as d:
        for k, lib in enumerate((a, b)):
            f = os.path.join(d, f"{k}.npz")
            env = dict(os.environ, AD_LIB=os.path.abspath(lib))
            subprocess.check_call([sys.executable, "-c", CHILD, f, *cfgs], env=env)
            res.append(dict(np.load(f)))
    ok = True
    for key in res[0]:
        x, y = res[0][key], res[1][key]
        same = np.array_equal(x, y)
        ok &= same
        print(f"{key:8s} {'equal' if same else 'DIFFER'}  n_diff {int((x != y).sum())}  max |d| {np.abs(x.astype(np.float64) - y).max():.3g}")
    print("ALL EQUAL" if ok else "NOT EQUAL")


if __name__ == "__main__":
    main()
