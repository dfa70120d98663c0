"""Launch the LS kernel a few times on a config (for ncu): python tools/prof_ls.py [cfg] [engine] [launches]"""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_solis_vasquezts25_b200 import ad, synth  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
engine = sys.argv[2] if len(sys.argv) > 2 else "tc"
launches = int(sys.argv[3]) if len(sys.argv) > 3 else 3
w = synth.make_config(cfg)
ctx = ad.Context(0)
ctx.upload_grid(w.grid)
lid = ctx.upload_ligand(w.ligands[0], w.ff)
start = torch.from_numpy(w.genes).cuda()
for _ in range(launches):
    g = start.clone()
    ctx.local_search(lid, g, max_iters=w.iters, engine=engine, warps_per_cta=(64 if engine == "paper" else 0),
                     pop_per_run=w.pop)
torch.cuda.synchronize()
print("done")
