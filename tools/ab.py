"""A/B timing of library builds / launch shapes / intra modes, interleaved subprocess runs.

usage: python tools/ab.py CFG ENGINE LIB[:W[:MODE[:LAYOUT[:NAME=VALUE...]]]] ...   (3 rounds x 5 timed launches each)
Prints the median ms per LS launch (config CFG, full workload) per variant.
"""
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import os, sys, json, torch
sys.path.insert(0, %r)
from paper_conf_sc_solis_vasquezts25_b200 import ad, synth
cfg, eng, w = int(sys.argv[1]), sys.argv[2], int(sys.argv[3])
wl = synth.make_config(cfg)
if os.environ.get("AB_ITERS"): wl.iters = int(os.environ["AB_ITERS"])  # shorter trajectories (A/B of code, not of trajectory luck)
ctx = ad.Context(0); ctx.upload_grid(wl.grid); lid = ctx.upload_ligand(wl.ligands[0], wl.ff)
start = torch.from_numpy(wl.genes).cuda(); g = start.clone()
flush = torch.empty(64 * 1024 * 1024, device='cuda')
ts = []
for k in range(8):
    g.copy_(start); flush.fill_(k)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); ctx.local_search(lid, g, max_iters=wl.iters, engine=eng, warps_per_cta=w); b.record()
    torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
print(json.dumps({"ms": sorted(ts[3:]), "launch": ad.ad_last_launch(ctx.h), "evals": wl.n_poses * wl.iters}))
""" % ROOT


def main():
    cfg, eng = sys.argv[1], sys.argv[2]
    variants = sys.argv[3:]
    res = {v: [] for v in variants}
    meta = {}
    for _ in range(3):
        for v in variants:
            parts = v.split(":")
            lib, w, mode = parts[0], (parts[1] if len(parts) > 1 else "0") or "0", (parts[2] if len(parts) > 2 else "")
            layout = parts[3] if len(parts) > 3 else ""
            env = dict(os.environ, AD_LIB=os.path.abspath(lib))
            if mode:
                env["AD_INTRA_MODE"] = mode
            if layout:
                env["AD_GRID_LAYOUT"] = layout
            for kv in parts[4:]:  # extra NAME=VALUE environment settings
                k, _, val = kv.partition("=")
                env[k] = val
            out = subprocess.check_output([sys.executable, "-c", CHILD, cfg, eng, w], env=env, text=True)
            d = json.loads(out.strip().splitlines()[-1])
            res[v] += d["ms"]
            meta[v] = (d["launch"], d["evals"])
    for v in variants:
        med = statistics.median(res[v])
        launch, evals = meta[v]
        print(f"{v:44s} median {med:8.3f} ms  {evals / (med / 1e3) / 1e6:8.2f} M evals/s  min {min(res[v]):8.3f}  {launch}")


if __name__ == "__main__":
    main()
