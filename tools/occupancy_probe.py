"""LS launch time of config 2 vs the number of poses (resident warps per SM), for
the 80- and 128-register kernels: how well fewer warps hide latency.
python tools/occupancy_probe.py"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r"""
import sys, json, torch
sys.path.insert(0, %r)
from paper_conf_sc_solis_vasquezts25_b200 import ad, synth
n = int(sys.argv[1])
wl = synth.make_config(2)
ctx = ad.Context(0); ctx.upload_grid(wl.grid); lid = ctx.upload_ligand(wl.ligands[0], wl.ff)
start = torch.from_numpy(wl.genes[:n].copy()).cuda(); g = start.clone()
ts = []
for k in range(6):
    g.copy_(start)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); ctx.local_search(lid, g, max_iters=wl.iters, engine="simt"); b.record()
    torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
print(json.dumps({"n": n, "ms": sorted(ts[2:])[1], "launch": ad.ad_last_launch(ctx.h)}))
""" % ROOT
for reg in ("80", "128"):
    for n in (3000, 2220, 1500, 1480, 740):
        env = dict(os.environ, AD_MAXREG=reg)
        out = subprocess.run([sys.executable, "-c", CHILD, str(n)], env=env, capture_output=True, text=True)
        try:
            d = json.loads(out.stdout.strip().splitlines()[-1])
            print(f"regs {reg:>3} poses {n:5d}  {d['ms']:8.3f} ms  {d['ms'] / n * 1e3:7.3f} us/pose  {d['launch']}", flush=True)
        except Exception:
            print(reg, n, out.stderr[-300:])
