"""Exploratory GPU run: dump libad outputs on seeded inputs to an .npz for
offline comparison against the oracle (which runs on the CPU side)."""
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_solis_vasquezts25_b200 import ad, synth  # noqa: E402

out = {}
torch.cuda.init()
ctx = ad.Context(0)


def ev_time(fn, reps=3):
    ts = []
    for _ in range(reps):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        s.record()
        fn()
        e.record()
        torch.cuda.synchronize()
        ts.append(s.elapsed_time(e))
    return ts


os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
for cfg, nscore, nls, ls_iters in ((1, 256, 64, 50), (2, 512, 64, 300), (3, 256, 16, 60)):
    w = synth.make_config(cfg)
    L = w.ligands[0]
    ctx.upload_grid(w.grid)
    lid = ctx.upload_ligand(L, w.ff)
    q = ad.ad_query(ctx.h, lid)
    print(f"cfg{cfg}: N={L.n_atoms} T={L.n_tors} P={L.n_pairs} query={q}", flush=True)
    g = torch.from_numpy(w.genes[:nscore]).cuda()
    E, G, A = ctx.score(lid, g, grad=True, aux=True)
    E0, _, _ = ctx.score(lid, g, grad=False)
    out[f"c{cfg}_score_E"] = E.cpu().numpy()
    out[f"c{cfg}_score_E_nograd"] = E0.cpu().numpy()
    out[f"c{cfg}_score_G"] = G.cpu().numpy()
    out[f"c{cfg}_score_A"] = A.cpu().numpy()
    for eng in ("simt", "tc", "paper"):
        g2 = torch.from_numpy(w.genes[:nls]).cuda()
        r = ctx.local_search(lid, g2, max_iters=ls_iters, engine=eng, trace=True,
                             warps_per_cta=(64 if eng == "paper" else 0))
        torch.cuda.synchronize()
        out[f"c{cfg}_ls_{eng}_trace"] = r["trace"].cpu().numpy()
        out[f"c{cfg}_ls_{eng}_bestE"] = r["best_energy"].cpu().numpy()
        out[f"c{cfg}_ls_{eng}_genes"] = g2.cpu().numpy()
    np.savez_compressed(os.path.join(ROOT, "gpurun_out", "probe.npz"), **out)
    # throughput of the full workload
    full = torch.from_numpy(w.genes).cuda()
    n = full.shape[0]
    iters = w.iters if cfg != 1 else 300
    for eng, wpc in (() if "--perf" not in sys.argv else (("simt", 0), ("tc", 0), ("paper", 64), ("paper", 128))):
        if cfg == 3 and eng == "paper" and wpc == 64:
            pass
        gg = full.clone()

        def run():
            ctx.local_search(lid, gg, max_iters=iters, engine=eng, warps_per_cta=wpc)
        try:
            run()
            ts = ev_time(run, 2)
            evs = n * iters / (min(ts) / 1e3)
            print(f"  cfg{cfg} {eng:5s} w={wpc}: {min(ts):8.2f} ms  {evs / 1e6:9.2f} M evals/s", flush=True)
            out[f"c{cfg}_perf_{eng}_{wpc}_ms"] = np.array(ts)
        except Exception as ex:  # noqa: BLE001
            print(f"  cfg{cfg} {eng} w={wpc}: FAILED {ex}", flush=True)

# reduction microbench
for P in (128, 1024):
    for Cc in (8, 40):
        x = torch.from_numpy(synth.make_reduction_partials(0, 148 * 8, P, Cc, "logmag")).cuda()
        for eng in ("simt", "tc", "paper"):
            o = torch.empty(x.shape[0], Cc, device="cuda")
            try:
                ad.ad_reduce_blocks(ctx.h, ad.ENGINES[eng], x, o)
            except Exception as ex:  # noqa: BLE001
                print("reduce failed", P, Cc, eng, ex, flush=True)
                continue
            torch.cuda.synchronize()
            out[f"red_{P}_{Cc}_{eng}"] = o.cpu().numpy()
            ts = ev_time(lambda: ad.ad_reduce_blocks(ctx.h, ad.ENGINES[eng], x, o), 3)
            print(f"reduce P={P} C={Cc} {eng}: {min(ts) * 1e3:.1f} us", flush=True)
ctx.close()
os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
np.savez_compressed(os.path.join(ROOT, "gpurun_out", "probe.npz"), **out)
print("saved")
