"""A14: per-phase cycle shares of the ADADELTA kernel from the instrumented
build (ad_ls_params.phase_cycles), per engine and config, and the paper's Amdahl
reading of them (Eq 6): f = reduction cycles / kernel cycles; the
speedup a reduction engine S times faster would give is 1 / (f / S + 1 - f).
usage: python tools/phases.py [out.json] [configs, default 2,3]"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_solis_vasquezts25_b200 import ad, report, synth  # noqa: E402

PHASES = ("pose_inter", "intra", "assemble", "reduce", "update")


def main():
    out_path = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/phases.json"
    cfgs = [int(c) for c in (sys.argv[2] if len(sys.argv) > 2 else "2,3").split(",")]
    res = {"phases": PHASES, "configs": {}}
    for cfg in cfgs:
        w = synth.make_config(cfg)
        ctx = ad.Context(0)
        ctx.upload_grid(w.grid)
        lid = ctx.upload_ligand(w.ligands[0], w.ff)
        rows = {}
        for eng in ("simt", "tc", "paper", "paper_tcec"):
            wpc = 64 if eng.startswith("paper") else 0
            if eng.startswith("paper") and 6 + w.ligands[0].n_tors > 64:
                continue
            g = torch.from_numpy(w.genes).cuda()
            out = ctx.local_search(lid, g, max_iters=w.iters, engine=eng, warps_per_cta=wpc, phases=True)
            torch.cuda.synchronize()
            ph = out["phase_cycles"].cpu().numpy().astype(np.float64)
            tot = ph.sum(axis=1)
            share = ph.sum(axis=0) / tot.sum()
            f = float(share[PHASES.index("reduce")])
            rows[eng] = {"share": dict(zip(PHASES, map(float, share))), "f": f,
                         "cycles_per_eval_per_pose": float(tot.mean() / w.iters),
                         "amdahl_bound_S_inf": 1.0 / (1.0 - f),
                         "amdahl_S_4": report.amdahl_speedup(f, 4.0)}
            print(cfg, eng, {k: round(v, 3) for k, v in rows[eng]["share"].items()}, "f=%.3f" % f, flush=True)
        res["configs"][f"config{cfg}"] = rows
        ctx.close()
    os.makedirs(os.path.dirname(out_path) or ".", exist_ok=True)
    with open(out_path, "w") as fh:
        json.dump(res, fh, indent=1)


if __name__ == "__main__":
    main()
