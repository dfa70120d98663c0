"""Small invocations of every kernel family of libad, one per case, for
compute-sanitizer (racecheck / synccheck / memcheck / initcheck; VERDICT r01
"Sanitizer gate").  python tools/sanitize_cases.py CASE[:K=V,...] ...

Cases cover every engine (simt, tc, tc_fp16, paper, paper_tcec), every
pair-loop mode (cherry records in shared memory, scatter with the schedule in
shared or global memory, pre-decoded global-memory places, owner, hybrid:
selected through libad's A/B environment knobs, which sanitize.sh sets per
case), scoring with and without gradients, a multi-ligand screen launch,
ad_lga_run and ad_reduce_blocks.  Workloads are cut to a few poses and
iterations so that racecheck finishes in minutes; the code paths are those of
the full runs.
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_solis_vasquezts25_b200 import ad, synth  # noqa: E402

CASES = ["score_c1_grad", "score_c1_energy", "score_c2_grad",
         "ls_c2_simt", "ls_c2_tc", "ls_c2_tc_fp16", "ls_c2_paper", "ls_c2_paper_tcec",
         "ls_c1_simt", "ls_c3_simt", "ls_c3_tc", "ls_c3_paper",
         "screen", "lga", "reduce"]


def ls(cfg, engine, n, iters=3, wpc=0):
    w = synth.make_config(cfg)
    ctx = ad.Context(0)
    ctx.upload_grid(w.grid)
    lid = ctx.upload_ligand(w.ligands[0], w.ff)
    g = torch.from_numpy(w.genes[:n].copy()).cuda()
    pop = 16 if n % 16 == 0 else 0
    out = ctx.local_search(lid, g, max_iters=iters, engine=engine, pop_per_run=pop,
                           warps_per_cta=(64 if engine.startswith("paper") else wpc), trace=True)
    torch.cuda.synchronize()
    ctx.sync()
    assert torch.isfinite(out["best_energy"]).all() or engine == "tc_fp16"
    ctx.close()


def score(cfg, grad, n):
    w = synth.make_config(cfg)
    ctx = ad.Context(0)
    ctx.upload_grid(w.grid)
    lid = ctx.upload_ligand(w.ligands[0], w.ff)
    E, G, A = ctx.score(lid, torch.from_numpy(w.genes[:n].copy()).cuda(), grad=grad, aux=True)
    torch.cuda.synchronize()
    ctx.sync()
    ctx.close()


def main(case):
    if case == "score_c1_grad":
        score(1, True, 64)
    elif case == "score_c1_energy":
        score(1, False, 64)
    elif case == "score_c2_grad":
        score(2, True, 32)
    elif case.startswith("ls_c"):
        cfg = int(case[4])
        engine = case[6:]
        ls(cfg, engine, 32 if cfg != 3 else 16, iters=3 if cfg != 3 else 2)
    elif case == "screen":
        from paper_conf_sc_solis_vasquezts25_b200 import screen
        spec = synth.ScreenSpec(n_ligands=6, runs=2, pop=8, iters=2)
        ligs = [spec.ligand(k) for k in range(spec.n_ligands)]
        genes = np.concatenate([spec.genes(k) for k in range(spec.n_ligands)])
        ctx = ad.Context(0)
        ctx.upload_grid(spec.grid)
        rec, _ = screen.run_screen(ctx, spec.grid, synth.FFParams(), ligs, genes, spec.runs, spec.pop, spec.iters,
                                   n_buckets=2)
        torch.cuda.synchronize()
        ctx.close()
    elif case == "lga":
        w = synth.make_config(1)
        ctx = ad.Context(0)
        ctx.upload_grid(w.grid)
        lid = ctx.upload_ligand(w.ligands[0], w.ff)
        pop, runs = 16, 2
        g = torch.from_numpy(w.genes[:pop * runs].copy()).cuda()
        ctx.lga(lid, g, runs, pop_size=pop, max_gens=2, max_evals=10 ** 9, ls_iters=2)
        torch.cuda.synchronize()
        ctx.sync()
        ctx.close()
    elif case == "reduce":
        ctx = ad.Context(0)
        x = torch.from_numpy(synth.make_reduction_partials(7, 4, 256, 40, "uniform")).cuda()
        out = torch.empty(4, 40, dtype=torch.float32, device="cuda")
        for eng in ("simt", "tc", "paper", "tc_fp16"):
            ad.ad_reduce_blocks(ctx.h, ad.ENGINES[eng], x, out)
        torch.cuda.synchronize()
        ctx.close()
    else:
        raise SystemExit(f"unknown case {case}; one of {CASES}")
    print("case ok", case)


if __name__ == "__main__":
    # CASE or CASE:KEY=VAL,KEY=VAL (libad reads its A/B knobs when a context is
    # created or a grid uploaded, so one process can run many cases)
    for spec in sys.argv[1:]:
        case, _, env = spec.partition(":")
        saved = {}
        for kv in filter(None, env.split(",")):
            k, v = kv.split("=")
            saved[k] = os.environ.get(k)
            os.environ[k] = v
        print("=== case", spec, flush=True)
        main(case)
        for k, v in saved.items():
            if v is None:
                os.environ.pop(k)
            else:
                os.environ[k] = v
