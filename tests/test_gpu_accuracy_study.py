"""NEXT-2 accuracy study: FP32 SIMT vs error-corrected TF32 (TCEC) vs FP16 without
EC (Schieffer-Peng, Lst 1 bottom P:L236-258) reductions inside the same ADADELTA
local search (config 2 workload, synthetic).  Measures
  (a) per-evaluation energy / gradient error vs the FP64 oracle on relaxed poses,
  (b) per-run best energies after the full LS vs the SIMT engine: median |dE|,
      fraction worse by > 1 kcal/mol (the paper's score-success threshold),
      non-finite runs,
  (c) the config-4 reduction error of each engine vs math.fsum,
and asserts the qualitative Fig 1 vs Fig 3 finding: the
error-corrected TF32 engine matches FP32 SIMT, the uncorrected FP16 engine does not.
The report is written as JSON to $AD_STUDY_OUT when set (profiles/accuracy_*.json):
    AD_STUDY_OUT=profiles/accuracy_r01.json python -m pytest tests/test_gpu_accuracy_study.py -m gpu -s
"""
import json
import math
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")

from oracle import oracle as O  # noqa: E402
from paper_conf_sc_solis_vasquezts25_b200 import synth  # noqa: E402

pytestmark = pytest.mark.gpu

ENG = ("simt", "tc", "tc_fp16")


def test_accuracy_study():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_solis_vasquezts25_b200 import ad
    w = synth.make_config(2)
    L = w.ligands[0]
    Gn, stride = L.n_genes, w.genes.shape[1]
    ctx = ad.Context(0)
    ctx.upload_grid(w.grid)
    lid = ctx.upload_ligand(L, w.ff)
    res = {"workload": "config2 (40 atoms, 8 torsions), 20 runs x 150 pop x 300 iterations", "engines": list(ENG)}
    # (b) full LS per engine from the same starts
    best = {}
    for e in ENG:
        g = torch.from_numpy(w.genes).cuda()
        out = ctx.local_search(lid, g, max_iters=w.iters, engine=e, pop_per_run=w.pop)
        torch.cuda.synchronize()
        best[e] = out["run_best"].cpu().numpy()[:, 0].astype(np.float64)
    runs = {}
    for e in ENG:
        d = best[e] - best["simt"]
        fin = np.isfinite(best[e])
        runs[e] = {"median_best_E": float(np.median(best[e][fin])) if fin.any() else None,
                   "median_abs_dE_vs_simt": float(np.median(np.abs(d[fin]))) if fin.any() else None,
                   "frac_worse_by_1kcal": float(np.mean(~fin | (d > 1.0))),
                   "non_finite_runs": int((~fin).sum())}
    res["run_best"] = runs
    # (a) per-evaluation error on relaxed poses (the TC engine's LS best genes)
    n = 256
    g = torch.from_numpy(w.genes[:n]).cuda()
    ctx.local_search(lid, g, max_iters=w.iters, engine="tc")
    relaxed = g.cpu().numpy()
    Eo, Go, aux, _ = O.score(L, w.grid, w.ff, relaxed)
    per = {}
    for e in ENG:
        gg = torch.from_numpy(relaxed).cuda()
        out = ctx.local_search(lid, gg, max_iters=1, engine=e, trace=True)
        tr = out["trace"].cpu().numpy()[:, 0]
        dE = np.abs(tr[:, 0].astype(np.float64) - Eo)
        gr = tr[:, 1 + stride:1 + stride + Gn].astype(np.float64)
        rel = np.linalg.norm(gr - Go[:, :Gn], axis=1) / np.maximum(np.linalg.norm(Go[:, :Gn], axis=1), 1e-6)
        fin = np.isfinite(dE) & np.isfinite(rel)
        per[e] = {"median_abs_dE": float(np.median(dE[fin])), "p95_abs_dE": float(np.percentile(dE[fin], 95)),
                  "median_grad_rel_err": float(np.median(rel[fin])),
                  "p95_grad_rel_err": float(np.percentile(rel[fin], 95)),
                  "non_finite_evals": int((~fin).sum()), "n": int(len(fin))}
    res["per_eval_relaxed_poses"] = per
    # (c) config-4 reduction accuracy
    red = {}
    x = synth.make_reduction_partials(7, 256, 256, 16, "uniform")
    ex = np.array([[math.fsum(x[b, :, c].astype(np.float64)) for c in range(16)] for b in range(256)])
    for e in ("simt", "tc", "tc_fp16", "paper"):
        o = torch.empty(256, 16, device="cuda")
        ad.ad_reduce_blocks(ctx.h, ad.ENGINES[e], torch.from_numpy(x).cuda(), o)
        torch.cuda.synchronize()
        err = np.abs(o.cpu().numpy().astype(np.float64) - ex)
        red[e] = {"median_abs_err": float(np.median(err)), "max_abs_err": float(err.max())}
    res["reduction_256x16_uniform"] = red
    ctx.close()
    out_path = os.environ.get("AD_STUDY_OUT")
    if out_path:
        os.makedirs(os.path.dirname(out_path) or ".", exist_ok=True)
        with open(out_path, "w") as f:
            json.dump(res, f, indent=1)
    print(json.dumps(res, indent=1))
    # the qualitative finding: TCEC ~ SIMT, FP16 without EC clearly worse
    assert red["tc"]["max_abs_err"] <= 4 * red["simt"]["max_abs_err"] + 1e-6
    assert red["tc_fp16"]["median_abs_err"] > 100 * red["tc"]["median_abs_err"]
    assert per["tc"]["median_grad_rel_err"] <= 10 * per["simt"]["median_grad_rel_err"] + 1e-7
    assert per["tc_fp16"]["median_grad_rel_err"] > 10 * per["tc"]["median_grad_rel_err"]
    assert runs["tc"]["frac_worse_by_1kcal"] <= 0.05
