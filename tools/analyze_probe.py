"""Compare gpurun_out/probe.npz (GPU outputs) against the FP64 oracle, here on the CPU."""
import math
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from oracle import oracle as O  # noqa: E402
from paper_conf_sc_solis_vasquezts25_b200 import synth  # noqa: E402
from tests.parity import energy_gate, energy_scale, grad_gate, rel_grad_err  # noqa: E402

d = np.load(os.path.join(ROOT, "gpurun_out", sys.argv[1] if len(sys.argv) > 1 else "probe.npz"))
for cfg in (1, 2, 3):
    w = synth.make_config(cfg)
    L = w.ligands[0]
    Gn = L.n_genes
    if f"c{cfg}_score_E" not in d:
        continue
    E = d[f"c{cfg}_score_E"]
    n = len(E)
    Eo, Go, aux, ag = O.score(L, w.grid, w.ff, w.genes[:n])
    okE = energy_gate(E, Eo, energy_scale(aux))
    okG = grad_gate(d[f"c{cfg}_score_G"][:, :Gn], Go[:, :Gn], ag[:, :Gn])
    rg = rel_grad_err(d[f"c{cfg}_score_G"][:, :Gn], Go[:, :Gn], ag[:, :Gn])
    dE = np.abs(E - Eo)
    kink = (aux[:, O.AUX_MARGIN_E] < 1e-4) | (aux[:, O.AUX_MARGIN_G] < 1e-4)
    print(f"cfg{cfg} score n={n}: E gate {okE.mean():.4f}  G gate {okG.mean():.4f}  max|dE| {dE.max():.3e} "
          f"median|dE| {np.median(dE):.2e}  max relG {rg.max():.2e} median relG {np.median(rg):.2e}  kink {kink.sum()}")
    bad = np.nonzero(~okE | ~okG)[0]
    for b in bad[:5]:
        print(f"   bad pose {b}: E {E[b]:.6g} oracle {Eo[b]:.6g} A_E {aux[b, 2]:.3g} relG {rg[b]:.3g} "
              f"margins {aux[b, 3]:.2e} {aux[b, 4]:.2e}")
    en = d[f"c{cfg}_score_E_nograd"]
    print(f"   energy-only == grad-mode energy: {np.array_equal(en, E)}  max diff {np.abs(en - E).max():.2e}")
    A = d[f"c{cfg}_score_A"]
    print(f"   aux E_inter max diff {np.abs(A[:, 0] - aux[:, 0]).max():.2e}  E_intra {np.abs(A[:, 1] - aux[:, 1]).max():.2e}")
    for eng in ("simt", "tc", "paper"):
        tr = d[f"c{cfg}_ls_{eng}_trace"]  # [n, iters, 1 + 2*stride]
        nls, iters, _ = tr.shape
        stride = (tr.shape[2] - 1) // 2
        genes_k = tr[:, :, 1:1 + stride].reshape(-1, stride)
        Ek = tr[:, :, 0].reshape(-1)
        gk = tr[:, :, 1 + stride:].reshape(-1, stride)
        sel = np.arange(0, nls * iters, max(1, (nls * iters) // 600))
        Eo2, Go2, aux2, ag2 = O.score(L, w.grid, w.ff, genes_k[sel])
        okE2 = energy_gate(Ek[sel], Eo2, energy_scale(aux2))
        okG2 = grad_gate(gk[sel, :Gn], Go2[:, :Gn], ag2[:, :Gn])
        # ADADELTA step from the GPU's own gradient history (fp64)
        worst_step = 0.0
        for p in range(min(nls, 8)):
            eg2 = np.zeros(Gn)
            ed2 = np.zeros(Gn)
            for k in range(iters - 1):
                x = tr[p, k, 1:1 + Gn].astype(np.float64)
                eg2, ed2, xn = O.adadelta_step(tr[p, k, 1 + stride:1 + stride + Gn], eg2, ed2, x)
                step = xn - x
                got = tr[p, k + 1, 1:1 + Gn].astype(np.float64)
                # FP32 genes: allow one rounding of x plus 1e-5 relative of the step
                err = np.abs(got - xn) / (1e-5 * np.abs(step) + 2.0 ** -23 * np.abs(xn) + 1e-30)
                worst_step = max(worst_step, err.max())
        bE = d[f"c{cfg}_ls_{eng}_bestE"]
        best_ok = np.array_equal(bE, tr[:, :, 0].min(axis=1))
        print(f"   LS {eng:5s}: per-step E gate {okE2.mean():.4f}  G gate {okG2.mean():.4f}  "
              f"max|dE| {np.abs(Ek[sel] - Eo2).max():.2e}  step rel err {worst_step:.2e}  best==min(trace) {best_ok}  "
              f"mean bestE {bE.mean():.3f}")
for key in sorted(k for k in d.files if k.startswith("red_")):
    _, P, Cc, eng = key.split("_")
    P, Cc = int(P), int(Cc)
    x = synth.make_reduction_partials(0, 148 * 8, P, Cc, "logmag")
    o = d[key]
    exact = np.array([[math.fsum(x[b, :, c].astype(np.float64)) for c in range(Cc)] for b in range(0, x.shape[0], 37)])
    absx = np.abs(x[::37].astype(np.float64)).sum(axis=1)
    err = np.abs(o[::37] - exact) / absx
    bound = (math.ceil(math.log2(P)) + 2) * 2.0 ** -24
    print(f"reduce P={P} C={Cc} {eng:5s}: max err/sum|x| = {err.max() / 2 ** -24:.2f} ulp-units (bound {bound / 2 ** -24:.0f})")
