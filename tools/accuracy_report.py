"""Host side of the accuracy probe: the FP64 oracle on the genotypes the GPU
probe evaluated (tools/accuracy_probe.py), Z18 gates and plain north_star
metrics per config / pose kind / engine, and the Z19 (ii) free-running
trajectory comparison.  Prints a table; --json writes the summary."""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from oracle import oracle as O  # noqa: E402
from paper_conf_sc_solis_vasquezts25_b200 import synth  # noqa: E402
from tests import parity as P  # noqa: E402

KINK = 1e-4


def summarize(L, Eo, Go, aux, ag, E, G):
    Gn = L.n_genes
    Go, ag, G = Go[:, :Gn], ag[:, :Gn], G[:, :Gn].astype(np.float64)
    dE = np.abs(E.astype(np.float64) - Eo)
    sane = P.sane(aux)
    kinkG = aux[:, O.AUX_MARGIN_G] < KINK
    kinkE = aux[:, O.AUX_MARGIN_E] < KINK
    rel = P.rel_grad_err(G, Go)
    relz = P.rel_grad_err(G, Go, ag)
    okE = P.energy_gate(E, Eo, aux)
    okG = P.grad_gate(G, Go, ag)
    d = np.abs(G - Go)
    grp = {"trans": slice(0, 3), "orient": slice(3, 6), "tors": slice(6, Gn)}
    out = {
        "n": int(len(E)), "n_sane": int(sane.sum()), "n_kinkG": int(kinkG.sum()), "n_kinkE": int(kinkE.sum()),
        "energy_gate_pass": float(okE.mean()), "grad_gate_pass": float(okG.mean()),
        "energy_fail_not_kink": int((~okE & ~kinkE).sum()), "grad_fail_not_kink": int((~okG & ~kinkG & ~kinkE).sum()),
    }
    if sane.any():
        s = sane
        out.update({
            "sane_max_dE": float(dE[s].max()), "sane_p99_dE": float(np.quantile(dE[s], 0.99)),
            "sane_frac_dE_le_1e-3": float((dE[s] <= 1e-3).mean()),
            "sane_max_rel_g": float(rel[s].max()), "sane_med_rel_g": float(np.median(rel[s])),
            "sane_frac_rel_g_le_1e-4": float((rel[s] <= 1e-4).mean()),
            "sane_nokink_max_rel_g": float(rel[s & ~kinkG].max()) if (s & ~kinkG).any() else None,
            "sane_nokink_frac_rel_g_le_1e-4": float((rel[s & ~kinkG] <= 1e-4).mean()) if (s & ~kinkG).any() else None,
            "sane_max_relz_g": float(relz[s].max()),
            "sane_med_AE": float(np.median(aux[s, O.AUX_ABS_E])),
            "sane_med_Agrad_over_g": float(np.median(np.linalg.norm(ag[s], axis=1) / np.linalg.norm(Go[s], axis=1))),
        })
        worst = np.argsort(-rel * s)[:3]
        out["sane_worst"] = [{
            "i": int(i), "rel_g": float(rel[i]), "dE": float(dE[i]), "A_E": float(aux[i, O.AUX_ABS_E]),
            "g": float(np.linalg.norm(Go[i])), "margin_g": float(aux[i, O.AUX_MARGIN_G]),
            **{k: float(np.linalg.norm(d[i, v])) for k, v in grp.items()}} for i in worst]
        worstE = np.argsort(-dE * s)[:3]
        out["sane_worstE"] = [{"i": int(i), "dE": float(dE[i]), "A_E": float(aux[i, O.AUX_ABS_E]),
                               "S_E": float(aux[i, O.AUX_SENS_E]), "margin_e": float(aux[i, O.AUX_MARGIN_E]),
                               "E": float(Eo[i])} for i in worstE]
    out["max_dE"] = float(dE.max())
    out["max_relz_g"] = float(relz.max())
    return out


def trajectories(L, w, starts, trace, aux0):
    """Z19 (ii): GPU free-running trace energies vs the oracle's from the same starts."""
    n, iters = trace.shape[:2]
    _, _, otr = O.local_search(L, w.grid, w.ff, starts, max_iters=iters, trace=True)
    tE = otr[..., 0]
    gE = trace[:, :, 0].astype(np.float64)
    dE = np.abs(gE - tE)
    aux = np.zeros(otr.shape[:2] + (O.AUX_N,))
    aux[..., O.AUX_ABS_E], aux[..., O.AUX_SENS_E] = otr[..., 1], otr[..., 2]
    bad = dE > P.energy_tol(aux)
    first = np.where(bad.any(1), bad.argmax(1), iters)
    # gradient kink at step j changes step j + 1; energy discontinuity at step j changes step j
    kink = np.zeros_like(otr[..., 0], dtype=bool)
    kink[:, 1:] = otr[:, :-1, 4] < KINK
    kink |= otr[..., 3] < KINK
    fkink = np.where(kink.any(1), kink.argmax(1), iters)
    unexplained = (first < 20) & (first < fkink)
    return {
        "n_diverged_k20": int((first < 20).sum()), "n_diverged_k20_no_prior_kink": int(unexplained.sum()),
        "unexplained_poses": [int(i) for i in np.nonzero(unexplained)[0]],
        "n": int(n), "iters": int(iters),
        "first_divergence_median": float(np.median(first)), "first_divergence_p5": float(np.quantile(first, 0.05)),
        "first_divergence_min": int(first.min()), "frac_within_k20": float((first >= 20).mean()),
        "best_E_gpu_median": float(np.median(gE.min(1))), "best_E_oracle_median": float(np.median(tE.min(1))),
        "best_E_abs_diff_median": float(np.median(np.abs(gE.min(1) - tE.min(1)))),
    }, first


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("npz")
    ap.add_argument("--json")
    ap.add_argument("--no-traj", action="store_true")
    a = ap.parse_args()
    z = np.load(a.npz)
    rep = {}
    for cfg in (1, 2, 3):
        w = synth.make_config(cfg)
        L = w.ligands[0]
        for kind in ("relaxed", "start"):
            key = f"c{cfg}_{kind}_score_E"
            if key not in z:
                continue
            n = len(z[key])
            genes = (z[f"c{cfg}_relaxed"] if kind == "relaxed" else w.genes)[:n]
            Eo, Go, aux, ag = O.score(L, w.grid, w.ff, genes)
            for eng in ("score", "simt", "tc", "paper", "paper_tcec"):
                E, G = z[f"c{cfg}_{kind}_{eng}_E"], z[f"c{cfg}_{kind}_{eng}_G"]
                if eng == "score":
                    E, G = z[f"c{cfg}_{kind}_score_E"], z[f"c{cfg}_{kind}_score_G"]
                s = summarize(L, Eo, Go, aux, ag, E, G)
                rep[f"c{cfg}/{kind}/{eng}"] = s
                print(f"c{cfg} {kind:8s} {eng:10s} n={s['n']:5d} sane={s['n_sane']:5d} "
                      f"Epass={s['energy_gate_pass']:.4f} Gpass={s['grad_gate_pass']:.4f} "
                      f"Efail!k={s['energy_fail_not_kink']} Gfail!k={s['grad_fail_not_kink']} "
                      + (f"sane: maxdE={s['sane_max_dE']:.2e} f(dE<=1e-3)={s['sane_frac_dE_le_1e-3']:.4f} "
                         f"maxrel={s['sane_max_rel_g']:.2e} f(rel<=1e-4)={s['sane_frac_rel_g_le_1e-4']:.4f} "
                         f"nokink maxrel={s['sane_nokink_max_rel_g']}" if s['n_sane'] else ""))
            if not a.no_traj and f"c{cfg}_{kind}_trace" in z:
                tr = z[f"c{cfg}_{kind}_trace"]
                st = genes[:len(tr)]
                _, _, aux0, _ = O.score(L, w.grid, w.ff, st)
                t, first = trajectories(L, w, st, tr, aux0[:, O.AUX_ABS_E])
                t["n_sane_start"] = int(P.sane(aux0).sum())
                rep[f"c{cfg}/{kind}/traj"] = t
                print(f"c{cfg} {kind:8s} traj {t}")
    if a.json:
        with open(a.json, "w") as f:
            json.dump(rep, f, indent=1)


if __name__ == "__main__":
    main()
