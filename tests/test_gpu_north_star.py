"""The north_star tolerance taken literally (DESIGN.md
"Tolerances"), on the CUDA path through the C ABI against the FP64 oracle.

* Relaxed poses (the genotypes the ADADELTA search returns) of configs 2
  and 3 with A_E < 500: plain |dE| <= 1e-3 kcal/mol and ||dg|| / ||g|| <= 1e-4
  on every pose; the only excusal is an atom within 1e-4 A of a gradient kink
  (trilinear cell face, smoothing-band edge), where FP32 may legitimately land
  on the other side -- such poses are counted and must stay rare.
* Z19 (ii) free-running trajectories: GPU LS and oracle LS from identical
  starts (config 1; config-2 starts with A_E < 500) agree step by step within
  the per-step energy gate for k <= 20, up to the first kink contact of the
  oracle trajectory (after it the two may take different sides: legitimate
  divergence, counted).  FP32 vs FP64 trajectories of a chaotic map cannot all
  agree for a fixed horizon: the FP64 oracle itself, restarted from its start
  genotype moved by one FP32 ulp, leaves the gate within 20 steps for 10-35 %
  of relaxed config-2 starts (tools/accuracy_report.py).
  So the k <= 20 gate is statistical: at most 5 % of the trajectories may leave
  it before a kink contact (each is reported), and the median first
  divergence must be beyond k = 20.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from oracle import oracle as O  # noqa: E402
from tests import parity as P  # noqa: E402

pytestmark = pytest.mark.gpu
KINK = 1e-4


@pytest.fixture(scope="module")
def ctx():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_solis_vasquezts25_b200 import ad
    c = ad.Context(0)
    yield c
    c.close()


def _relax(ctx, w, n):
    ctx.upload_grid(w.grid)
    lid = ctx.upload_ligand(w.ligands[0], w.ff)
    g = torch.from_numpy(w.genes[:n].copy()).cuda()
    ctx.local_search(lid, g, max_iters=w.iters, engine="simt")
    torch.cuda.synchronize()
    relaxed = g.cpu().numpy()
    E, G, _ = ctx.score(lid, torch.from_numpy(relaxed).cuda(), grad=True)
    torch.cuda.synchronize()
    return lid, relaxed, E.cpu().numpy(), G.cpu().numpy()


@pytest.mark.parametrize("which,n", [("cfg2", 512), ("cfg3", 192)])
def test_relaxed_sane_poses_meet_north_star(ctx, which, n, request):
    w = request.getfixturevalue(which)
    L = w.ligands[0]
    Gn = L.n_genes
    _, relaxed, E, G = _relax(ctx, w, n)
    Eo, Go, aux, ag = O.score(L, w.grid, w.ff, relaxed)
    sane = P.sane(aux)
    assert sane.sum() >= 16, f"only {sane.sum()} sane relaxed poses"
    dE = np.abs(E.astype(np.float64) - Eo)
    rel = P.rel_grad_err(G[:, :Gn], Go[:, :Gn])
    kink = aux[:, O.AUX_MARGIN_G] < KINK
    okE, okG = dE <= 1e-3, rel <= 1e-4
    bad = sane & ~(okE & (okG | kink))
    assert not bad.any(), (f"{which}: {bad.sum()} sane relaxed poses outside the plain north_star gate: "
                           f"max dE {dE[sane].max():.3e}, max rel grad {rel[sane & ~kink].max():.3e}")
    assert (sane & kink & ~okG).sum() <= max(1, int(0.02 * sane.sum()))
    # every pose (sane or not) inside the Z18 gates
    assert np.all(P.energy_gate(E, Eo, aux))
    assert np.all(P.grad_gate(G[:, :Gn], Go[:, :Gn], ag[:, :Gn]) | kink)


@pytest.mark.parametrize("which,n,only_sane", [("cfg1", 64, False), ("cfg2", 256, True)])
def test_free_running_trajectories(ctx, which, n, only_sane, request):
    w = request.getfixturevalue(which)
    L = w.ligands[0]
    K = 20
    starts = w.genes[:n].copy()
    if only_sane:
        _, _, aux0, _ = O.score(L, w.grid, w.ff, starts)
        starts = starts[P.sane(aux0)]
        assert len(starts) >= 16
    ctx.upload_grid(w.grid)
    lid = ctx.upload_ligand(L, w.ff)
    g = torch.from_numpy(starts.copy()).cuda()
    out = ctx.local_search(lid, g, max_iters=K, engine="simt", trace=True)
    torch.cuda.synchronize()
    tE = out["trace"][:, :, 0].cpu().numpy().astype(np.float64)
    _, _, otr = O.local_search(L, w.grid, w.ff, starts, max_iters=K, trace=True)
    aux = np.zeros(otr.shape[:2] + (O.AUX_N,))
    aux[..., O.AUX_ABS_E], aux[..., O.AUX_SENS_E] = otr[..., 1], otr[..., 2]
    bad = np.abs(tE - otr[..., 0]) > P.energy_tol(aux)
    first_bad = np.where(bad.any(1), bad.argmax(1), K)
    # contact with a gradient kink at step j can change step j + 1 (the ADADELTA
    # update), one with an energy discontinuity changes step j itself
    kink = np.zeros((len(starts), K), dtype=bool)
    kink[:, 1:] = otr[:, :-1, 4] < KINK
    kink |= otr[..., 3] < KINK
    first_kink = np.where(kink.any(1), kink.argmax(1), K)
    unexplained = (first_bad < K) & (first_bad < first_kink)
    print(f"{which}: {len(starts)} trajectories, {(first_bad < K).sum()} leave the gate within {K} steps, "
          f"{unexplained.sum()} before a kink contact (poses {np.nonzero(unexplained)[0].tolist()}, "
          f"steps {first_bad[unexplained].tolist()})")
    assert unexplained.mean() <= 0.05, f"{which}: {unexplained.sum()} of {len(starts)} leave the gate before a kink"
    assert np.median(first_bad) >= K
    assert (first_bad < K).mean() <= 0.25, f"{which}: {(first_bad < K).sum()} of {len(starts)} diverge within {K} steps"
