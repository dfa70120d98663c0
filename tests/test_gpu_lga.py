"""NEXT-3: the Lamarckian GA driver (Alg 1) on the GPU, against the
oracle's GA generation (same counter-based generator implemented on each side)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from oracle import oracle as O  # noqa: E402
from paper_conf_sc_solis_vasquezts25_b200 import synth  # noqa: E402
from tests.parity import energy_gate  # noqa: E402

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def setup():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_solis_vasquezts25_b200 import ad
    w = synth.make_config(2)
    ctx = ad.Context(0)
    ctx.upload_grid(w.grid)
    lid = ctx.upload_ligand(w.ligands[0], w.ff)
    yield ad, ctx, lid, w
    ctx.close()


KW = dict(elitism=1, cross_rate=0.8, mut_rate=0.02, tour_rate=0.6, dmov=16.0, dang=90.0)


def test_ga_generation_bit_exact(setup):
    """One generation without LS: the new population equals the oracle's GA
    generation bit for bit (selection on the GPU's own FP32 energies)."""
    ad, ctx, lid, w = setup
    L = w.ligands[0]
    runs, pop, seed = 4, 50, 1234
    g0 = w.genes[:runs * pop].copy()
    E0, _, _ = ctx.score(lid, torch.from_numpy(g0).cuda(), grad=False)
    E0 = E0.cpu().numpy()
    g = torch.from_numpy(g0).cuda()
    out = ctx.lga(lid, g, runs, pop_size=pop, max_gens=1, max_evals=10 ** 9, ls_rate=0.0, seed=seed, ls_iters=5, **KW)
    got = g.cpu().numpy()
    prm = O.ga_params(pop, L.n_genes, g0.shape[1], ls_rate=0.0, **KW)
    for r in range(runs):
        s = slice(r * pop, (r + 1) * pop)
        exp = O.ga_generation(prm, g0[s], E0[s], seed, 0, r)
        assert np.array_equal(got[s, :L.n_genes], exp[:, :L.n_genes]), r
    # the energies returned are those of the new population
    Eo, _, aux, _ = O.score(L, w.grid, w.ff, got)
    assert np.all(energy_gate(out["energies"].cpu().numpy(), Eo, aux))
    assert np.all(out["n_gens"].cpu().numpy() == 1)
    assert np.all(out["n_evals"].cpu().numpy() == 2 * pop)


def test_lga_budget_and_elitism(setup):
    """Several generations with LS: the evaluation count of every run is exactly
    pop (initial) + per generation pop + LS individuals x iterations, where the LS
    individuals are the oracle generator's coins; runs stop at the first
    generation reaching max_evals; the best energy never rises (elitism + LS)."""
    ad, ctx, lid, w = setup
    runs, pop, seed, iters = 6, 40, 77, 20
    ls_rate = 0.5
    max_evals = pop + 3 * (pop + int(0.5 * pop) * iters)  # about three generations
    g0 = w.genes[:runs * pop].copy()
    E0, _, _ = ctx.score(lid, torch.from_numpy(g0).cuda(), grad=False)
    E0 = E0.cpu().numpy()
    g = torch.from_numpy(g0).cuda()
    out = ctx.lga(lid, g, runs, pop_size=pop, max_gens=50, max_evals=max_evals, ls_rate=ls_rate, seed=seed,
                  ls_iters=iters, **KW)
    ev, gens = out["n_evals"].cpu().numpy(), out["n_gens"].cpu().numpy()
    prm = O.ga_params(pop, w.ligands[0].n_genes, g0.shape[1], ls_rate=ls_rate, **KW)
    for r in range(runs):
        e, k = pop, 0
        while e < max_evals and k < 50:
            e += pop + int(O.ls_select(prm, seed, k, r).sum()) * iters
            k += 1
        assert ev[r] == e and gens[r] == k, (r, ev[r], e, gens[r], k)
    E = out["energies"].cpu().numpy()
    rb = out["run_best"].cpu().numpy()
    for r in range(runs):
        s = slice(r * pop, (r + 1) * pop)
        assert rb[r, 0] == E[s].min() <= E0[s].min()
    # deterministic
    g2 = torch.from_numpy(g0).cuda()
    out2 = ctx.lga(lid, g2, runs, pop_size=pop, max_gens=50, max_evals=max_evals, ls_rate=ls_rate, seed=seed,
                   ls_iters=iters, **KW)
    assert torch.equal(g, g2) and torch.equal(out["energies"], out2["energies"])


def test_lga_improves_over_ls_alone(setup):
    """End to end on the config-2 receptor: a short LGA (10 generations) finds
    better run minima than the same number of start poses relaxed once by LS."""
    ad, ctx, lid, w = setup
    runs, pop = 8, 50
    g0 = w.genes[:runs * pop].copy()
    g = torch.from_numpy(g0).cuda()
    out = ctx.lga(lid, g, runs, pop_size=pop, max_gens=10, max_evals=10 ** 9, seed=5, ls_iters=100, **KW)
    gl = torch.from_numpy(g0).cuda()
    ls = ctx.local_search(lid, gl, max_iters=100, pop_per_run=pop)
    assert np.median(out["run_best"][:, 0].cpu().numpy()) < np.median(ls["run_best"][:, 0].cpu().numpy())
