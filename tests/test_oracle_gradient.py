"""Pins for the oracle's gene gradient (O-4; Gtrans/Grigidrot/Grotbond P:L83).

Central finite differences (5-point stencil, error O(h^4)) on every gene of
synthetic ligands, away from the non-smooth points (grid-cell faces,
smoothing-band edges, cutoffs), at relative error <= 1e-6."""
import numpy as np
import pytest

from oracle import oracle as O
from tests.util import ff_default


def _fd(L, G, ff, g, k, h):
    def f(d):
        x = g.copy()
        x[k] += d
        return O.eval_one(L, G, ff, x)[0]
    return (-f(2 * h) + 8 * f(h) - 8 * f(-h) + f(-2 * h)) / (12 * h)


@pytest.mark.parametrize("which,npose", [("cfg1", 12), ("cfg2", 8), ("cfg3", 3)])
def test_finite_difference_all_genes(which, npose, request):
    w = request.getfixturevalue(which)
    L, G, ff = w.ligands[0], w.grid, ff_default()
    checked = 0
    worst = 0.0
    for p in range(len(w.genes)):
        g = w.genes[p].astype(np.float64)[:L.n_genes]
        E, grad, aux, agrad, X = O.eval_one(L, G, ff, g)
        if aux[O.AUX_MARGIN_E] < 2e-4 or aux[O.AUX_MARGIN_G] < 2e-4 or abs(E) > 1e4:
            continue
        for k in range(L.n_genes):
            fd = _fd(L, G, ff, g, k, 1e-4)
            scale = max(abs(grad[k]), 1e-2 * np.linalg.norm(grad), 1e-6)
            rel = abs(fd - grad[k]) / scale
            worst = max(worst, rel)
            assert rel <= 1e-6, (p, k, fd, grad[k])
        checked += 1
        if checked == npose:
            break
    assert checked == npose
    print(f"{which}: worst relative FD error {worst:.2e}")


def test_alpha_zero_axis_genes_have_zero_gradient(cfg2):
    """At alpha = 0 the rotation is the identity for every axis (phi, theta)."""
    L, G, ff = cfg2.ligands[0], cfg2.grid, ff_default()
    for p in range(5):
        g = cfg2.genes[p].astype(np.float64)[:L.n_genes]
        g[5] = 0.0
        E, grad, *_ = O.eval_one(L, G, ff, g)
        assert grad[3] == 0.0 and grad[4] == 0.0
