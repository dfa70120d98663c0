"""Pins for the oracle's ADADELTA (O-6; Alg 3; Zeiler [19] P:L406),
best-of-run (O-8) and exact reduction (O-7; Eq 1-5)."""
import json
import math
import os

import numpy as np

from oracle import oracle as O
from tests.util import ff_default

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def test_first_adadelta_step_closed_form():
    # E[g^2]_1 = (1-rho) g^2, E[dx^2]_0 = 0  =>  dx_1 = -g sqrt(eps) / sqrt((1-rho) g^2 + eps)
    rho, eps = 0.8, 0.01
    g = 3.7
    eg2, ed2, x = O.adadelta_step([g], [0.0], [0.0], [1.0], rho, eps)
    assert abs((x[0] - 1.0) - (-0.22319963)) < 1e-7            # = -0.37 / sqrt(2.748)
    assert abs(eg2[0] - 0.2 * 13.69) < 1e-12
    assert abs(ed2[0] - 0.2 * 0.22319963 ** 2) < 1e-8
    # second step with the same gradient, closed form
    eg2b, ed2b, x2 = O.adadelta_step([g], eg2, ed2, x, rho, eps)
    e1 = 0.8 * 2.738 + 0.2 * 13.69
    d2 = -g * math.sqrt(ed2[0] + eps) / math.sqrt(e1 + eps)
    assert abs((x2[0] - x[0]) - d2) < 1e-12
    # zero gradient -> no move, decaying state
    eg2c, ed2c, x3 = O.adadelta_step([0.0], [1.0], [2.0], [5.0], rho, eps)
    assert x3[0] == 5.0 and abs(eg2c[0] - 0.8) < 1e-15 and abs(ed2c[0] - 1.6) < 1e-15


def test_local_search_composition_and_best_tracking(cfg1):
    L, G, ff = cfg1.ligands[0], cfg1.grid, ff_default()
    genes = cfg1.genes[:6]
    iters = 25
    best, bE = O.local_search(L, G, ff, genes, max_iters=iters, threads=2)
    for p in range(len(genes)):
        x = genes[p].astype(np.float64)[:L.n_genes]
        eg2 = np.zeros_like(x)
        ed2 = np.zeros_like(x)
        traj = []
        for _ in range(iters):
            E, grad, *_ = O.eval_one(L, G, ff, x)
            traj.append((E, x.copy()))
            eg2, ed2, x = O.adadelta_step(grad, eg2, ed2, x)
        Es = [e for e, _ in traj]
        k = int(np.argmin(Es))                      # first minimum: strict < keeps the earliest
        assert bE[p] == Es[k]
        assert np.array_equal(best[p, :L.n_genes], traj[k][1])
        assert bE[p] <= Es[0]


def test_best_of_run_ties_lowest_index():
    E = np.array([3.0, 1.0, 1.0, 2.0, 5.0, 5.0, 5.0, 5.0, -1.0, 0.0, -1.0, 7.0])
    assert O.best_of_run(E, 4).tolist() == [1, 4, 8]
    rng = np.random.default_rng(0)
    E = rng.integers(0, 5, 600).astype(float)
    got = O.best_of_run(E, 150)
    assert got.tolist() == [r * 150 + int(np.argmin(E[r * 150:(r + 1) * 150])) for r in range(4)]


def test_exact_sum_matches_fsum():
    rng = np.random.default_rng(1)
    for _ in range(20):
        x = (10.0 ** rng.uniform(-4, 4, 1000) * rng.choice([-1, 1], 1000)).astype(np.float32)
        assert O.exact_sum(x) == math.fsum(x.astype(np.float64))
    x = np.array([1e30, 1.0, -1e30, 1e-30], np.float32)
    assert O.exact_sum(x) == math.fsum(x.astype(np.float64))
    xi = rng.integers(-1000, 1000, 5000).astype(np.float32)
    assert O.exact_sum(xi) == float(xi.astype(np.int64).sum())


def test_eq1_tensor_core_tile_algebra():
    """Eq 1-4: A P sums rows, Q V folds rows mod 4; W[0:4,0] = totals."""
    meta = json.load(open(os.path.join(GOLDEN, "eq1_reduction_tile.json")))
    rng = np.random.default_rng(meta["vectors_seed"])
    vec = rng.integers(-50, 50, size=(64, 4)).astype(np.float64)    # {x, y, z, e}
    A = np.zeros((16, 16))
    for c in range(16):
        for j in range(4):
            A[4 * j:4 * j + 4, c] = vec[4 * c + j]
    P = np.ones((16, 16))
    Q = np.kron(np.ones((4, 4)), np.eye(4))
    W = Q @ (A @ P)
    assert np.array_equal(W[0:4, 0], vec.sum(0))
    assert np.all(W == W[:, :1])                                     # every column equal


def test_amdahl_tab5_golden():
    from paper_conf_sc_solis_vasquezts25_b200.report import amdahl_speedup
    meta = json.load(open(os.path.join(GOLDEN, "tab5_amdahl.json")))
    for row in meta["rows"]:
        assert abs(amdahl_speedup(row["f_eff"], row["S"]) - row["predicted"]) <= meta["tolerance_abs"], row
