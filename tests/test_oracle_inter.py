"""Pins for the oracle's InterGradient (O-2; readings Z3-Z5)."""
import numpy as np
from scipy.ndimage import map_coordinates

from oracle import oracle as O
from paper_conf_sc_solis_vasquezts25_b200.synth import Grid
from tests.util import affine_grid, ff_default, hand_ligand


def _one_atom(q, t=0, nt=1):
    return hand_ligand([[0.0, 0.0, 0.0]], types=[t], charges=[q], tp=np.zeros((nt, nt, 5)) + [0, 0, 4, 12, 6])


def _genes_at(G, u, T=0):
    g = np.zeros(6 + T)
    g[:3] = u          # translation genes are grid units
    return g


def test_affine_field_reproduced_exactly():
    # dyadic coefficients: every grid value is exact in FP32
    coefs = [(0.75, np.array([0.25, -0.125, 0.0625])),      # type map
             (-1.5, np.array([-0.5, 0.125, 0.25])),         # electrostatic
             (0.25, np.array([0.015625, 0.03125, -0.03125]))]  # desolvation
    G = affine_grid(coefs)
    ff = ff_default()
    rng = np.random.default_rng(0)
    for q in (0.37, -0.52, 0.0):
        q = float(np.float32(q))        # charges are FP32 inputs
        L = _one_atom(q)
        for _ in range(20):
            u = rng.uniform(0.0, G.nx - 1.0 - 1e-6, 3)
            E, grad, aux, _, X = O.eval_one(L, G, ff, _genes_at(G, u))
            w = [1.0, q, abs(q)]
            want_E = sum(wk * (a + b @ u) for wk, (a, b) in zip(w, coefs))
            want_g = sum(wk * b for wk, (a, b) in zip(w, coefs))    # dE/du in grid units
            assert abs(E - want_E) < 1e-12
            assert np.allclose(grad[:3], want_g, atol=1e-12)        # translation genes are grid units
            assert np.allclose(grad[3:6], 0.0, atol=1e-12)          # a single atom at the centre


def test_constant_map_zero_gradient():
    G = affine_grid([(2.5, np.zeros(3)), (1.0, np.zeros(3)), (-3.0, np.zeros(3))])
    L = _one_atom(0.4)
    E, grad, *_ = O.eval_one(L, G, ff_default(), _genes_at(G, np.array([3.3, 7.1, 4.9])))
    q = float(np.float32(0.4))
    assert abs(E - (2.5 + q - 3.0 * q)) < 1e-12
    assert np.allclose(grad, 0.0, atol=1e-12)


def test_brute_force_against_scipy_map_coordinates():
    rng = np.random.default_rng(1)
    n = 9
    maps = rng.normal(size=(4, n, n, n)).astype(np.float32)   # 2 type maps + e + d
    G = Grid(nx=n, ny=n, nz=n, spacing=0.375, origin=np.array([0.1, -0.2, 0.3], np.float32), maps=maps)
    ff = ff_default()
    for t in (0, 1):
        for q in (0.3, -0.8):
            q = float(np.float32(q))
            L = _one_atom(q, t=t, nt=2)
            for _ in range(25):
                u = rng.uniform(0.0, n - 1.0 - 1e-9, 3)
                E, *_ = O.eval_one(L, G, ff, _genes_at(G, u))
                zyx = np.array([[u[2]], [u[1]], [u[0]]])
                mc = [map_coordinates(maps[m].astype(np.float64), zyx, order=1)[0] for m in (t, 2, 3)]
                want = mc[0] + q * mc[1] + abs(q) * mc[2]
                assert abs(E - want) < 1e-12


def test_gradient_equals_axis_finite_difference():
    """Inside one cell the interpolant is affine along each axis, so a central
    difference along x/y/z equals dE/du to rounding."""
    rng = np.random.default_rng(2)
    n = 8
    maps = rng.normal(size=(3, n, n, n)).astype(np.float32)
    G = Grid(nx=n, ny=n, nz=n, spacing=0.5, origin=np.zeros(3, np.float32), maps=maps)
    L = _one_atom(0.6)
    ff = ff_default()
    for _ in range(20):
        u = np.floor(rng.uniform(0, n - 1, 3)) + rng.uniform(0.1, 0.9, 3)
        E, grad, *_ = O.eval_one(L, G, ff, _genes_at(G, u))
        for k in range(3):
            d = np.zeros(3)
            d[k] = 1e-3
            ep = O.eval_one(L, G, ff, _genes_at(G, u + d))[0]
            em = O.eval_one(L, G, ff, _genes_at(G, u - d))[0]
            assert abs((ep - em) / 2e-3 - grad[k]) < 1e-9


def test_out_of_grid_restraint():
    G = affine_grid([(0.0, np.zeros(3))] * 3, n=12)
    ff = ff_default()
    L = _one_atom(0.5)
    c = 0.5 * (12 - 1)
    for u in ([-0.5, 3.0, 4.0], [3.0, 11.0, 4.0], [12.5, -2.0, 30.0], [0.0, 11.0 - 1e-9, 5.0]):
        u = np.array(u)
        E, grad, aux, *_ = O.eval_one(L, G, ff, _genes_at(G, u))
        out = np.any(u < 0) or np.any(u >= 11.0)
        if out:
            assert abs(E - ff.w_out * np.sum((u - c) ** 2)) < 1e-9
            # d/du in grid units = 2 w_out (u - c)
            assert np.allclose(grad[:3], 2 * ff.w_out * (u - c), atol=1e-9)
        else:
            assert abs(E) < 1e-12
