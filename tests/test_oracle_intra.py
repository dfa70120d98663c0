"""Pins for the oracle's IntraGradient (O-3; readings Z6-Z10).

Each pin uses a property the mathematics fixes (zero crossing / minimum of the
Lennard-Jones-type forms, textbook Coulomb when the dielectric is constant,
Gaussian ratios, Newton's third law, rigid-motion invariance) rather than a
re-typed copy of the oracle's formula."""
import dataclasses

import numpy as np
import pytest

from oracle import oracle as O
from tests.util import const_grid, f32, ff_default, hand_ligand, identity_genes

EPS = 0.25
R0 = 4.0


def _tp(m, n, eps=EPS, r0=R0):
    # AD4-style table entry with the FE weight folded in = 1
    cA = eps * r0 ** m * n / (m - n)
    cB = eps * r0 ** n * m / (m - n)
    return np.array([[[cA, cB, r0, m, n]]], np.float32)


def _pair_E(r, tp, ff, q=(0.0, 0.0), S=(0.0,), V=(0.0,)):
    L = hand_ligand([[-r / 2, 0, 0], [r / 2, 0, 0]], pairs=[(0, 1)], charges=q, tp=tp, S=S, V=V)
    G = const_grid(n=80, h=0.375)
    E, grad, aux, *_ = O.eval_one(L, G, ff, identity_genes(G, (0, 0, 0), 0))
    return E, aux


def test_vdw_flat_band_is_minimum():
    ff = ff_default()
    d = 0.5 * ff.smooth
    tp = _tp(12, 6)
    cA, cB, r0 = [float(v) for v in tp[0, 0, :3]]
    for r in (R0 - d + 1e-6, R0 - 0.1, R0, R0 + 0.2, R0 + d - 1e-6):
        E, _ = _pair_E(r, tp, ff)
        assert abs(E - (-EPS)) < 1e-5        # minimum of eps[(r0/s)^12 - 2(r0/s)^6] is -eps
    tp10 = _tp(12, 10)
    E, _ = _pair_E(R0 + 0.1, tp10, ff)
    assert abs(E - (-EPS)) < 1e-5            # 12-10 H-bond minimum is also -eps


def test_vdw_zero_crossing_and_shift_direction():
    ff = ff_default()
    d = 0.5 * ff.smooth
    # 12-6 crosses zero at s = r0 2^(-1/6); below the band s = r + delta
    s0 = R0 * 2.0 ** (-1.0 / 6.0)
    E, _ = _pair_E(s0 - d, _tp(12, 6), ff)
    assert abs(E) < 1e-5
    # above the band s = r - delta; at (r0/s)^6 = 1/2 the value is -3/4 eps
    s1 = R0 * 2.0 ** (1.0 / 6.0)
    E, _ = _pair_E(s1 + d, _tp(12, 6), ff)
    assert abs(E - (-0.75 * EPS)) < 1e-5
    # 12-10 crosses zero at s = r0 sqrt(5/6)
    s2 = R0 * np.sqrt(5.0 / 6.0)
    E, _ = _pair_E(s2 - d, _tp(12, 10), ff)
    assert abs(E) < 1e-5


def test_vdw_cutoff():
    ff = ff_default()
    E_in, _ = _pair_E(ff.cut_vdw - 1e-3, _tp(12, 6), ff)
    E_out, _ = _pair_E(ff.cut_vdw + 1e-3, _tp(12, 6), ff)
    assert E_in < 0.0 and E_out == 0.0


def test_coulomb_limits():
    q = (float(np.float32(0.4)), float(np.float32(-0.3)))
    # constant dielectric eps = 1 (B = 0, A = 1): textbook Coulomb c q q / r
    ff = dataclasses.replace(ff_default(), diel_A=1.0, diel_B=0.0)
    for r in (1.5, 3.0, 9.0, 20.0):
        E, _ = _pair_E(r, _tp(12, 6, eps=0.0), ff, q=q)
        assert abs(E - f32(ff.coeff_el) * q[0] * q[1] / r) < 1e-6
    # beyond the electrostatic cutoff: nothing
    E, _ = _pair_E(ff.cut_el + 0.01, _tp(12, 6, eps=0.0), ff, q=q)
    assert E == 0.0
    # r below el_rmin is clamped to el_rmin
    ff2 = dataclasses.replace(ff, el_rmin=1.0)
    E, _ = _pair_E(0.5, _tp(12, 6, eps=0.0), ff2, q=q)
    assert abs(E - f32(ff.coeff_el) * q[0] * q[1] / 1.0) < 1e-9
    # lambda = 0: eps = A + B / (1 + k) everywhere
    ff3 = dataclasses.replace(ff_default(), diel_lambda=0.0)
    epsc = f32(ff3.diel_A) + f32(ff3.diel_B) / (1 + f32(ff3.diel_k))
    E, _ = _pair_E(5.0, _tp(12, 6, eps=0.0), ff3, q=q)
    assert abs(E - f32(ff3.coeff_el) * q[0] * q[1] / (5.0 * epsc)) < 1e-6
    # Mehler-Solmajer: far field approaches the bulk value A + B = 78.4
    ff4 = ff_default()
    E, _ = _pair_E(19.0, _tp(12, 6, eps=0.0), ff4, q=q)
    eps_eff = f32(ff4.coeff_el) * q[0] * q[1] / (19.0 * E)
    assert 70.0 < eps_eff < 78.4


def test_desolvation_gaussian():
    ff = ff_default()
    S, V = (float(np.float32(-0.002)),), (float(np.float32(30.0)),)
    tp = _tp(12, 6, eps=0.0)
    q = (0.0, 0.0)
    s = f32(ff.sigma_ds)
    E0, _ = _pair_E(1e-3, tp, ff, q=q, S=S, V=V)
    E1, _ = _pair_E(s * np.sqrt(2.0), tp, ff, q=q, S=S, V=V)
    assert abs(E1 / E0 - np.exp(-1.0)) < 1e-6
    # prefactor at r -> 0 is c_ds [(S + 0) V + (S + 0) V] for equal types, no charge
    assert abs(E0 - f32(ff.coeff_ds) * 2 * S[0] * V[0]) < 1e-8
    assert _pair_E(ff.cut_el + 0.01, tp, ff, q=q, S=S, V=V)[0] == 0.0


def test_torsion_gradient_closed_form_coulomb():
    """Atom 3 fixed at (0,d,0); atom 2 at (1,d,0) rotates about the x axis
    (torsion 0 -> 1): r^2 = 1 + 2 d^2 (1 - cos t), dr/dt = d^2 sin t / r.
    With a constant dielectric E = c q q / r, so dE/dt = -c q q d^2 sin t / r^3."""
    d = 1.25          # exact in FP32
    q = (0.0, 0.0, float(np.float32(0.5)), float(np.float32(-0.7)))
    L = hand_ligand([[0, 0, 0], [1, 0, 0], [1, d, 0], [0, d, 0]], tors_axis=[(0, 1)], moving=[(1, 2)],
                    pairs=[(2, 3)], charges=q, tp=_tp(12, 6, eps=0.0))
    ff = dataclasses.replace(ff_default(), diel_A=1.0, diel_B=0.0)
    G = const_grid(n=40)
    for tdeg in (30.0, 75.0, 140.0):
        g = identity_genes(G, (0, 0, 0), 1)
        g[6] = tdeg
        E, grad, *_ = O.eval_one(L, G, ff, g)
        t = np.radians(tdeg)
        r = np.sqrt(1 + 2 * d * d * (1 - np.cos(t)))
        c = f32(ff.coeff_el) * q[2] * q[3]
        assert abs(E - c / r) < 1e-9
        assert abs(grad[6] - (-c * d * d * np.sin(t) / r ** 3) * np.pi / 180.0) < 1e-9


@pytest.mark.parametrize("which", ["cfg1", "cfg2"])
def test_newton_third_law_and_rigid_invariance(which, request):
    w = request.getfixturevalue(which)
    L = w.ligands[0]
    G = const_grid(n=96, n_type_maps=L.n_types)       # zero maps, wide: intra only
    ff = ff_default()
    rng = np.random.default_rng(4)
    for p in range(6):
        g = w.genes[p].astype(np.float64)[:L.n_genes]
        g[:3] = 0.5 * (G.nx - 1) + rng.uniform(-2, 2, 3)   # keep every atom in the grid
        E, grad, aux, agrad, X = O.eval_one(L, G, ff, g)
        scale = max(1.0, np.linalg.norm(agrad))
        assert np.all(np.abs(grad[:6]) <= 1e-10 * scale)      # sum of forces and torque vanish
        g2 = g.copy()
        g2[:6] = [0.5 * (G.nx - 1) + 1.0, 0.5 * (G.nx - 1) - 0.5, 0.5 * (G.nx - 1), rng.uniform(0, 360), rng.uniform(0, 180), rng.uniform(0, 360)]
        E2, *_ = O.eval_one(L, G, ff, g2)
        assert abs(E2 - E) <= 1e-10 * max(1.0, aux[O.AUX_ABS_E])


def test_pair_order_permutation(cfg2):
    L = cfg2.ligands[0]
    G, ff = cfg2.grid, ff_default()
    g = cfg2.genes[7].astype(np.float64)
    E, grad, *_ = O.eval_one(L, G, ff, g)
    rng = np.random.default_rng(9)
    P = L.pairs[rng.permutation(L.n_pairs)][:, ::-1].copy()    # shuffled and i <-> j swapped
    L2 = dataclasses.replace(L, pairs=np.ascontiguousarray(P))
    E2, grad2, *_ = O.eval_one(L2, G, ff, g)
    assert abs(E2 - E) < 1e-9 * max(1, abs(E))
    assert np.allclose(grad2, grad, rtol=1e-10, atol=1e-9)
