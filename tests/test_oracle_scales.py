"""Pins for the oracle's tolerance scales (Z18; DESIGN.md
"Tolerances"): A_E (aux[AUX_ABS_E]), A_grad (agrad) and the clash-gate S_E
(aux[AUX_SENS_E]).  A bug that inflated them would silently widen every parity
gate, so each is pinned on cases whose value the mathematics fixes without
re-typing the oracle's formula: trilinear weights summing to 1, linearity of
the energy in its terms, single-summand cases, and central finite differences
of the energy itself."""
import dataclasses

import numpy as np

from oracle import oracle as O
from tests.util import affine_grid, const_grid, ff_default, hand_ligand, identity_genes

EPS, R0 = 0.25, 4.0


def _tp(m=12, n=6, eps=EPS, r0=R0, a=1.0, b=1.0):
    cA = a * eps * r0 ** m * n / (m - n)
    cB = b * eps * r0 ** n * m / (m - n)
    return np.array([[[cA, cB, r0, m, n]]], np.float32)


def test_abs_energy_constant_maps():
    """Constant maps t, e, d: every trilinear weight is >= 0 and they sum to 1, so
    A_E = |t| + |q e| + ||q| d| while E = t + q e + |q| d."""
    n = 12
    for t, e, d, q in ((0.75, -1.5, 0.25, 0.375), (-2.0, 0.5, -0.125, -0.625), (1.0, 1.0, 1.0, 0.0)):
        G = const_grid(n=n, n_type_maps=1)
        G.maps[0], G.maps[1], G.maps[2] = t, e, d
        L = hand_ligand([[0.0, 0.0, 0.0]], charges=[q])
        g = identity_genes(G, (0.1, -0.2, 0.3), 0)
        E, _, aux, _, _ = O.eval_one(L, G, ff_default(), g)
        assert abs(E - (t + q * e + abs(q) * d)) < 1e-12
        assert abs(aux[O.AUX_ABS_E] - (abs(t) + abs(q * e) + abs(abs(q) * d))) < 1e-12


def test_abs_energy_is_sum_of_term_magnitudes():
    """One pair with a vdW wall + well, charges of opposite sign and desolvation:
    A_E equals the sum of |E| of the four parts evaluated separately (linearity),
    while E is their signed sum."""
    ff = ff_default()
    G = const_grid(n=80)
    r = 3.4
    xyz = [[-r / 2, 0, 0], [r / 2, 0, 0]]
    q = (0.4, -0.3)
    S, V = (-0.002,), (30.0,)

    def E_of(tp, q, S, V, f=ff):
        L = hand_ligand(xyz, pairs=[(0, 1)], charges=q, tp=tp, S=S, V=V)
        E, _, aux, _, _ = O.eval_one(L, G, f, identity_genes(G, (0, 0, 0), 0))
        return E, aux[O.AUX_ABS_E]

    E_all, A_all = E_of(_tp(), q, S, V)
    no_el = dataclasses.replace(ff, coeff_el=0.0)
    parts = [E_of(_tp(b=0.0), (0, 0), (0,), (0,))[0],      # repulsive cA s^-12
             E_of(_tp(a=0.0), (0, 0), (0,), (0,))[0],      # attractive -cB s^-6
             E_of(_tp(eps=0.0), q, (0,), (0,))[0],          # electrostatics
             E_of(_tp(eps=0.0), q, S, V, no_el)[0]]         # desolvation (charge-dependent part included)
    assert parts[0] > 0 > parts[1] and parts[2] < 0 and parts[3] != 0
    assert abs(E_all - sum(parts)) < 1e-12 * max(1.0, abs(E_all))
    assert abs(A_all - sum(abs(p) for p in parts)) < 1e-12 * A_all
    assert A_all > abs(E_all)


def _off_centre_atom_case(q):
    coefs = [(0.75, np.array([0.25, -0.125, 0.0625])), (-1.5, np.array([-0.5, 0.125, 0.25])),
             (0.25, np.array([0.015625, 0.03125, -0.03125]))]
    return affine_grid(coefs, n=24)


def test_agrad_single_summand_is_abs_gradient():
    """One atom, no pairs: every gene's chain rule has ONE summand, so A_grad = |grad|."""
    G = _off_centre_atom_case(0.3)
    L = hand_ligand([[0.7, -0.3, 0.4]], charges=[0.3])
    rng = np.random.default_rng(3)
    for _ in range(5):
        g = np.array([11.0, 12.5, 10.25, rng.uniform(0, 360), rng.uniform(0, 180), rng.uniform(0, 360)])
        E, grad, aux, agrad, _ = O.eval_one(L, G, ff_default(), g)
        assert np.allclose(agrad, np.abs(grad), rtol=1e-12, atol=1e-14)
        assert np.linalg.norm(grad[3:]) > 1e-3          # off-centre: a real torque


def test_agrad_adds_atom_magnitudes():
    """Two atoms with no pair term: A_grad = |grad(atom 1 alone)| + |grad(atom 2 alone)|
    gene by gene, while grad = grad1 + grad2 (opposite charges: the translation
    gradient cancels almost completely)."""
    # flat type and desolvation maps, sloped electrostatic map
    G = affine_grid([(0.75, np.zeros(3)), (-1.5, np.array([-0.5, 0.125, 0.25])), (0.25, np.zeros(3))], n=24)
    ff = ff_default()
    xyz = [[0.7, -0.3, 0.4], [-0.6, 0.2, -0.5]]
    q = [0.375, -0.375]
    g = np.array([11.0, 12.5, 10.25, 40.0, 70.0, 125.0])
    _, grad, _, agrad, _ = O.eval_one(hand_ligand(xyz, charges=q), G, ff, g)
    _, g1, *_ = O.eval_one(hand_ligand(xyz[:1], charges=q[:1]), G, ff, g)
    _, g2, *_ = O.eval_one(hand_ligand(xyz[1:], charges=q[1:]), G, ff, g)
    assert np.allclose(grad, g1 + g2, rtol=1e-12, atol=1e-13)
    assert np.allclose(agrad, np.abs(g1) + np.abs(g2), rtol=1e-12, atol=1e-13)
    assert np.all(agrad[:3] > 5 * np.abs(grad[:3]))


def _pair_fd(r, ff, G, tp, q=(0.0, 0.0), step=2.0 ** -9):
    """dE/dr by the 5-point central stencil; r and the step are dyadic, so the FP32
    reference coordinates +-r/2 are exact."""
    def E(rr):
        L = hand_ligand([[-rr / 2, 0, 0], [rr / 2, 0, 0]], pairs=[(0, 1)], charges=q, tp=tp)
        return O.eval_one(L, G, ff, identity_genes(G, (0, 0, 0), 0))[0]
    return (-E(r + 2 * step) + 8 * E(r + step) - 8 * E(r - step) + E(r - 2 * step)) / (12 * step)


def test_agrad_pair_translation_and_rotation():
    """A single pair on a zero grid, atoms at -+r/2 on the x axis around the rotation
    centre: each atom's translation summand is h F_x, so A_grad[0] = 2 h |dE/dr|
    (dE/dr by central differences of E), A_grad[1, 2] = 0, and the rotation summands
    vanish (the central force is parallel to X_i - T), while grad = 0 (Newton)."""
    ff = ff_default()
    G = const_grid(n=80)
    h = G.spacing
    for r, q in ((3.125, (0.0, 0.0)), (4.875, (0.5, 0.25)), (2.25, (-0.3, 0.6))):
        L = hand_ligand([[-r / 2, 0, 0], [r / 2, 0, 0]], pairs=[(0, 1)], charges=q, tp=_tp())
        E, grad, aux, agrad, _ = O.eval_one(L, G, ff, identity_genes(G, (0, 0, 0), 0))
        dEdr = _pair_fd(r, ff, G, _tp(), q)
        assert abs(agrad[0] - 2 * h * abs(dEdr)) <= 1e-6 * abs(dEdr) + 1e-9
        assert agrad[1] == 0.0 and agrad[2] == 0.0
        assert np.all(agrad[3:] <= 1e-12 * agrad[0])
        assert np.all(np.abs(grad) <= 1e-12 * agrad[0])
        # S_E (clash gate only) = |dE/dr| (|X_i| + |X_j|) = |dE/dr| r
        assert abs(aux[O.AUX_SENS_E] - abs(dEdr) * r) <= 1e-6 * abs(dEdr) * r


def test_agrad_torsion_pair_single_summand():
    """Atom 2 rotates about the 0->1 axis, atom 3 is fixed: the pair's torsion
    summands are |J_2 . F| and |J_3 . F| = 0, so A_grad[6] = |grad[6]|."""
    d = 1.25
    L = hand_ligand([[0, 0, 0], [1, 0, 0], [1, d, 0], [0, d, 0]], tors_axis=[(0, 1)], moving=[(1, 2)],
                    pairs=[(2, 3)], charges=(0.0, 0.0, 0.5, -0.7), tp=_tp())
    G = const_grid(n=40)
    for tdeg in (25.0, 80.0, 150.0):
        g = identity_genes(G, (0, 0, 0), 1)
        g[6] = tdeg
        _, grad, _, agrad, _ = O.eval_one(L, G, ff_default(), g)
        assert abs(grad[6]) > 1e-6
        assert abs(agrad[6] - abs(grad[6])) <= 1e-12 * abs(grad[6])


def test_sens_energy_single_atom_affine():
    """S_E of one atom on an affine grid = |grad_X E| |X| with grad_X E = (b_T + q b_E + |q| b_D) / h."""
    G = _off_centre_atom_case(0.3)
    q = -0.4375
    L = hand_ligand([[0.0, 0.0, 0.0]], charges=[q])
    u = np.array([9.3, 13.7, 11.1])
    g = np.concatenate([u, [0.0, 0.0, 0.0]])
    E, grad, aux, _, X = O.eval_one(L, G, ff_default(), g)
    b = np.array([0.25, -0.125, 0.0625]) + q * np.array([-0.5, 0.125, 0.25]) + abs(q) * np.array(
        [0.015625, 0.03125, -0.03125])
    want = np.linalg.norm(b / G.spacing) * np.linalg.norm(X[0])
    assert abs(aux[O.AUX_SENS_E] - want) <= 1e-12 * want


def test_scales_are_gauge_free():
    """A_E does not depend on the orientation of a rigid ligand on a zero grid (it is
    a sum over pair terms of functions of r only)."""
    L = dataclasses.replace(hand_ligand([[-1.6, 0, 0], [1.6, 0.2, 0], [0.1, 2.0, 0.3]],
                                        pairs=[(0, 1), (0, 2), (1, 2)], charges=(0.3, -0.2, 0.1), tp=_tp()))
    G = const_grid(n=80)
    A = []
    for ang in ((0, 0, 0), (30, 60, 90), (200, 100, 300)):
        g = identity_genes(G, (0.2, -0.1, 0.3), 0)
        g[3:6] = ang
        A.append(O.eval_one(L, G, ff_default(), g)[2][O.AUX_ABS_E])
    assert np.ptp(A) <= 1e-12 * A[0]
