"""Pins for the oracle's PoseCalculation (O-1; Alg 4; genotype P:L53)."""
import numpy as np
import pytest
from scipy.spatial.transform import Rotation

from oracle import oracle as O
from tests.util import const_grid, hand_ligand, identity_genes


def _rand_genes(rng, T, grid):
    g = np.zeros(6 + T)
    g[:3] = rng.uniform(5, grid.nx - 6, 3)
    g[3] = rng.uniform(0, 360)
    g[4] = rng.uniform(0, 180)
    g[5] = rng.uniform(0, 360)
    g[6:] = rng.uniform(-180, 180, T)
    return g


def test_identity_genes_translate_only(cfg2):
    L, G = cfg2.ligands[0], cfg2.grid
    pt = np.array([1.25, -0.5, 2.0])
    g = identity_genes(G, pt, L.n_tors)
    g[3] = 123.0          # phi is irrelevant when theta = 0 and alpha = 0
    X = O.pose(L, G, g)
    assert np.allclose(X, L.ref_xyz.astype(float) + pt, atol=1e-12)


def test_worked_example_torsion_90():
    # a=(0,0,0) -> c=(1.5,0,0) axis +x; atom 2 at (2,1,0) moves; +90 deg
    # (right-handed about +x) sends +y to +z: (2,1,0) -> (2,0,1).
    L = hand_ligand([[0, 0, 0], [1.5, 0, 0], [2.0, 1.0, 0.0]], tors_axis=[(0, 1)], moving=[(1, 2)])
    G = const_grid()
    g = identity_genes(G, (0, 0, 0), 1)
    g[6] = 90.0
    X = O.pose(L, G, g)
    assert np.allclose(X, [[0, 0, 0], [1.5, 0, 0], [2.0, 0.0, 1.0]], atol=1e-12)


def test_worked_example_orientation():
    # phi = 0, theta = 90 -> axis u = +x; alpha = 90: (0,1,0) -> (0,0,1), (0,0,1) -> (0,-1,0)
    L = hand_ligand([[0, 1, 0], [0, 0, 1], [1, 0, 0]])
    G = const_grid()
    g = identity_genes(G, (0, 0, 0), 0)
    g[3], g[4], g[5] = 0.0, 90.0, 90.0
    X = O.pose(L, G, g)
    assert np.allclose(X, [[0, 0, 1], [0, -1, 0], [1, 0, 0]], atol=1e-12)


@pytest.mark.parametrize("which", ["cfg1", "cfg2", "cfg3"])
def test_matches_leaf_first_reference_axis_chain(which, request):
    """Independent construction with scipy rotations: apply each atom's torsions
    leaf -> root about their REFERENCE-frame axes, then R(u, alpha), then T.
    Equal to the oracle's root -> leaf current-axis definition (SURVEY O-1)."""
    w = request.getfixturevalue(which)
    L, G = w.ligands[0], w.grid
    rng = np.random.default_rng(11)
    ref = L.ref_xyz.astype(float)
    for _ in range(5):
        g = _rand_genes(rng, L.n_tors, G)
        X = O.pose(L, G, g)
        out = np.empty_like(ref)
        for i in range(L.n_atoms):
            x = ref[i].copy()
            for b in reversed(range(L.n_tors)):
                if L.tors_moving[b, i]:
                    a, c = L.tors_axis[b]
                    u = ref[c] - ref[a]
                    u /= np.linalg.norm(u)
                    x = ref[a] + Rotation.from_rotvec(u * np.radians(g[6 + b])).apply(x - ref[a])
            out[i] = x
        ph, th, al = np.radians(g[3:6])
        ax = np.array([np.sin(th) * np.cos(ph), np.sin(th) * np.sin(ph), np.cos(th)])
        T = G.origin.astype(float) + G.spacing * g[:3]
        out = Rotation.from_rotvec(ax * al).apply(out) + T
        assert np.allclose(X, out, atol=1e-10)


def test_intra_fragment_distances_invariant(cfg2):
    L, G = cfg2.ligands[0], cfg2.grid
    rng = np.random.default_rng(3)
    ref = L.ref_xyz.astype(float)
    same = L.frag[:, None] == L.frag[None, :]
    d0 = np.linalg.norm(ref[:, None] - ref[None], axis=2)
    for _ in range(5):
        X = O.pose(L, G, _rand_genes(rng, L.n_tors, G))
        d = np.linalg.norm(X[:, None] - X[None], axis=2)
        assert np.allclose(d[same], d0[same], atol=1e-10)
        # bonded distances are preserved for every bond (rotatable too)
        b = L.bonds
        assert np.allclose(d[b[:, 0], b[:, 1]], d0[b[:, 0], b[:, 1]], atol=1e-10)


def test_torsion_360_periodic(cfg2):
    L, G = cfg2.ligands[0], cfg2.grid
    g = _rand_genes(np.random.default_rng(5), L.n_tors, G)
    X = O.pose(L, G, g)
    for b in range(L.n_tors):
        g2 = g.copy()
        g2[6 + b] += 360.0
        assert np.allclose(O.pose(L, G, g2), X, atol=1e-10)
    g2 = g.copy()
    g2[5] += 360.0
    assert np.allclose(O.pose(L, G, g2), X, atol=1e-10)
