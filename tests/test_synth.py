"""Generator tests: determinism and the structural rules of DESIGN.md's input recipe."""
import numpy as np

from paper_conf_sc_solis_vasquezts25_b200 import synth


def _graph_dist(n, bonds):
    adj = [[] for _ in range(n)]
    for u, v in bonds:
        adj[u].append(v)
        adj[v].append(u)
    D = np.full((n, n), 99)
    for s in range(n):
        D[s, s] = 0
        fr = [s]
        while fr:
            nx = []
            for u in fr:
                for v in adj[u]:
                    if D[s, v] == 99:
                        D[s, v] = D[s, u] + 1
                        nx.append(v)
            fr = nx
    return D, adj


def test_deterministic():
    a = synth.make_ligand(123, 30, 5, 6)
    b = synth.make_ligand(123, 30, 5, 6)
    for f in ("ref_xyz", "atom_type", "charge", "tors_axis", "tors_moving", "pairs", "tp_coef"):
        assert np.array_equal(getattr(a, f), getattr(b, f))
    ga = synth.make_genotypes(7, 10, 5, synth.make_grid(1, 16, synth.TYPESETS[3], 50))
    gb = synth.make_genotypes(7, 10, 5, synth.make_grid(1, 16, synth.TYPESETS[3], 50))
    assert np.array_equal(ga, gb)


def test_ligand_rules(cfg2):
    L = cfg2.ligands[0]
    N = L.n_atoms
    assert (N, L.n_tors, L.n_types) == (40, 8, 6)
    assert len(L.bonds) == N - 1                      # a tree
    D, adj = _graph_dist(N, L.bonds)
    assert D.max() < 99                               # connected
    bl = np.linalg.norm(L.ref_xyz[L.bonds[:, 0]] - L.ref_xyz[L.bonds[:, 1]], axis=1)
    assert np.all(np.abs(bl - 1.5) <= 0.05 + 1e-5)
    dd = np.linalg.norm(L.ref_xyz[:, None] - L.ref_xyz[None], axis=2)
    iu = np.triu_indices(N, 1)
    nb = D[iu] > 1
    assert dd[iu][nb].min() >= 2.0                    # no non-bonded pair under 2 A
    assert np.allclose(L.ref_xyz.mean(0), 0, atol=1e-5)
    assert abs(L.charge.sum()) < 1e-4
    # pair list: different fragment AND graph distance >= 4, complete
    want = {(i, j) for i in range(N) for j in range(i + 1, N) if L.frag[i] != L.frag[j] and D[i, j] >= 4}
    got = {tuple(p) for p in L.pairs.tolist()}
    assert got == want
    # torsions: axis is a bond; moving set = c side, closed subtree, a not in it
    for b, (a, c) in enumerate(L.tors_axis):
        assert D[a, c] == 1
        m = L.tors_moving[b].astype(bool)
        assert m[c] and not m[a]
        for u in np.nonzero(m)[0]:
            for v in adj[u]:
                if not (u == c and v == a):
                    assert m[v], "moving set must be closed under bonds except the axis"
    # root -> leaf order: a parent torsion's moving set contains the child's
    for b in range(L.n_tors):
        for b2 in range(b + 1, L.n_tors):
            mb = L.tors_moving[b].astype(bool)
            m2 = L.tors_moving[b2].astype(bool)
            assert not (mb & m2).any() or (m2 <= mb).all() or (mb <= m2).all()
            assert not ((mb <= m2).all() and (mb != m2).any()), "child listed before parent"


def test_hbond_table():
    L = synth.make_ligand(5, 40, 8, 6)
    names = L.type_names
    hd = names.index("HD")
    oa = names.index("OA")
    c = names.index("C")
    assert L.tp_coef[hd, oa, 4] == 10.0 and L.tp_coef[oa, hd, 4] == 10.0
    assert L.tp_coef[c, oa, 4] == 6.0
    assert np.allclose(L.tp_coef, L.tp_coef.transpose(1, 0, 2))


def test_genotype_ranges(cfg2):
    g = cfg2.genes
    n = cfg2.grid.nx
    assert g.shape == (3000, 14)
    assert np.all(g[:, :3] >= 0.25 * (n - 1) - 1e-4) and np.all(g[:, :3] <= 0.75 * (n - 1) + 1e-4)
    assert np.all((g[:, 3] >= 0) & (g[:, 3] < 360)) and np.all((g[:, 4] >= 0) & (g[:, 4] <= 180))
    assert np.all(np.abs(g[:, 6:]) <= 180)


def test_grid_shapes(cfg1, cfg2):
    assert cfg1.grid.maps.shape == (5, 32, 32, 32)
    assert cfg2.grid.maps.shape == (8, 60, 60, 60)
    assert np.isfinite(cfg2.grid.maps).all()
