"""NEXT-4: AutoGrid .fld/.map and PDBQT inputs (P:L499, P:L507-508,
P:L520-521 `-ffile protein.maps.fld -lfile ligand.pdbqt`), host side, no GPU.

Pinned on hand-written fixtures (tests/golden/autogrid/: a 3x3x3-point map set
whose values encode their own indices, and a 6-atom chain with two nested
rotatable bonds whose fragments, moving sets and pair list are worked out by
hand below), on round trips through the writers, and on the oracle: a
ligand/grid read back from files scores exactly like the arrays they came from.
"""
import os

import numpy as np
import pytest

from paper_conf_sc_solis_vasquezts25_b200 import io as adio
from paper_conf_sc_solis_vasquezts25_b200 import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden", "autogrid")


def test_read_map_layout_and_origin():
    hdr, v = adio.read_map(os.path.join(GOLD, "tiny.OA.map"))
    assert hdr["points"] == (3, 3, 3) and hdr["spacing"] == 0.5
    assert hdr["origin"] == [0.5, 1.5, 2.5]          # CENTER - h * NELEMENTS / 2
    k, j, i = np.meshgrid(range(3), range(3), range(3), indexing="ij")
    assert np.array_equal(v, 100 + 9 * k + 3 * j + i)  # x fastest, then y, then z


def test_read_fld_orders_maps_type_elec_desolv():
    g, names = adio.read_fld(os.path.join(GOLD, "tiny.maps.fld"))
    assert names == ["C", "OA"]
    assert (g.nx, g.ny, g.nz, g.n_maps) == (3, 3, 3, 4) and g.spacing == 0.5
    assert np.allclose(g.origin, [0.5, 1.5, 2.5])
    # the fixture lists e / d before OA: the ABI order is C, OA, e, d
    assert [int(m[0, 0, 0]) for m in g.maps] == [0, 100, 200, 300]


def test_map_errors(tmp_path):
    p = tmp_path / "bad.map"
    p.write_text("SPACING 0.5\nNELEMENTS 2 2 2\nCENTER 0 0 0\n1\n2\n")
    with pytest.raises(adio.FormatError, match="values"):
        adio.read_map(str(p))
    q = tmp_path / "bad.maps.fld"
    q.write_text("ndim=3\nvariable 1 file=x.C.map filetype=ascii skip=6\n")
    with pytest.raises(adio.FormatError, match="e.map"):
        adio.read_fld(str(q))


def test_write_maps_round_trip(tmp_path):
    names = synth.TYPESETS[3]
    g = synth.make_grid(11, 13, names, 60)  # 13 points per axis: NELEMENTS 12
    adio.write_maps(g, names, str(tmp_path / "rec"))
    g2, n2 = adio.read_fld(str(tmp_path / "rec.maps.fld"))
    assert n2 == names and (g2.nx, g2.ny, g2.nz) == (g.nx, g.ny, g.nz)
    assert np.allclose(g2.origin, g.origin, atol=1e-4) and g2.spacing == pytest.approx(g.spacing)
    assert np.allclose(g2.maps, g.maps, rtol=1e-5, atol=1e-5)
    with pytest.raises(ValueError):
        adio.write_maps(synth.make_grid(11, 12, names, 60), names, str(tmp_path / "even"))


def test_read_pdbqt_hand_worked_chain():
    lig, c = adio.read_pdbqt(os.path.join(GOLD, "butanol.pdbqt"), ["C", "OA", "HD"])
    xyz = np.array([[0, 0, 0], [1.52, 0, 0], [2.03, 1.43, 0], [3.55, 1.43, 0], [4.02, 2.78, 0], [4.99, 2.78, 0]])
    assert np.allclose(c, xyz.mean(0)) and np.allclose(lig.ref_xyz, xyz - xyz.mean(0), atol=1e-6)
    assert np.allclose(lig.charge, [-0.1, 0.05, 0.04, 0.2, -0.4, 0.21])
    assert lig.type_names == ["C", "OA", "HD"] and lig.atom_type.tolist() == [0, 0, 0, 0, 1, 2]
    assert lig.atom_map.tolist() == [0, 0, 0, 0, 1, 2]
    # chain bonds 1-2-3-4-5-6 inferred from covalent radii
    assert sorted(map(tuple, lig.bonds.tolist())) == [(0, 1), (1, 2), (2, 3), (3, 4), (4, 5)]
    # BRANCH 2 3 (root -> leaf), then the nested BRANCH 4 5
    assert lig.tors_axis.tolist() == [[1, 2], [3, 4]]
    assert lig.tors_moving.tolist() == [[0, 0, 1, 1, 1, 1], [0, 0, 0, 0, 1, 1]]
    assert lig.frag.tolist() == [0, 0, 1, 1, 2, 2]
    # pairs: different fragment and >= 4 bonds apart: C1-O5 (4), C1-H6 (5), C2-H6 (4)
    assert sorted(map(tuple, lig.pairs.tolist())) == [(0, 4), (0, 5), (1, 5)]
    # 12-10 for the donor H x acceptor pair only (HD x OA), 12-6 otherwise
    assert lig.tp_coef[2, 1, 4] == 10 and lig.tp_coef[1, 2, 4] == 10 and lig.tp_coef[0, 2, 4] == 6
    with pytest.raises(adio.FormatError, match="no grid map"):
        adio.read_pdbqt(os.path.join(GOLD, "butanol.pdbqt"), ["C", "OA"])


def test_pdbqt_errors(tmp_path):
    p = tmp_path / "x.pdbqt"
    p.write_text("ROOT\nATOM      1  C1  LIG A   1       0.000   0.000   0.000  1.00  0.00    -0.100 C \n"
                 "ENDROOT\nBRANCH   1   2\nATOM      2  C2  LIG A   1       1.500   0.000   0.000  1.00  0.00"
                 "     0.100 C \n")
    with pytest.raises(adio.FormatError, match="unclosed"):
        adio.read_pdbqt(str(p), ["C"])
    p.write_text("ROOT\nATOM      1  C1  LIG A   1       0.000   0.000   0.000  1.00  0.00    -0.100 Xx\nENDROOT\n")
    with pytest.raises(adio.FormatError, match="unknown"):
        adio.read_pdbqt(str(p), ["C"])


def _tors_perm(L, R, inv):
    """perm[b] = the torsion of L that is R's torsion b (same axis)."""
    axis = {tuple(inv[a].tolist()): k for k, a in enumerate(L.tors_axis)}
    return np.array([axis[tuple(a)] for a in R.tors_axis.tolist()], dtype=np.int64)


@pytest.mark.parametrize("cfg", [1, 2, 3])
def test_pdbqt_round_trip_of_synthetic_ligands(tmp_path, cfg):
    w = synth.make_config(cfg)
    L = w.ligands[0]
    center = np.array([1.25, -2.5, 0.75])
    order = adio.write_pdbqt(L, str(tmp_path / "lig.pdbqt"), centroid=center)
    R, c = adio.read_pdbqt(str(tmp_path / "lig.pdbqt"), L.type_names)
    inv = np.empty_like(order)
    inv[order] = np.arange(L.n_atoms)
    assert R.n_atoms == L.n_atoms and R.n_tors == L.n_tors and R.n_pairs == L.n_pairs
    assert np.allclose(R.ref_xyz + c, L.ref_xyz[order] + center, atol=6e-4)
    assert np.allclose(R.charge, L.charge[order], atol=6e-4)
    assert [L.type_names[t] for t in L.atom_type[order]] == [R.type_names[t] for t in R.atom_type]
    # the same torsions (axes and moving sets); PDBQT lists them depth-first, the
    # generator breadth-first -- both root -> leaf (every torsion after its parent)
    perm = _tors_perm(L, R, inv)
    assert np.array_equal(inv[L.tors_axis[perm]], R.tors_axis)
    assert np.array_equal(L.tors_moving[perm][:, order], R.tors_moving)
    for b in range(R.n_tors):
        parents = [c for c in range(b) if R.tors_moving[c][R.tors_moving[b].astype(bool)].all()]
        assert all(R.tors_moving[c].sum() > R.tors_moving[b].sum() for c in parents)
    assert sorted(map(tuple, np.sort(inv[L.pairs], axis=1).tolist())) == sorted(map(tuple, R.pairs.tolist()))


def test_read_inputs_score_like_their_arrays(tmp_path):
    """Oracle energies and gradients of a config-2 ligand + grid written as
    PDBQT / AutoGrid files and read back equal those of the arrays (the same
    rounded coordinates and charges, atoms permuted): the reader rebuilds the
    torsion tree, pair list and type tables the scoring needs."""
    from oracle import oracle as O
    names = synth.TYPESETS[6]
    L = synth.make_config(2).ligands[0]
    g = synth.make_grid(2100, 61, names, 2000)       # 61 points: an AutoGrid NELEMENTS 60 grid
    adio.write_maps(g, names, str(tmp_path / "rec"))
    G2, n2 = adio.read_fld(str(tmp_path / "rec.maps.fld"))
    center = np.array([0.3, -0.2, 0.1])
    order = adio.write_pdbqt(L, str(tmp_path / "lig.pdbqt"), centroid=center)
    R, c = adio.read_pdbqt(str(tmp_path / "lig.pdbqt"), n2)
    # the arrays as the files store them: coordinates / charges rounded, maps as read
    Lr = synth.Ligand(ref_xyz=R.ref_xyz[np.argsort(order)], atom_map=L.atom_map, atom_type=L.atom_type,
                      charge=R.charge[np.argsort(order)], tors_axis=L.tors_axis, tors_moving=L.tors_moving,
                      pairs=L.pairs, tp_coef=L.tp_coef, type_S=L.type_S, type_V=L.type_V, type_names=L.type_names)
    rng = np.random.default_rng(5)
    genes = np.zeros((16, 6 + L.n_tors), np.float32)
    genes[:, :3] = adio.input_genes(c, G2, L.n_tors)[:3] + rng.uniform(-2, 2, (16, 3))
    genes[:, 3:] = rng.uniform(-60, 60, (16, 3 + L.n_tors))
    genes[0] = adio.input_genes(c, G2, L.n_tors)
    inv = np.empty_like(order)
    inv[order] = np.arange(L.n_atoms)
    perm = _tors_perm(L, R, inv)                     # R's torsion b is L's torsion perm[b]
    genes_L = genes.copy()
    genes_L[:, 6 + perm] = genes[:, 6:]
    E1, G1, _, _ = O.score(R, G2, synth.FFParams(), genes)
    E0, G0, _, _ = O.score(Lr, G2, synth.FFParams(), genes_L)
    assert np.allclose(E1, E0, rtol=1e-9, atol=1e-9)
    assert np.allclose(G1[:, :6], G0[:, :6], rtol=1e-7, atol=1e-7)
    assert np.allclose(G1[:, 6:], G0[:, 6 + perm], rtol=1e-7, atol=1e-7)
    # identity genes reproduce the file's conformation
    X = O.pose(R, G2, genes[0].astype(np.float64))
    assert np.allclose(X, R.ref_xyz + c, atol=1e-4)
