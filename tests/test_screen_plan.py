"""Config 5 (virtual screen) host logic on CPU: the lazy ScreenSpec reproduces
make_screen, the sharding plan covers every (ligand, run) unit exactly once on
every world size, and launch buckets never mix >32-gene ligands with narrow ones."""
import numpy as np

from paper_conf_sc_solis_vasquezts25_b200 import screen, synth


def test_screen_spec_matches_materialised_screen():
    spec = synth.ScreenSpec(n_ligands=6, runs=2, pop=4)
    w = synth.make_screen(n_ligands=6, runs=2, pop=4)
    assert np.array_equal(spec.grid.maps, w.grid.maps)
    for k in range(6):
        L, M = spec.ligand(k), w.ligands[k]
        assert (L.n_atoms, L.n_tors) == spec.sizes[k] == (M.n_atoms, M.n_tors)
        assert np.array_equal(L.pairs, M.pairs) and np.array_equal(L.ref_xyz, M.ref_xyz)
        assert np.array_equal(spec.genes(k), w.genes[k * 8:(k + 1) * 8])
    # sizes follow the config-5 recipe: N ~ U{20..110}, T ~ U{0..min(32, N/3)}
    big = synth.ScreenSpec(n_ligands=2000)
    n = np.array([s[0] for s in big.sizes])
    t = np.array([s[1] for s in big.sizes])
    assert n.min() >= 20 and n.max() <= 110 and np.all(t <= np.minimum(32, n // 3)) and t.min() == 0


def test_pair_estimate_tracks_the_generator():
    spec = synth.ScreenSpec(n_ligands=40)
    real = np.array([spec.ligand(k).n_pairs for k in range(40)], float)
    est = np.array([spec.n_pairs(k) for k in range(40)])
    assert np.corrcoef(real, est)[0, 1] > 0.9
    assert 0.7 < real.sum() / est.sum() < 1.4


def test_plan_covers_units_on_every_world_size():
    spec = synth.ScreenSpec(n_ligands=64, runs=5, pop=4)
    for world in (1, 2, 4, 8):
        units, shards = screen.plan(spec, world)
        assert len(units) == 64 * 5 and len(set(units)) == len(units)
        flat = sorted(u for s in shards for u in s)
        assert flat == list(range(len(units)))
        # LPT on the spec's costs: per-rank loads within 4/3 of the mean (many small units)
        from paper_conf_sc_solis_vasquezts25_b200 import dist as addist
        cost = [addist.unit_cost(*spec.sizes[k], spec.n_pairs(k), spec.pop, spec.iters) for k, _ in units]
        loads = [sum(cost[u] for u in s) for s in shards]
        assert max(loads) <= 4.0 / 3.0 * max(sum(cost) / world, max(cost)) + 1e-6


def test_buckets_split_wide_and_narrow():
    spec = synth.ScreenSpec(n_ligands=48, runs=2, pop=4)
    ligs = {k: spec.ligand(k) for k in range(48)}
    mine = [(k, r) for k in range(48) for r in range(2)]
    buckets = screen.make_buckets(mine, ligs, 5)
    assert sorted(u for b in buckets for u in b) == sorted(mine)
    for b in buckets:
        wide = {6 + ligs[k].n_tors > 32 for k, _ in b}
        assert len(wide) == 1
    # within each class the buckets are ordered by pair count
    narrow = [b for b in buckets if 6 + ligs[b[0][0]].n_tors <= 32]
    for a, c in zip(narrow, narrow[1:]):
        assert max(ligs[k].n_pairs for k, _ in a) <= min(ligs[k].n_pairs for k, _ in c)


def test_buckets_never_mix_pair_loop_kinds():
    """Launches run the specialised kernel twins only when every ligand shares the pair
    loop (ad.pair_loop_kind), so buckets are kind-pure; every unit lands once."""
    spec = synth.ScreenSpec(n_ligands=48, runs=2, pop=4)
    ligs = {k: spec.ligand(k) for k in range(48)}
    mine = [(k, r) for k in range(48) for r in range(2)]
    kind = {k: (1 if ligs[k].n_pairs < 500 else 2) if k % 7 else 0 for k in ligs}
    buckets = screen.make_buckets(mine, ligs, 6, kind)
    assert sorted(u for b in buckets for u in b) == sorted(mine)
    for b in buckets:
        assert len({kind[k] for k, _ in b}) == 1 and len({6 + ligs[k].n_tors > 32 for k, _ in b}) == 1


def test_list_spec_slices_start_genes():
    spec = synth.ScreenSpec(n_ligands=3, runs=2, pop=4)
    ligs = [spec.ligand(k) for k in range(3)]
    genes = np.concatenate([spec.genes(k) for k in range(3)])
    ls = screen.ListSpec(spec.grid, ligs, genes, 2, 4, 300)
    assert ls.n_ligands == 3 and ls.stride == genes.shape[1]
    for k in range(3):
        assert np.array_equal(ls.genes(k), spec.genes(k)) and ls.n_pairs(k) == ligs[k].n_pairs
    got = screen.generate(ls, [2, 0])
    assert set(got) == {0, 2} and got[2][0] is ligs[2]
