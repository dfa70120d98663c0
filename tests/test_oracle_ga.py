"""Pins of the oracle's NEXT-3 GA generation: the generator
against published SplitMix64 values, and every operator against brute force /
invariants on tiny populations."""
import itertools

import numpy as np
import pytest

from oracle import oracle as O


def test_rng_is_splitmix64():
    """The mix step is SplitMix64 (state += golden gamma, then the finaliser): the
    reference generator seeded with 0 emits 0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4,
    0x06C45D188009454F (state = k * gamma before the step)."""
    gamma = 0x9E3779B97F4A7C15
    mix = O.lib().ado_rng_mix
    assert mix(0) == 0xE220A8397B1DCDAF
    assert mix(gamma) == 0x6E789E6AA1B965F4
    assert mix((2 * gamma) % 2 ** 64) == 0x06C45D188009454F
    # the counter chain: rng = mix(mix(mix(seed ^ (gen << 32 | run)) ^ (ind << 32 | d)))
    assert O.rng(5, 1, 2, 3, 4) == mix(mix(mix(5 ^ (1 << 32 | 2)) ^ (3 << 32 | 4)))
    # u24 / index draws are uniform: mean and range over many counters
    u = np.array([(O.rng(7, 1, 2, k, 3) >> 40) / 2.0 ** 24 for k in range(20000)])
    assert u.min() >= 0.0 and u.max() < 1.0 and abs(u.mean() - 0.5) < 0.01
    idx = np.array([(O.rng(7, 1, 2, k, 4) >> 32) % 10 for k in range(20000)])
    assert np.all(np.bincount(idx, minlength=10) > 1800)


def _pop(n, stride, seed=0):
    rng = np.random.default_rng(seed)
    return rng.uniform(-50, 50, (n, stride)).astype(np.float32), rng.permutation(n).astype(np.float32) - 3.5


@pytest.mark.parametrize("elitism", [0, 1, 3])
def test_elitism_keeps_the_best_in_order(elitism):
    g, E = _pop(12, 10)
    P = O.ga_params(12, 8, 10, elitism=elitism)
    out = O.ga_generation(P, g, E, 11, 4, 2)
    order = np.argsort(E, kind="stable")
    for k in range(elitism):
        assert np.array_equal(out[k], g[order[k]])


def test_tournament_rate_one_picks_the_better():
    # pop 2, no crossover / mutation: every child is a copy of the better individual
    # unless both draws hit the worse one (a == b == worse); brute force over the draws
    g, E = _pop(2, 8)
    P = O.ga_params(2, 8, 8, elitism=0, cross_rate=0.0, mut_rate=0.0, tour_rate=1.0)
    out = O.ga_generation(P, g, E, 5, 0, 0)
    better = int(np.argmin(E))
    for k in range(2):
        a = (O.rng(5, 0, 0, k, 0) >> 32) % 2
        b = (O.rng(5, 0, 0, k, 1) >> 32) % 2
        exp = better if better in (a, b) else a
        assert np.array_equal(out[k], g[exp])


def test_selection_only_copies_rows():
    g, E = _pop(9, 10)
    P = O.ga_params(9, 10, 10, elitism=1, cross_rate=0.0, mut_rate=0.0, tour_rate=0.6)
    out = O.ga_generation(P, g, E, 3, 1, 1)
    for row in out:
        assert any(np.array_equal(row, r) for r in g)


def test_two_point_crossover_structure():
    g, E = _pop(6, 12)
    P = O.ga_params(6, 12, 12, elitism=0, cross_rate=1.0, mut_rate=0.0, tour_rate=0.6)
    out = O.ga_generation(P, g, E, 9, 2, 0)
    for row in out:
        ok = False
        for A, B in itertools.product(range(6), repeat=2):
            diff = np.nonzero(row != g[A])[0]
            if diff.size == 0:
                ok = True
                break
            lo, hi = diff.min(), diff.max() + 1
            if np.array_equal(row[lo:hi], g[B, lo:hi]) and np.array_equal(np.delete(row, range(lo, hi)),
                                                                          np.delete(g[A], range(lo, hi))):
                ok = True
                break
        assert ok


def test_mutation_bounds_and_centering():
    pop, G = 400, 10
    g = np.zeros((pop, G), np.float32)
    E = np.zeros(pop, np.float32)
    P = O.ga_params(pop, G, G, elitism=0, cross_rate=0.0, mut_rate=1.0, tour_rate=1.0, dmov=2.0, dang=90.0)
    out = O.ga_generation(P, g, E, 1, 0, 0)  # parents are all zero rows: out = the deltas
    assert np.all(np.abs(out[:, :3]) <= 2.0) and np.all(np.abs(out[:, 3:]) <= 90.0)
    assert abs(out[:, 3:].mean()) < 3.0 and out[:, 3:].std() > 45.0   # U(-90, 90): sd 52
    # delta = (2u - 1) * max exactly: (delta / max + 1) / 2 is a multiple of 2^-24
    u = (out[:, 3:].astype(np.float64) / 90.0 + 1.0) / 2.0
    assert np.allclose(u * 2 ** 24, np.round(u * 2 ** 24), atol=2e-6 * 2 ** 24 / 90.0)
    P0 = O.ga_params(pop, G, G, elitism=0, cross_rate=0.0, mut_rate=0.0, tour_rate=1.0)
    assert np.array_equal(O.ga_generation(P0, g, E, 1, 0, 0), g)


def test_ls_selection_rate():
    P = O.ga_params(5000, 8, 8, ls_rate=0.8)
    assert abs(O.ls_select(P, 3, 0, 0).mean() - 0.8) < 0.02
    P = O.ga_params(100, 8, 8, ls_rate=0.0)
    assert not O.ls_select(P, 3, 0, 0).any()
