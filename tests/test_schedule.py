"""CPU checks of libad's intra-pair schedule (host code, no GPU): the
conflict-free read-modify-write design of the pair loop is only race-free if
every step's gradient targets are distinct."""
import ctypes as C

import numpy as np
import pytest

from paper_conf_sc_solis_vasquezts25_b200 import synth


@pytest.fixture(scope="module")
def lib():
    from paper_conf_sc_solis_vasquezts25_b200 import build
    L = C.CDLL(build.build())
    L.adx_debug_schedule.restype = C.c_int32
    L.adx_debug_cherries.restype = C.c_int32
    return L


def _schedule(lib, n_atoms, pairs):
    pairs = np.ascontiguousarray(pairs, np.int32).reshape(-1, 2)
    steps, slots = C.c_int32(), C.c_int32()
    cap = 64 * (len(pairs) + 64)
    rec = np.zeros(cap, np.uint32)
    slot = np.zeros(max(n_atoms, 1), np.int32)
    rc = lib.adx_debug_schedule(n_atoms, len(pairs), pairs.ctypes.data_as(C.c_void_p), C.byref(steps),
                                C.byref(slots), rec.ctypes.data_as(C.c_void_p), cap, slot.ctypes.data_as(C.c_void_p))
    assert rc == 0
    return steps.value, slots.value, rec[:steps.value * 64], slot[:n_atoms]


@pytest.mark.parametrize("n_atoms,n_tors,seed", [(12, 2, 1), (40, 8, 2), (110, 32, 3), (70, 20, 4), (200, 4, 5)])
def test_schedule_covers_pairs_with_distinct_targets(lib, n_atoms, n_tors, seed):
    L = synth.make_ligand(seed, n_atoms, n_tors, 8, chainlike=n_atoms > 80)
    R, K, rec, slot = _schedule(lib, L.n_atoms, L.pairs)
    npad = (L.n_atoms + 7) & ~7
    assert sorted(slot.tolist()) == sorted(set(slot.tolist())) and slot.max() < npad   # injective storage rows
    assert R * 64 >= L.n_pairs and 1 <= K <= 8
    i, j = rec & 0xff, (rec >> 8) & 0xff
    si, sj = (rec >> 16) & 0xf, (rec >> 20) & 0xf
    real = si != K                                                        # empty places: spare slot K
    got = sorted(tuple(sorted(p)) for p in zip(i[real].tolist(), j[real].tolist()))
    assert got == sorted(tuple(sorted(p)) for p in slot[L.pairs].tolist())  # every pair exactly once
    assert np.all(si[real] < K) and np.all(sj[real] < K)
    assert np.all(si[~real] == K) and np.all(sj[~real] == K)             # empty places -> spare row
    for r in range(R):
        s = slice(64 * r, 64 * r + 64)
        m = real[s]
        targets = np.concatenate([si[s][m] * npad + i[s][m], sj[s][m] * npad + j[s][m]])
        assert len(np.unique(targets)) == len(targets), f"step {r}: RMW targets collide"
    # the type-pair index keeps the caller's orientation
    assert np.all((rec >> 24)[real] == 0)


def test_schedule_empty_and_tiny(lib):
    R, K, rec, _ = _schedule(lib, 5, np.zeros((0, 2), np.int32))
    assert R == 0
    R, K, rec, _ = _schedule(lib, 2, [[0, 1]])
    assert R == 1 and (((rec >> 16) & 0xf) != K).sum() == 1


def _quarter_wavefronts(rec, npad):
    """128-bit shared accesses are serviced per quarter-warp (8 lanes): wavefronts of
    one access = max over bank groups (addr mod 8) of the distinct rows hit."""
    i, j = rec & 0xff, (rec >> 8) & 0xff
    si, sj = (rec >> 16) & 0xf, (rec >> 20) & 0xf
    total = 0
    for addr in (i, j, si * npad + i, sj * npad + j):
        for g in range(0, len(rec), 8):
            rows = set(addr[g:g + 8].tolist())
            total += max(np.bincount([r % 8 for r in rows], minlength=8))
    return total


@pytest.mark.parametrize("cfg,max_ratio", [(2, 1.1), (3, 1.0)])
def test_schedule_is_bank_conflict_free(lib, cfg, max_ratio):
    """Residue balancing + cross-step rebalancing + matching placement: the pair
    loop's X and gradient accesses hit (near) the ideal 1 wavefront per quarter-warp."""
    L = synth.make_config(cfg).ligands[0]
    R, K, rec, slot = _schedule(lib, L.n_atoms, L.pairs)
    assert R <= -(-L.n_pairs // 64) + 2
    npad = (L.n_atoms + 7) & ~7
    ideal = 4 * len(rec) // 8
    assert _quarter_wavefronts(rec, npad) <= max_ratio * ideal


# ---- cherry schedule (the shared-memory mode of the scatter pair loop) ----

def _cherries(lib, n_atoms, pairs, effort=2):
    pairs = np.ascontiguousarray(pairs, np.int32).reshape(-1, 2)
    steps, slots = C.c_int32(), C.c_int32()
    cap = 32 * (len(pairs) + 64)
    out = np.zeros((cap, 8), np.int32)
    slot = np.zeros(max(n_atoms, 1), np.int32)
    rc = lib.adx_debug_cherries(n_atoms, len(pairs), pairs.ctypes.data_as(C.c_void_p), effort, C.byref(steps),
                                C.byref(slots), out.ctypes.data_as(C.c_void_p), cap, slot.ctypes.data_as(C.c_void_p))
    assert rc == 0
    return steps.value, slots.value, out[:steps.value * 32], slot[:n_atoms]


@pytest.mark.parametrize("n_atoms,n_tors,seed", [(12, 2, 1), (40, 8, 2), (65, 16, 6), (20, 0, 7), (110, 32, 3)])
def test_cherries_cover_pairs_with_distinct_targets(lib, n_atoms, n_tors, seed):
    """Every pair is one end of exactly one cherry (c; e0, e1) whose two pairs share
    the centre c; per step the gradient targets (slot, row) of all centres and ends
    are distinct (the kernel's read-modify-writes are race-free without atomics).
    (110, 32): config 3's shape, whose 87-step schedule streams from global memory;
    the 8-bit row indices of the records cap the slots at K npad + 8 <= 256."""
    L = synth.make_ligand(seed, n_atoms, n_tors, 8, chainlike=n_atoms > 80)
    R, K, o, slot = _cherries(lib, L.n_atoms, L.pairs)
    npad = (L.n_atoms + 7) & ~7
    c, e, p, k = o[:, 0], o[:, 1:3], o[:, 3:5], o[:, 5:8]
    live = c >= 0
    assert 1 <= K <= 8 and np.all(k[live][:, 0] < K)
    assert K * npad + 8 <= 256
    got = []
    for lane in np.nonzero(live)[0]:
        for t in range(2):
            if p[lane, t] >= 0:
                got.append((p[lane, t], tuple(sorted((c[lane], e[lane, t])))))
            else:
                assert e[lane, t] < 0
    assert sorted(q for q, _ in got) == list(range(L.n_pairs))                  # every pair exactly once
    rows = slot[L.pairs]
    for q, ends in got:
        assert ends == tuple(sorted(rows[q]))                                    # ... as (centre, end)
    assert np.all(e[live][:, 0] != e[live][:, 1])                                # two different ends
    for r in range(R):
        s = slice(32 * r, 32 * r + 32)
        tg = [k[s][l, 0] * npad + c[s][l] for l in range(32) if c[s][l] >= 0]
        tg += [k[s][l, 1 + t] * npad + e[s][l, t] for l in range(32) for t in range(2) if c[s][l] >= 0 and e[s][l, t] >= 0]
        assert len(set(tg)) == len(tg), f"step {r}: targets collide"
        assert np.all(k[s][c[s] >= 0] < K)


def test_cherries_config2_shape(lib):
    """Config 2 (40 atoms, 510 pairs): 255 full cherries in 8 steps (the pair
    loop's 510 pairs take 8 steps of 64 either way) and a placement within 15 %
    of one wavefront per quarter-warp access."""
    L = synth.make_config(2).ligands[0]
    R, K, o, _ = _cherries(lib, L.n_atoms, L.pairs)
    assert R == 8 and K <= 6
    full = ((o[:, 3] >= 0) & (o[:, 4] >= 0)).sum()
    assert full == L.n_pairs // 2
    cost = 0
    for g in range(0, len(o), 8):
        Q = o[g:g + 8]
        Q = Q[Q[:, 0] >= 0]
        for acc in range(3):
            rows = Q[:, acc][Q[:, acc] >= 0]
            if len(rows):
                cost += np.bincount(rows & 7, minlength=8).max()
    assert cost <= 1.15 * 12 * R
