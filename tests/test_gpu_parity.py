"""GPU parity of the CUDA path (through the C ABI) against the FP64 oracle.

Gates (tests/parity.py): the Z18 energy gate |dE| <=
1e-3 + 2^-20 A_E on sane poses (A_E < 500), the labelled clash gate 1e-3 +
2^-20 (A_E + S_E) on clashing ones; gradient ||dg|| <= 1e-4 max(||g||, 1e-2
||A_grad||) on every pose.
Evaluations within 1e-4 A of a non-smooth point of the scoring function (grid
cell face / boundary, smoothing-band edge, cutoff; aux margins from the oracle)
may legitimately fall on the other side in FP32; they are counted, must stay
rare (< 2 %), and are excluded from the gate.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from oracle import oracle as O  # noqa: E402
from paper_conf_sc_solis_vasquezts25_b200 import synth  # noqa: E402
from tests.parity import energy_gate, energy_tol, grad_gate  # noqa: E402

pytestmark = pytest.mark.gpu
KINK = 1e-4


@pytest.fixture(scope="module")
def ad():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_solis_vasquezts25_b200 import ad as _ad
    return _ad


@pytest.fixture(scope="module")
def ctx(ad):
    c = ad.Context(0)
    yield c
    c.close()


_uploaded = {}


def _setup(ctx, w, key):
    """Upload grid + ligands of workload w (grid replaced when the key changes)."""
    if _uploaded.get("grid") != key:
        ctx.upload_grid(w.grid)
        _uploaded.clear()
        _uploaded["grid"] = key
    ids = []
    for k, L in enumerate(w.ligands):
        lk = (key, k)
        if lk not in _uploaded:
            _uploaded[lk] = ctx.upload_ligand(L, w.ff)
        ids.append(_uploaded[lk])
    return ids


def check_scores(L, grid, ff, genes, E, G=None, label=""):
    n = len(genes)
    Eo, Go, aux, ag = O.score(L, grid, ff, genes)
    kinkE = aux[:, O.AUX_MARGIN_E] < KINK
    kinkG = aux[:, O.AUX_MARGIN_G] < KINK
    gE = energy_gate(E, Eo, aux)
    okE = gE | kinkE
    assert okE.all(), f"{label}: {np.sum(~okE)} energies outside the gate, e.g. {np.nonzero(~okE)[0][:5]}"
    excused = ~gE
    if G is not None:
        Gn = L.n_genes
        gG = grad_gate(G[:, :Gn], Go[:, :Gn], ag[:, :Gn])
        okG = gG | kinkG | kinkE
        assert okG.all(), f"{label}: {np.sum(~okG)} gradients outside the gate, e.g. {np.nonzero(~okG)[0][:5]}"
        excused |= ~gG
    # gate misses are only ever excused at a kink, and stay rare
    assert excused.sum() <= max(1, int(0.02 * n)), f"{label}: {excused.sum()} kink-excused misses of {n}"
    return Eo, aux


@pytest.mark.parametrize("which,n", [("cfg1", 256), ("cfg2", 512), ("cfg3", 192)])
def test_score_poses_parity(ctx, which, n, request):
    w = request.getfixturevalue(which)
    (lid,) = _setup(ctx, w, which)
    L = w.ligands[0]
    g = torch.from_numpy(w.genes[:n]).cuda()
    E, G, A = ctx.score(lid, g, grad=True, aux=True)
    E0, _, _ = ctx.score(lid, g, grad=False)
    torch.cuda.synchronize()
    E, G, A, E0 = E.cpu().numpy(), G.cpu().numpy(), A.cpu().numpy(), E0.cpu().numpy()
    Eo, aux = check_scores(L, w.grid, w.ff, w.genes[:n], E, G, which)
    check_scores(L, w.grid, w.ff, w.genes[:n], E0, None, which + " energy-only")
    # aux: inter / intra split and Gtrans / Grigidrot consistency with the gradient
    tol = energy_tol(aux)
    assert np.all(np.abs(A[:, 0] - aux[:, O.AUX_EINTER]) <= tol)
    assert np.all(np.abs(A[:, 1] - aux[:, O.AUX_EINTRA]) <= tol)
    h = w.grid.spacing
    assert np.allclose(G[:, :3], h * A[:, 5:8], rtol=1e-5, atol=1e-5 * np.abs(G[:, :3]).max())
    # dE/dalpha = (pi/180) u . tau
    ph, th = np.radians(w.genes[:n, 3]), np.radians(w.genes[:n, 4])
    u = np.stack([np.sin(th) * np.cos(ph), np.sin(th) * np.sin(ph), np.cos(th)], 1)
    ga = np.radians(1.0) * np.sum(u * A[:, 2:5], 1)
    assert np.allclose(G[:, 5], ga, rtol=1e-4, atol=1e-4 * (np.abs(ga).max() + 1))


def _ls(ctx, lid, genes, engine, iters, **kw):
    g = torch.from_numpy(genes).cuda()
    nev = torch.zeros(1, dtype=torch.int64, device="cuda")
    out = ctx.local_search(lid, g, max_iters=iters, engine=engine, trace=True, n_evals=nev, **kw)
    torch.cuda.synchronize()
    return (out["trace"].cpu().numpy(), out["best_energy"].cpu().numpy(), g.cpu().numpy(), int(nev.item()), out)


@pytest.mark.parametrize("engine", ["simt", "tc", "paper", "paper_tcec"])
@pytest.mark.parametrize("which,n,iters", [("cfg1", 32, 40), ("cfg2", 32, 60), ("cfg3", 8, 12)])
def test_local_search_shadowed_parity(ctx, engine, which, n, iters, request):
    """Z19 (i): every traced step (genes_k, E_k, grad_k) re-evaluated by the oracle;
    each ADADELTA update re-applied in FP64 from the GPU's own gradient history."""
    w = request.getfixturevalue(which)
    (lid,) = _setup(ctx, w, which)
    L = w.ligands[0]
    Gn = L.n_genes
    wpc = 64 if engine.startswith("paper") else 0
    tr, bE, best_genes, nev, _ = _ls(ctx, lid, w.genes[:n], engine, iters, warps_per_cta=wpc)
    stride = w.genes.shape[1]
    assert nev == n * iters
    # best tracking: strict <, earliest wins; genes out = genes at that step
    k = np.argmin(tr[:, :, 0], axis=1)
    assert np.array_equal(bE, tr[np.arange(n), k, 0])
    assert np.array_equal(best_genes[:, :Gn], tr[np.arange(n), k, 1:1 + Gn])
    # step 0 evaluates the start genes exactly
    assert np.array_equal(tr[:, 0, 1:1 + Gn], w.genes[:n, :Gn])
    # per-step energy + gradient parity on a sample of steps
    rng = np.random.default_rng(0)
    sel = rng.choice(n * iters, size=min(n * iters, 160), replace=False)
    flat = tr.reshape(n * iters, -1)
    check_scores(L, w.grid, w.ff, flat[sel, 1:1 + stride], flat[sel, 0], flat[sel, 1 + stride:], f"{which} {engine}")
    # ADADELTA updates (FP64 replay of the GPU's gradients)
    for p in range(min(n, 8)):
        eg2 = np.zeros(Gn)
        ed2 = np.zeros(Gn)
        for s in range(iters - 1):
            x = tr[p, s, 1:1 + Gn].astype(np.float64)
            eg2, ed2, xn = O.adadelta_step(tr[p, s, 1 + stride:1 + stride + Gn], eg2, ed2, x)
            got = tr[p, s + 1, 1:1 + Gn].astype(np.float64)
            tol = 1e-5 * np.abs(xn - x) + 2.0 ** -22 * np.abs(xn) + 1e-30
            assert np.all(np.abs(got - xn) <= tol), (p, s)


def test_run_best_and_determinism(ctx, cfg2):
    (lid,) = _setup(ctx, cfg2, "cfg2")
    n, pop = 600, 150
    outs = []
    for _ in range(2):
        g = torch.from_numpy(cfg2.genes[:n]).cuda()
        o = ctx.local_search(lid, g, max_iters=20, engine="tc", pop_per_run=pop)
        torch.cuda.synchronize()
        outs.append((o["best_energy"].cpu().numpy(), o["run_best"].cpu().numpy(), g.cpu().numpy()))
    bE, rb, genes = outs[0]
    assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][2], outs[1][2]), "not deterministic"
    for r in range(n // pop):
        i = r * pop + int(np.argmin(bE[r * pop:(r + 1) * pop]))
        assert rb[r, 0] == bE[i]
        assert np.array_equal(rb[r, 1:], genes[i])
    ref = O.best_of_run(bE.astype(np.float64), pop)
    assert np.array_equal(ref, [r * pop + int(np.argmin(bE[r * pop:(r + 1) * pop])) for r in range(n // pop)])


def test_engines_agree_on_first_steps(ctx, cfg2):
    (lid,) = _setup(ctx, cfg2, "cfg2")
    trs = {e: _ls(ctx, lid, cfg2.genes[:16], e, 3, warps_per_cta=(64 if e.startswith("paper") else 0))[0]
           for e in ("simt", "tc", "paper", "paper_tcec")}
    for e in ("tc", "paper", "paper_tcec"):
        d = np.abs(trs[e][:, 0, 0].astype(np.float64) - trs["simt"][:, 0, 0])
        assert np.all(d <= 1e-5 * np.abs(trs["simt"][:, 0, 0]) + 1e-3)


@pytest.mark.parametrize("which,engine", [("cfg2", "simt"), ("cfg2", "tc"), ("cfg3", "simt")])
def test_full_size_sampled(ctx, which, engine, request):
    """BASELINE configs 2 and 3 at full size (3000 / 15000 poses x 300 iterations) in
    the bench launch configuration (library-chosen CTA shape and register variant;
    simt = the bench default engine): properties on all poses (on the device),
    oracle parity on sampled evaluations of the trace."""
    w = request.getfixturevalue(which)
    (lid,) = _setup(ctx, w, which)
    L = w.ligands[0]
    stride = w.genes.shape[1]
    n, iters = w.n_poses, w.iters
    g = torch.from_numpy(w.genes).cuda()
    nev = torch.zeros(1, dtype=torch.int64, device="cuda")
    out = ctx.local_search(lid, g, max_iters=iters, engine=engine, trace=True, n_evals=nev, pop_per_run=w.pop)
    torch.cuda.synchronize()
    tr = out["trace"].view(n, iters, -1)
    bE = out["best_energy"]
    assert int(nev.item()) == n * iters
    assert torch.equal(bE, tr[:, :, 0].min(dim=1).values)
    assert bool(torch.isfinite(bE).all())
    # the search makes progress: best energy well below the start energy for most poses
    assert float((bE < tr[:, 0, 0]).float().mean()) > 0.9
    rng = np.random.default_rng(1)
    sel = torch.from_numpy(rng.choice(n * iters, size=96, replace=False)).cuda()
    flat = tr.reshape(n * iters, -1)[sel].cpu().numpy()
    del out, tr
    check_scores(L, w.grid, w.ff, flat[:, 1:1 + stride], flat[:, 0], flat[:, 1 + stride:], f"{which} full {engine}")


def test_edge_cases(ctx, ad):
    from tests.util import hand_ligand
    grid = synth.make_grid(77, 24, synth.TYPESETS[3], 100)
    ff = synth.FFParams()
    _uploaded.clear()
    ctx.upload_grid(grid)
    # rigid ligand (no torsions, no pairs) and a single atom
    rigid = hand_ligand([[0, 0, 0], [1.5, 0, 0], [1.5, 1.5, 0]], types=[0, 1, 2], charges=[0.2, -0.3, 0.1],
                        tp=np.tile(np.array([0, 0, 4, 12, 6], np.float32), (3, 3, 1)))
    one = hand_ligand([[0, 0, 0]], types=[1], charges=[0.4], tp=np.tile(np.array([0, 0, 4, 12, 6], np.float32), (2, 2, 1)))
    for L in (rigid, one):
        lid = ctx.upload_ligand(L, ff)
        genes = synth.make_genotypes(3, 40, 0, grid)
        genes[0, :3] = [-5.0, 3.0, 4.0]           # out of the grid
        genes[1, :3] = [40.0, 40.0, 40.0]
        g = torch.from_numpy(genes).cuda()
        E, G, _ = ctx.score(lid, g)
        torch.cuda.synchronize()
        check_scores(L, grid, ff, genes, E.cpu().numpy(), G.cpu().numpy(), "edge")
        tr, bE, *_ = _ls(ctx, lid, genes, "simt", 5)
        assert np.all(np.isfinite(bE))
    # n_poses == 0 is a no-op
    lid = ctx.upload_ligand(rigid, ff)
    e = torch.empty(0, 6, device="cuda")
    ad.ad_score_poses(ctx.h, lid, None, e, torch.empty(0, device="cuda"))
    ad.ad_local_search(ctx.h, lid, None, e, torch.empty(0, device="cuda"))
    # argument errors
    with pytest.raises(ad.AdError) as ex:
        ad.ad_score_poses(ctx.h, 10 ** 6, None, torch.zeros(4, 6, device="cuda"), torch.empty(4, device="cuda"))
    assert ex.value.code == ad.AD_ERR_INVALID_ARG
    with pytest.raises(ad.AdError):
        ad.ad_score_poses(ctx.h, lid, None, torch.zeros(4, 5, device="cuda"), torch.empty(4, device="cuda"))
    with pytest.raises(ad.AdError):
        ctx.local_search(lid, torch.zeros(4, 6, device="cuda"), engine=7)
    # out-of-range pose_ligand ids surface on the next call
    pl = torch.tensor([lid, 9999, lid, lid], dtype=torch.int32, device="cuda")
    ad.ad_score_poses(ctx.h, lid, pl, torch.zeros(4, 6, device="cuda"), torch.empty(4, device="cuda"))
    torch.cuda.synchronize()
    with pytest.raises(ad.AdError) as ex:
        ad.ad_score_poses(ctx.h, lid, None, torch.zeros(4, 6, device="cuda"), torch.empty(4, device="cuda"))
    assert ex.value.code == ad.AD_ERR_INVALID_ARG
    _uploaded.clear()


def test_large_ligand_limits(ctx):
    """Biggest shapes: 58 torsions (64 genes) and 200 atoms."""
    grid = synth.make_grid(78, 96, synth.TYPESETS[8], 3000)
    ff = synth.FFParams()
    _uploaded.clear()
    ctx.upload_grid(grid)
    for seed, n_at, n_t in ((1, 150, 58), (2, 200, 4)):
        L = synth.make_ligand(seed, n_at, n_t, 8, chainlike=True)
        lid = ctx.upload_ligand(L, ff)
        genes = synth.make_genotypes(seed, 24, n_t, grid, frac=0.1)
        g = torch.from_numpy(genes).cuda()
        E, G, _ = ctx.score(lid, g)
        torch.cuda.synchronize()
        check_scores(L, grid, ff, genes, E.cpu().numpy(), G.cpu().numpy(), f"N={n_at} T={n_t}")
    _uploaded.clear()


def test_multi_ligand_pose_ligand(ctx, ad):
    grid = synth.make_grid(79, 40, synth.TYPESETS[6], 800)
    ff = synth.FFParams()
    _uploaded.clear()
    ctx.upload_grid(grid)
    ligs = [synth.make_ligand(100 + k, n, t, 6) for k, (n, t) in enumerate(((30, 5), (18, 3), (36, 9)))]
    ids = [ctx.upload_ligand(L, ff) for L in ligs]
    big = max(range(3), key=lambda k: ligs[k].n_pairs)
    per = 8
    stride = 6 + max(L.n_tors for L in ligs)
    genes = np.zeros((3 * per, stride), np.float32)
    pl = np.repeat(np.array(ids, np.int32), per)
    for k, L in enumerate(ligs):
        genes[k * per:(k + 1) * per] = synth.make_genotypes(k, per, L.n_tors, grid, stride=stride, frac=0.3)
    g = torch.from_numpy(genes).cuda()
    E = torch.empty(3 * per, device="cuda")
    Gd = torch.zeros(3 * per, stride, device="cuda")
    ad.ad_score_poses(ctx.h, ids[big], torch.from_numpy(pl).cuda(), g, E, Gd)
    torch.cuda.synchronize()
    for k, L in enumerate(ligs):
        s = slice(k * per, (k + 1) * per)
        check_scores(L, grid, ff, genes[s], E.cpu().numpy()[s], Gd.cpu().numpy()[s], f"ligand {k}")
    _uploaded.clear()


def test_launch_set_and_id_reuse(ad):
    """ad_set_launch_ligands: pose_ligand launches are sized for the launch set
    only; a pose whose ligand is outside the set's footprint is reported on the
    next call (device-side check); freed ids are reused."""
    grid = synth.make_grid(81, 40, synth.TYPESETS[6], 800)
    ff = synth.FFParams()
    c = ad.Context(0)
    try:
        c.upload_grid(grid)
        small, large = synth.make_ligand(201, 16, 2, 6), synth.make_ligand(202, 60, 12, 6)
        i_s, i_l = c.upload_ligand(small, ff), c.upload_ligand(large, ff)
        stride = 6 + 12
        genes = np.concatenate([synth.make_genotypes(1, 8, 2, grid, stride=stride, frac=0.3),
                                synth.make_genotypes(2, 8, 12, grid, stride=stride, frac=0.3)])
        pl = torch.tensor([i_s] * 8 + [i_l] * 8, dtype=torch.int32, device="cuda")
        g = torch.from_numpy(genes).cuda()
        E = torch.empty(16, device="cuda")
        # the small ligand alone: the large ligand's poses must be flagged
        c.set_launch_ligands([i_s])
        ad.ad_score_poses(c.h, i_s, pl, g, E)
        torch.cuda.synchronize()
        with pytest.raises(ad.AdError):
            ad.ad_score_poses(c.h, i_s, pl[:8], g[:8], E[:8])
        # both ligands: every pose scores, and matches the oracle
        c.set_launch_ligands([i_s, i_l])
        ad.ad_score_poses(c.h, i_l, pl, g, E)
        torch.cuda.synchronize()
        Eh = E.cpu().numpy()
        check_scores(small, grid, ff, genes[:8, :8], Eh[:8], label="small")
        check_scores(large, grid, ff, genes[8:], Eh[8:], label="large")
        with pytest.raises(ad.AdError):
            c.set_launch_ligands([i_l + 5])  # not a live ligand
        c.set_launch_ligands(None)
        c.free_ligand(i_s)
        assert c.upload_ligand(small, ff) == i_s  # lowest free id is reused
    finally:
        c.close()


@pytest.mark.parametrize("effort", [0, 1])
def test_schedule_effort_parity(ad, cfg2, effort):
    """A cheaper pair-schedule placement evaluates the same pairs: oracle parity
    holds and energies agree with the default placement to FP32 rounding."""
    L = cfg2.ligands[0]
    c = ad.Context(0)
    try:
        c.upload_grid(cfg2.grid)
        ref = c.upload_ligand(L, cfg2.ff)
        c.set_schedule_effort(effort)
        lid = c.upload_ligand(L, cfg2.ff)
        g = torch.from_numpy(cfg2.genes[:128]).cuda()
        E0, G0, _ = c.score(ref, g)
        E1, G1, _ = c.score(lid, g)
        torch.cuda.synchronize()
        check_scores(L, cfg2.grid, cfg2.ff, cfg2.genes[:128], E1.cpu().numpy(), G1.cpu().numpy(), f"effort {effort}")
        Eo, *_ = O.score(L, cfg2.grid, cfg2.ff, cfg2.genes[:128])
        d = np.abs(E1.cpu().numpy().astype(np.float64) - E0.cpu().numpy())
        assert np.all(d <= 1e-5 * np.abs(Eo) + 1e-3)
        with pytest.raises(ad.AdError):
            c.set_schedule_effort(3)
    finally:
        c.close()


@pytest.mark.parametrize("engine", ["simt", "tc", "paper", "paper_tcec"])
def test_phase_instrumentation(ctx, cfg2, engine):
    """A14: the instrumented kernel computes exactly what the plain kernel computes
    (same arithmetic, FMA contraction off) and reports positive cycles for every
    phase; the reduction share f is a proper fraction."""
    (lid,) = _setup(ctx, cfg2, "cfg2")
    wpc = 64 if engine.startswith("paper") else 0
    outs = []
    for phases in (False, True):
        g = torch.from_numpy(cfg2.genes[:300]).cuda()
        o = ctx.local_search(lid, g, max_iters=20, engine=engine, warps_per_cta=wpc, phases=phases)
        torch.cuda.synchronize()
        outs.append((o["best_energy"].cpu().numpy(), g.cpu().numpy(), o["phase_cycles"]))
    if engine.startswith("paper"):
        # the paper-style kernel accumulates intra gradients with shared-memory float
        # atomics (order not fixed): equal up to rounding, not bit for bit
        d = np.abs(outs[0][0].astype(np.float64) - outs[1][0])
        assert np.mean(d > 1e-2 * (1 + np.abs(outs[0][0]))) < 0.05
    else:
        assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][1], outs[1][1])
    ph = outs[1][2].cpu().numpy()
    assert ph.shape == (300, 5) and np.all(ph > 0)
    f = ph[:, 3].sum() / ph.sum()
    assert 0.0 < f < 0.5


@pytest.mark.parametrize("engine", ["simt", "tc", "paper"])
def test_reduction_engines_accuracy(ctx, ad, engine):
    """Config 4: |S - S_exact| <= (ceil(log2 P) + 2) 2^-24 sum|x| (O-7)."""
    import math
    for P in (128, 256, 512, 1024):
        for Cc in (8, 16, 24, 32, 40):
            for dist in ("uniform", "logmag"):
                x = synth.make_reduction_partials(P * 7 + Cc, 64, P, Cc, dist)
                xd = torch.from_numpy(x).cuda()
                o = torch.empty(64, Cc, device="cuda")
                ad.ad_reduce_blocks(ctx.h, ad.ENGINES[engine], xd, o)
                torch.cuda.synchronize()
                o = o.cpu().numpy().astype(np.float64)
                ex = np.array([[math.fsum(x[b, :, c].astype(np.float64)) for c in range(Cc)] for b in range(64)])
                bound = (math.ceil(math.log2(P)) + 2) * 2.0 ** -24 * np.abs(x.astype(np.float64)).sum(axis=1)
                assert np.all(np.abs(o - ex) <= bound), (P, Cc, dist)


def test_reduction_fp16_no_ec_accuracy(ctx, ad):
    """NEXT-2, config 4: the Schieffer-Peng FP16 reduction without EC (Lst 1
    bottom) is correct to FP16 accuracy -- |S - S_exact| <=
    (4 + n_warps) 2^-11 sum|x| -- and measurably worse than TCEC (the Fig 1 vs
    Fig 3 finding, P:L177 / P:L199); large partials overflow FP16."""
    import math
    errs = {"tc": [], "tc_fp16": []}
    for P in (128, 256, 1024):
        Cc = 16
        x = synth.make_reduction_partials(P * 7 + Cc, 64, P, Cc, "uniform")
        xd = torch.from_numpy(x).cuda()
        ex = np.array([[math.fsum(x[b, :, c].astype(np.float64)) for c in range(Cc)] for b in range(64)])
        for eng in errs:
            o = torch.empty(64, Cc, device="cuda")
            ad.ad_reduce_blocks(ctx.h, ad.ENGINES[eng], xd, o)
            torch.cuda.synchronize()
            err = np.abs(o.cpu().numpy().astype(np.float64) - ex)
            errs[eng].append(err.ravel())
            if eng == "tc_fp16":
                bound = (4 + P // 32) * 2.0 ** -11 * np.abs(x.astype(np.float64)).sum(axis=1)
                assert np.all(err <= bound), P
    e16, etc = np.concatenate(errs["tc_fp16"]), np.concatenate(errs["tc"])
    assert np.median(e16) > 100 * max(np.median(etc), 1e-12)
    # magnitudes beyond FP16's range (65504) overflow without EC / TF32's exponent
    x = synth.make_reduction_partials(99, 8, 256, 8, "logmag")
    o = torch.empty(8, 8, device="cuda")
    ad.ad_reduce_blocks(ctx.h, ad.ENGINES["tc_fp16"], torch.from_numpy(x).cuda(), o)
    torch.cuda.synchronize()
    assert not np.all(np.isfinite(o.cpu().numpy()))


def test_local_search_fp16_engine(ctx, cfg2):
    """NEXT-2: the warp kernel with every sum on FP16 tensor cores without EC.
    On relaxed poses (sums within FP16 range) energies stay within FP16
    accumulation error of the oracle, and its gradient error is an order of
    magnitude above the error-corrected TF32 engine's (P:L177 vs P:L199)."""
    w = cfg2
    (lid,) = _setup(ctx, w, "cfg2")
    L = w.ligands[0]
    Gn = L.n_genes
    n = 64
    # relax start poses with the TC engine first (clashing starts overflow FP16)
    _, _, relaxed, _, _ = _ls(ctx, lid, w.genes[:n], "tc", 300)
    res = {}
    for eng in ("tc", "tc_fp16"):
        tr, _, _, nev, _ = _ls(ctx, lid, relaxed, eng, 1)
        assert nev == n
        res[eng] = tr[:, 0]
    stride = w.genes.shape[1]
    Eo, Go, aux, ag = O.score(L, w.grid, w.ff, relaxed)
    e16 = res["tc_fp16"][:, 0].astype(np.float64)
    assert np.all(np.isfinite(e16))
    assert np.all(np.abs(e16 - Eo) <= energy_tol(aux) + 34 * 2.0 ** -11 * aux[:, O.AUX_ABS_E])
    rel = {}
    for eng in res:
        g = res[eng][:, 1 + stride:1 + stride + Gn].astype(np.float64)
        rel[eng] = np.linalg.norm(g - Go[:, :Gn], axis=1) / np.maximum(np.linalg.norm(Go[:, :Gn], axis=1), 1e-6)
    assert np.median(rel["tc_fp16"]) > 10 * np.median(rel["tc"])
    assert np.median(rel["tc_fp16"]) < 0.05


@pytest.mark.parametrize("mode", ["owner", "hybrid"])
def test_alternative_intra_modes(ad, cfg2, mode, monkeypatch):
    """The two non-default pair-loop designs (AD_INTRA_MODE, read at context
    creation): same parity gates as the default scatter schedule, and
    the same LS trajectories to FP32 accuracy on the first steps."""
    monkeypatch.setenv("AD_INTRA_MODE", mode)
    c = ad.Context(0)
    try:
        w = cfg2
        c.upload_grid(w.grid)
        lid = c.upload_ligand(w.ligands[0], w.ff)
        n = 128
        g = torch.from_numpy(w.genes[:n]).cuda()
        E, G, _ = c.score(lid, g, grad=True)
        torch.cuda.synchronize()
        check_scores(w.ligands[0], w.grid, w.ff, w.genes[:n], E.cpu().numpy(), G.cpu().numpy(), f"cfg2 {mode}")
        tr, _, _, nev, _ = _ls(c, lid, w.genes[:16], "simt", 20)
        assert nev == 16 * 20
        stride = w.genes.shape[1]
        flat = tr.reshape(16 * 20, -1)
        check_scores(w.ligands[0], w.grid, w.ff, flat[::7, 1:1 + stride], flat[::7, 0], flat[::7, 1 + stride:],
                     f"cfg2 {mode} LS")
    finally:
        c.close()


@pytest.mark.parametrize("smooth", [0.5, 0.0])
def test_cherry_schedule_shapes(ctx, smooth):
    """The cherry pair loop (shared-memory schedules) on ligands that exercise its
    corner cases: a tiny ligand (empty lanes, singles), odd pair counts, 33-64 atoms
    (second atoms taken from the root fragment), no torsions; and smooth = 0 (no
    flat band: empty ends must read two distinct zero-charge rows, or their zero
    coefficients would multiply 1/0).  Score with gradients + a short shadowed LS."""
    grid = synth.make_grid(91, 40, synth.TYPESETS[8], 600)
    ff = synth.FFParams(smooth=smooth)
    _uploaded.clear()
    ctx.upload_grid(grid)
    for seed, n_atoms, n_tors in [(11, 9, 1), (12, 23, 5), (13, 33, 6), (14, 50, 12), (15, 30, 0)]:
        L = synth.make_ligand(seed, n_atoms, n_tors, 8)
        lid = ctx.upload_ligand(L, ff)
        genes = synth.make_genotypes(seed, 96, n_tors, grid)
        g = torch.from_numpy(genes).cuda()
        E, G, _ = ctx.score(lid, g)
        torch.cuda.synchronize()
        check_scores(L, grid, ff, genes, E.cpu().numpy(), G.cpu().numpy(), f"cherry n={n_atoms} smooth={smooth}")
        tr, bE, *_ = _ls(ctx, lid, genes[:16], "simt", 8)
        assert np.all(np.isfinite(bE)) and np.all(bE == tr[:, :, 0].min(axis=1))
        for it in (0, 7):  # the trace's energies are the oracle's energies of the traced genes
            Eo, _, aux, _ = O.score(L, grid, ff, tr[:, it, 1:1 + genes.shape[1]])
            assert np.all(energy_gate(tr[:, it, 0], Eo, aux) | (aux[:, O.AUX_MARGIN_E] < KINK))
    _uploaded.clear()
