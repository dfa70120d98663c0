"""The multi-GPU path (Alg 1 coarse level)
through the real kernels: two ranks (gloo, both on cuda:0 -- the box has one
GPU) each run their LPT shard of a screen and of config-3 runs, then gather the
best-pose records.  The gathered records must equal a one-rank run's bit for
bit: every pose's search is deterministic and independent of the launch shape
(ptxas --fmad=false, one warp per pose), so sharding cannot change a result."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _screen_inputs():
    from paper_conf_sc_solis_vasquezts25_b200 import synth
    rng = np.random.default_rng(11)
    grid = synth.make_grid(5200, 40, synth.TYPESETS[8], 800)
    ligs = []
    for k in range(10):
        n = int(rng.integers(20, 60))
        t = int(rng.integers(0, min(10, n // 3) + 1))
        ligs.append(synth.make_ligand(900 + k, n, t, 8))
    runs, pop, iters, stride = 3, 12, 20, 6 + 10
    genes = np.concatenate([synth.make_genotypes(k, runs * pop, L.n_tors, grid, stride=stride, frac=0.3)
                            for k, L in enumerate(ligs)])
    return grid, ligs, genes, runs, pop, iters


def _cfg3_runs(ctx, rank, world, runs=6, pop=8, iters=10):
    """Config-3 runs LPT-sharded over the ranks (equal costs: round robin by LPT),
    each rank's run records [run id, E, genes] gathered."""
    from paper_conf_sc_solis_vasquezts25_b200 import dist as addist, synth
    w = synth.make_config(3, runs=runs, pop=pop, iters=iters)
    L = w.ligands[0]
    shards = addist.lpt_shard([1.0] * runs, world)
    mine = shards[rank]
    n_max = max(len(s) for s in shards)
    ctx.upload_grid(w.grid)
    lid = ctx.upload_ligand(L, w.ff)
    rec = torch.full((n_max, 2 + w.genes.shape[1]), float("nan"), device="cuda")
    if mine:
        g = torch.from_numpy(np.concatenate([w.genes[r * pop:(r + 1) * pop] for r in mine])).cuda()
        out = ctx.local_search(lid, g, max_iters=iters, pop_per_run=pop)
        rec[:len(mine), 0] = torch.tensor(mine, dtype=torch.float32, device="cuda")
        rec[:len(mine), 1:] = out["run_best"]
    ctx.sync()
    return addist.gather_records(rec)


def _worker(rank, world, port, path):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch.distributed as dist

    from paper_conf_sc_solis_vasquezts25_b200 import ad, screen, synth
    if world > 1:
        dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    ctx = ad.Context(0)
    try:
        grid, ligs, genes, runs, pop, iters = _screen_inputs()
        rec, units = screen.run_screen(ctx, grid, synth.FFParams(), ligs, genes, runs, pop, iters, rank=rank,
                                       world=world, n_buckets=2)
        rec3 = _cfg3_runs(ctx, rank, world)
        if rank == 0:
            np.savez(path, screen=rec.cpu().numpy(), cfg3=rec3.cpu().numpy())
    finally:
        ctx.close()
        if world > 1:
            dist.barrier()
            dist.destroy_process_group()


def _run(world, path):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, path)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=600)
        assert p.exitcode == 0
    return np.load(path)


def _by_key(rec, key_cols):
    rows = rec[~np.isnan(rec[:, 0])]
    return {tuple(int(v) for v in r[:key_cols]): r[key_cols:] for r in rows}


def test_two_ranks_match_one_rank(tmp_path):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    one = _run(1, str(tmp_path / "one.npz"))
    two = _run(2, str(tmp_path / "two.npz"))
    s1, s2 = _by_key(one["screen"], 2), _by_key(two["screen"], 2)
    assert sorted(s1) == sorted(s2) and len(s1) == 10 * 3
    for k in s1:
        assert np.array_equal(s1[k], s2[k], equal_nan=True), k
    c1, c2 = _by_key(one["cfg3"], 1), _by_key(two["cfg3"], 1)
    assert sorted(c1) == sorted(c2) == [(r,) for r in range(6)]
    for k in c1:
        assert np.array_equal(c1[k], c2[k]), k
