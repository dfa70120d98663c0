"""Multi-GPU host logic on CPU: LPT sharding of independent (ligand, run) units
and the final gather of best-pose records, over a world_size-2 gloo group."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sc_solis_vasquezts25_b200 import dist as addist


def test_lpt_balances_and_covers():
    rng = np.random.default_rng(0)
    costs = rng.uniform(1, 100, 500).tolist()
    for n in (1, 2, 4, 8):
        shards = addist.lpt_shard(costs, n)
        flat = sorted(u for s in shards for u in s)
        assert flat == list(range(500))
        loads = [sum(costs[u] for u in s) for s in shards]
        # LPT guarantee: max load <= 4/3 OPT; OPT >= mean and >= max unit
        opt_lb = max(sum(costs) / n, max(costs))
        assert max(loads) <= 4.0 / 3.0 * opt_lb + 1e-9
    assert addist.lpt_shard([], 3) == [[], [], []]
    with pytest.raises(ValueError):
        addist.lpt_shard([1.0], 0)


def test_unit_cost_monotone():
    a = addist.unit_cost(40, 8, 510, 150, 300)
    b = addist.unit_cost(110, 32, 5548, 150, 300)
    assert b > 5 * a > 0


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    # each rank owns the runs LPT assigned to it; records are [E, genes...]
    costs = [float(c) for c in np.random.default_rng(1).integers(1, 10, 12)]
    shards = addist.lpt_shard(costs, world)
    mine = shards[rank]
    width = 1 + 8
    n_max = max(len(s) for s in shards)
    rec = torch.full((n_max, width + 1), float("nan"))
    for k, u in enumerate(mine):
        rec[k, 0] = float(u)                       # unit id
        rec[k, 1] = -float(u) * 0.5                # best energy
        rec[k, 2:] = torch.arange(8, dtype=torch.float32) + u
    got = addist.gather_records(rec)
    if rank == 0:
        out.put(got.numpy())
    dist.barrier()
    dist.destroy_process_group()


def test_gather_records_gloo_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    got = q.get(timeout=120)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    rows = got[~np.isnan(got[:, 0])]
    assert sorted(rows[:, 0].astype(int).tolist()) == list(range(12))
    for r in rows:
        u = int(r[0])
        assert r[1] == -u * 0.5 and np.array_equal(r[2:], np.arange(8) + u)


def test_gather_is_identity_without_process_group():
    t = torch.arange(6.0).reshape(2, 3)
    assert addist.gather_records(t) is t
