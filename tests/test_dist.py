"""Multi-rank host logic of paper_conf_sigmod_liuhh16_b200.dist on CPU (gloo, world 2).

The path shards (instances are independent): groups are split over ranks with no
data-path collective; the only collectives are the end-of-run MAX of the time and the
gather of per-source m_s / digests.  The runner here is the CPU oracle (test
infrastructure), standing in for Graph.run so the sharding and gathering logic is
exercised without a GPU.
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

import ibfs_gen
import oracle
from paper_conf_sigmod_liuhh16_b200 import dist as pdist


def test_shard_groups_partition_and_determinism():
    rng = np.random.default_rng(1)
    for ng in (1, 5, 32, 2048):
        costs = rng.random(ng) * (rng.random(ng) > 0.3)
        for world in (1, 2, 3, 8):
            for pol in ("lpt", "round_robin"):
                parts = [pdist.shard_groups(ng, world, r, costs, pol) for r in range(world)]
                allg = np.sort(np.concatenate(parts))
                np.testing.assert_array_equal(allg, np.arange(ng))
                again = [pdist.shard_groups(ng, world, r, costs, pol) for r in range(world)]
                for a, b in zip(parts, again):
                    np.testing.assert_array_equal(a, b)
    with pytest.raises(ValueError):
        pdist.shard_groups(4, 2, 2)


def test_lpt_balances_skewed_costs():
    # c4-like plan order: hub groups first, then near-free isolated-source groups
    costs = np.concatenate([np.full(100, 50.0), np.full(60, 0.0), np.full(40, 10.0)])
    world = 4
    loads = [costs[pdist.shard_groups(len(costs), world, r, costs, "lpt")].sum() for r in range(world)]
    assert max(loads) - min(loads) <= 50.0
    contiguous = [costs[r * 50:(r + 1) * 50].sum() for r in range(world)]
    assert max(loads) < max(contiguous)


def test_rows_of_groups_ragged_tail():
    rows = pdist.rows_of_groups(np.array([0, 2]), 70, 32)
    np.testing.assert_array_equal(rows, np.concatenate([np.arange(32), np.arange(64, 70)]))


def test_group_costs_isolated_zero():
    deg = np.array([0, 3, 0, 100], dtype=np.int64)
    c = pdist.group_costs(np.array([0, 2, 1, 3], dtype=np.uint32), deg, 2)
    assert c[0] == 0.0 and c[1] > 0


def _free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        cfg = ibfs_gen.CONFIGS["c1"]
        el = cfg.edges(threads=1)
        src = np.arange(0, el.nv, 5, dtype=np.uint32)  # 205 sources: ragged last group
        og = oracle.OracleGraph.from_edges(el)
        deg = og.degrees().astype(np.int64)
        costs = pdist.group_costs(src, deg, 64)

        def runner(s):
            r = og.bfs(s, threads=1)
            return r.depths, r.m_s, r.digest, 1.0 + rank

        res = pdist.run_sharded(src, 64, runner, world=world, rank=rank, costs=costs, policy="lpt")
        q.put((rank, res.rows.tolist(), res.max_ms, res.m_s.tolist(), res.digest.tolist(),
               res.edges_traversed, res.depths.tolist()))
    finally:
        dist.destroy_process_group()


def test_run_sharded_gloo_world2():
    import multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    out.sort()
    cfg = ibfs_gen.CONFIGS["c1"]
    el = cfg.edges(threads=1)
    src = np.arange(0, el.nv, 5, dtype=np.uint32)
    ref = oracle.bfs(el, src)
    rows0, rows1 = np.array(out[0][1]), np.array(out[1][1])
    assert len(np.intersect1d(rows0, rows1)) == 0
    np.testing.assert_array_equal(np.sort(np.concatenate([rows0, rows1])), np.arange(len(src)))
    for rank, rows, max_ms, m_s, dig, edges, depths in out:
        assert max_ms == 2.0  # MAX over ranks of (1 + rank)
        np.testing.assert_array_equal(np.array(m_s, dtype=np.uint64), ref.m_s)
        np.testing.assert_array_equal(np.array(dig, dtype=np.uint64), ref.digest)
        assert edges == int(ref.m_s.sum())
        np.testing.assert_array_equal(np.array(depths, dtype=np.int8), ref.depths[np.array(rows)])
