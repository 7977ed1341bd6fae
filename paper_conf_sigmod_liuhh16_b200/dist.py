"""Multi-GPU sharding of GroupBy groups over torch.distributed ranks (one process per GPU).

PAPER.md P:L1019: "as long as different GPUs work on independent BFSes, there is no need
for inter-GPU communication ... The longest time consumption of all the GPUs is
reported."  So: the graph is replicated on every rank (each rank builds it from the same
seed), every rank computes the same plan, groups are assigned by a deterministic policy,
each rank traverses its groups with no data-path collective, and the only collectives are
at the end: all_reduce(MAX) of the device time and all_gather of per-source (m_s, digest).
Depth rows stay on their rank.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


def group_costs(sources_plan_order: np.ndarray, deg: np.ndarray, group_bits: int) -> np.ndarray:
    """Cost proxy per group: sources of degree > 0 (an isolated source finishes at level 0)
    weighted by 1 + log2(1 + deg) (hub sources reach the giant component sooner)."""
    n = len(sources_plan_order)
    ng = (n + group_bits - 1) // group_bits
    d = deg[np.asarray(sources_plan_order, dtype=np.int64)].astype(np.float64)
    w = np.where(d > 0, 1.0 + np.log2(1.0 + d), 0.0)
    pad = ng * group_bits - n
    if pad:
        w = np.concatenate([w, np.zeros(pad)])
    return w.reshape(ng, group_bits).sum(axis=1)


def shard_groups(n_groups: int, world: int, rank: int, costs: np.ndarray | None = None,
                 policy: str = "lpt") -> np.ndarray:
    """Group ids of `rank`.  'round_robin': g % world == rank.  'lpt': longest processing
    time first -- groups by descending cost (ties: lower id) to the least-loaded rank
    (ties: lower rank).  Deterministic, identical on every rank."""
    if world < 1 or not (0 <= rank < world):
        raise ValueError("bad world/rank")
    if policy == "round_robin" or costs is None:
        return np.arange(rank, n_groups, world, dtype=np.int64)
    if policy != "lpt":
        raise ValueError(policy)
    order = sorted(range(n_groups), key=lambda gi: (-float(costs[gi]), gi))
    load = [0.0] * world
    mine = []
    for gi in order:
        r = min(range(world), key=lambda x: (load[x], x))
        load[r] += float(costs[gi])
        if r == rank:
            mine.append(gi)
    return np.asarray(sorted(mine), dtype=np.int64)


def rows_of_groups(group_ids: np.ndarray, n: int, group_bits: int) -> np.ndarray:
    """Row indices (into the plan-ordered source list) covered by these groups."""
    rows = [np.arange(gi * group_bits, min((gi + 1) * group_bits, n)) for gi in group_ids]
    return np.concatenate(rows) if rows else np.zeros(0, dtype=np.int64)


@dataclass
class ShardResult:
    group_ids: np.ndarray        # this rank's groups
    rows: np.ndarray             # this rank's rows (indices into the plan-ordered sources)
    depths: object               # this rank's depth rows (device tensor), row i <-> rows[i]
    local_ms: float              # this rank's device traversal time
    max_ms: float                # max over ranks (the reported time)
    m_s: np.ndarray              # [n] m_s of every source (all ranks)
    digest: np.ndarray | None    # [n] digests of every source (all ranks) or None
    edges_traversed: int         # sum over all ranks


def run_sharded(sources_plan_order, group_bits: int, runner, world: int = 1, rank: int = 0,
                costs=None, policy: str = "lpt", group=None, want_digest: bool = True,
                device=None) -> ShardResult:
    """Run this rank's groups with `runner(rank_sources) -> (depths, m_s, digest, ms)`
    (normally ``lambda s: graph.run(s, group_bits, ...)`` unpacked), then gather.

    Collectives (torch.distributed, NCCL on GPUs / gloo in CPU tests), end of run only:
    all_reduce(MAX) of the time, all_gather of per-source m_s and digest.
    """
    import torch
    import torch.distributed as dist

    src = np.asarray(sources_plan_order, dtype=np.uint32)
    n = len(src)
    ng = (n + group_bits - 1) // group_bits
    gids = shard_groups(ng, world, rank, costs, policy)
    rows = rows_of_groups(gids, n, group_bits)
    depths, m_local, dig_local, ms = runner(src[rows])
    m_full = np.zeros(n, dtype=np.uint64)
    d_full = np.zeros(n, dtype=np.uint64) if want_digest else None
    m_full[rows] = np.asarray(m_local, dtype=np.uint64)
    if want_digest:
        d_full[rows] = np.asarray(dig_local, dtype=np.uint64)
    max_ms = float(ms)
    if world > 1:
        dev = device if device is not None else torch.device("cpu")
        t = torch.tensor([float(ms)], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
        max_ms = float(t.item())
        # every rank owns disjoint rows; SUM of zero-padded vectors = all_gather + scatter
        mv = torch.from_numpy(m_full.view(np.int64).copy()).to(dev)
        dist.all_reduce(mv, op=dist.ReduceOp.SUM, group=group)
        m_full = mv.cpu().numpy().view(np.uint64)
        if want_digest:
            dv = torch.from_numpy(d_full.view(np.int64).copy()).to(dev)
            dist.all_reduce(dv, op=dist.ReduceOp.SUM, group=group)
            d_full = dv.cpu().numpy().view(np.uint64)
    return ShardResult(gids, rows, depths, float(ms), max_ms, m_full, d_full, int(m_full.sum()))
