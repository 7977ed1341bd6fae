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


def tuple_degrees(el) -> np.ndarray:
    """CSR row lengths straight from the tuple list (no device export): an undirected tuple
    (u, v) adds one entry to row u and one to row v; directed, row u only."""
    deg = np.bincount(np.asarray(el.u), minlength=el.nv).astype(np.int64)
    if not getattr(el, "directed", False):
        deg += np.bincount(np.asarray(el.v), minlength=el.nv)
    return deg


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
class GroupSchedule:
    """This rank's share of a plan and the order it runs it in -- the one schedule both
    ``bench.py`` and the full-size parity tests use.

    The plan-ordered source list is cut into W-wide groups; ``shard_groups`` gives this rank
    its groups; step k runs ``groups_per_step`` of them, cycling through the share:
    step k = share[(k*G + i) % len(share)], i < G.  A step is one ``Graph.run`` call (one
    or more launch batches of the library)."""
    n: int                    # sources in the whole plan
    group_bits: int
    world: int
    rank: int
    groups_per_step: int
    share: np.ndarray         # this rank's group ids (ascending)

    @classmethod
    def make(cls, n: int, group_bits: int, world: int = 1, rank: int = 0, costs=None,
             policy: str = "lpt", groups_per_step: int = 0) -> "GroupSchedule":
        ng = (n + group_bits - 1) // group_bits
        share = shard_groups(ng, world, rank, costs, policy)
        if len(share) == 0:  # more ranks than groups: this rank repeats one group (weak scaling)
            share = np.array([rank % max(ng, 1)], dtype=np.int64)
        G = int(groups_per_step) or len(share)
        return cls(int(n), int(group_bits), int(world), int(rank), G, share)

    @property
    def n_groups(self) -> int:
        return (self.n + self.group_bits - 1) // self.group_bits

    @property
    def steps_per_cycle(self) -> int:
        """Steps that together run every group of the share at least once."""
        return (len(self.share) + self.groups_per_step - 1) // self.groups_per_step

    def step_groups(self, k: int) -> np.ndarray:
        G, m = self.groups_per_step, len(self.share)
        return np.asarray([self.share[(k * G + i) % m] for i in range(G)], dtype=np.int64)

    def step_rows(self, k: int) -> np.ndarray:
        """Indices into the plan-ordered source list of step k, in run order (steps repeat
        with period len(share)/gcd: memoised)."""
        key = (k * self.groups_per_step) % len(self.share)
        cache = self.__dict__.setdefault("_rows", {})
        if key not in cache:
            cache[key] = rows_of_groups(self.step_groups(k), self.n, self.group_bits)
        return cache[key]


def gather_results(n: int, rows: np.ndarray, m_local, dig_local, ms: float, world: int = 1,
                   group=None, device=None):
    """End-of-run collectives (the only ones on the path): MAX of the device time,
    and every source's m_s / digest by SUM of zero-padded vectors (ranks own disjoint rows,
    so the SUM is an all-gather).  Returns (max_ms, m_full, d_full or None)."""
    import torch
    import torch.distributed as dist

    rows = np.asarray(rows, dtype=np.int64)
    m_full = np.zeros(n, dtype=np.uint64)
    m_full[rows] = np.asarray(m_local, dtype=np.uint64)
    d_full = None
    if dig_local is not None:
        d_full = np.zeros(n, dtype=np.uint64)
        d_full[rows] = np.asarray(dig_local, dtype=np.uint64)
    max_ms = float(ms)
    if world > 1:
        dev = device if device is not None else torch.device("cpu")
        t = torch.tensor([float(ms)], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
        max_ms = float(t.item())
        mv = torch.from_numpy(m_full.view(np.int64).copy()).to(dev)
        dist.all_reduce(mv, op=dist.ReduceOp.SUM, group=group)
        m_full = mv.cpu().numpy().view(np.uint64)
        if d_full is not None:
            dv = torch.from_numpy(d_full.view(np.int64).copy()).to(dev)
            dist.all_reduce(dv, op=dist.ReduceOp.SUM, group=group)
            d_full = dv.cpu().numpy().view(np.uint64)
    return max_ms, m_full, d_full


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
                device=None, groups_per_step: int = 0) -> ShardResult:
    """Run this rank's groups, ``groups_per_step`` per ``runner`` call (0 = all in one call),
    with ``runner(rank_sources) -> (depths, m_s, digest, ms)`` (normally ``Graph.run``
    unpacked), then gather (``gather_results``).  Depths are returned only for a one-call
    run (they stay on the rank; a multi-call run keeps only the statistics)."""
    src = np.asarray(sources_plan_order, dtype=np.uint32)
    n = len(src)
    sched = GroupSchedule.make(n, group_bits, world, rank, costs, policy, groups_per_step)
    if n == 0 or sched.n_groups == 0:
        return ShardResult(np.zeros(0, np.int64), np.zeros(0, np.int64), None, 0.0, 0.0,
                           np.zeros(0, np.uint64), np.zeros(0, np.uint64) if want_digest else None, 0)
    gids = sched.share
    rows_all, m_parts, d_parts, total_ms, depths = [], [], [], 0.0, None
    for k in range(sched.steps_per_cycle):
        rows = sched.step_rows(k)
        if k == sched.steps_per_cycle - 1:  # the last step may wrap around: keep new groups only
            seen = np.concatenate(rows_all) if rows_all else np.zeros(0, np.int64)
            keep = ~np.isin(rows, seen)
        else:
            keep = np.ones(len(rows), dtype=bool)
        d, m_local, dig_local, ms = runner(src[rows])
        total_ms += float(ms)
        rows_all.append(rows[keep])
        m_parts.append(np.asarray(m_local, dtype=np.uint64)[keep])
        if want_digest:
            d_parts.append(np.asarray(dig_local, dtype=np.uint64)[keep])
        if sched.steps_per_cycle == 1:
            depths = d
    rows = np.concatenate(rows_all)
    max_ms, m_full, d_full = gather_results(n, rows, np.concatenate(m_parts),
                                            np.concatenate(d_parts) if want_digest else None,
                                            total_ms, world, group, device)
    return ShardResult(gids, rows, depths, float(total_ms), max_ms, m_full, d_full, int(m_full.sum()))
