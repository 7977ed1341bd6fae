"""Pins for the oracle GroupBy planner (§5.2).

The plan does not change any depth, so parity is pinned by invariants, by hand-built
examples worked from Rule 1 / Rule 2 by hand, and by the direction of the paper's
sharing claim (GroupBy raises SD over random grouping)."""
from __future__ import annotations

import numpy as np

import ibfs_gen
import oracle
from oracle import planner, stats


def _csr(nv, pairs):
    g = oracle.OracleGraph.from_edges(ibfs_gen.from_pairs(nv, pairs))
    return g.adjacency()


def test_two_hub_example_by_hand():
    # hub A = 0 with leaves 2..9 (deg 8); hub B = 1 with leaves 10..15 (deg 6);
    # 16 isolated; 17-18 a separate edge (no neighbour above q).
    pairs = [(0, x) for x in range(2, 10)] + [(1, x) for x in range(10, 16)] + [(17, 18)]
    off, adj = _csr(19, pairs)
    sources = np.array([2, 10, 3, 11, 4, 12, 5, 13, 6, 7, 16, 17], dtype=np.uint32)
    perm = planner.groupby(off, adj, sources, group_bits=4, q=5)
    # Rule 1 (deg 1 < p=4) and Rule 2 (shared neighbour with deg > q=5) hold for the
    # leaves; buckets are visited by hub degree (A first); full groups of W=4 first,
    # then A's leftovers, then the isolated source, then the random remainder.
    assert perm.tolist() == [0, 2, 4, 6, 1, 3, 5, 7, 8, 9, 10, 11]


def test_uniform_graph_fallback_any_degree():
    # cycle: every degree is 2 <= q, so the hub is the max-degree neighbour of any
    # degree, ties to the lower id ("share some common vertices").
    n = 8
    off, adj = _csr(n, [(i, (i + 1) % n) for i in range(n)])
    hub, _ = planner.hubs(off, adj, np.arange(n, dtype=np.uint32), q=128)
    exp = [min((i - 1) % n, (i + 1) % n) for i in range(n)]
    assert hub.tolist() == exp


def test_permutation_invariants_and_determinism():
    el = ibfs_gen.rmat(12, 16, ibfs_gen.KRONECKER, seed=1)
    g = oracle.OracleGraph.from_edges(el)
    off, adj = g.adjacency()
    src = ibfs_gen.sample_sources(el, 300, seed=2)
    for W in (32, 64, 128):
        p1 = planner.groupby(off, adj, src, W)
        p2 = planner.groupby(off, adj, src, W)
        assert sorted(p1.tolist()) == list(range(300))
        np.testing.assert_array_equal(p1, p2)
    r = planner.random_plan(300, 3)
    assert sorted(r.tolist()) == list(range(300))
    assert planner.shuffle([], 1) == [] and planner.shuffle([7], 1) == [7]


def test_groupby_raises_sharing_on_apsp_pool():
    el = ibfs_gen.rmat(12, 16, ibfs_gen.KRONECKER, seed=1)
    g = oracle.OracleGraph.from_edges(el)
    off, adj = g.adjacency()
    deg = np.diff(off)
    src = np.flatnonzero(deg > 0).astype(np.uint32)
    W = 64
    res = g.bfs(src)

    def mean_sd(perm):
        sds = []
        for k in range(len(perm) // W):
            rows = res.depths[perm[k * W:(k + 1) * W]]
            sds.append(stats.sharing_degree(rows))
        return float(np.mean(sds))

    sd_g = mean_sd(planner.groupby(off, adj, src, W))
    sd_r = mean_sd(planner.random_plan(len(src), 3))
    assert sd_g > 1.2 * sd_r


def test_groupby_hops2_invariants_and_anchor_order():
    """hops = 2: a permutation, deterministic, full 1-hop groups first, and the
    remaining hubbed sources contiguous per 2-hop anchor."""
    el = ibfs_gen.rmat(12, 16, ibfs_gen.KRONECKER, seed=5)
    og = oracle.OracleGraph.from_edges(el)
    off, adj = og.adjacency()
    src = ibfs_gen.sample_sources(el, 1024, 7)
    p1 = planner.groupby(off, adj, src, 32)
    p2 = planner.groupby(off, adj, src, 32, hops=2)
    assert sorted(p2.tolist()) == list(range(len(src)))
    np.testing.assert_array_equal(p2, planner.groupby(off, adj, src, 32, hops=2))
    hub, sdeg = planner.hubs(off, adj, src, 128)
    deg = np.diff(off.astype(np.int64))
    # the full groups of step 3 are identical in both modes
    full = 0
    while full + 32 <= len(p1) and len(set(hub[p1[full:full + 32]].tolist())) == 1 and hub[p1[full]] >= 0:
        full += 32
    np.testing.assert_array_equal(p1[:full], p2[:full])
    # anchors of the hubbed tail are non-increasing in degree (each anchor one run)
    h2, _ = planner.hubs(off, adj, np.where(hub >= 0, hub, 0), 128)
    tail = [r for r in p2[full:] if sdeg[r] > 0 and hub[r] >= 0]
    anchors = []
    for r in tail:
        a, b = hub[r], h2[r]
        anchors.append(b if b >= 0 and (deg[b] > deg[a] or (deg[b] == deg[a] and b < a)) else a)
    runs = [anchors[0]] + [y for x, y in zip(anchors, anchors[1:]) if y != x]
    assert len(runs) == len(set(runs))
    assert all(deg[x] >= deg[y] for x, y in zip(runs, runs[1:]))


def test_groupby_hops2_worked_example_by_hand():
    """hops = 2 worked by hand from P:L577 ("it is not required that the source vertex
    directly connects to a high-outdegree vertex, as long as within the first several
    levels"), q = 3, p = (4,), W = 2.

    Core hub H = 0 (deg 5: A, B, 20, 21, 22).  Hubs A = 1 (H, 10, 11, 12), B = 2 (H, 13, 23,
    24), C = 3 (14, 25, 26, 27), all deg 4.  m = 12 (A, 15) has deg 2 <= q.  16 isolated;
    17 - 18 a separate edge.
    sources (index: vertex): 0:10  1:13  2:11  3:15  4:16  5:17  6:14
      1-hop hubs: 10, 11 -> A; 13 -> B; 14 -> C; 15, 17 none (their neighbours have deg <= q)
      step 3 (p = 4): buckets A [0, 2], B [1], C [6] visited A, B, C (deg 4 each, id asc);
        A holds W = 2 -> group [0, 2]; leftovers [1] (B), [6] (C)
      degree-0 sources: [4]
      hubless 15: max-degree neighbour m(15) = 12, hub(12) = A -> hub 1, reached a level
        later; 17: m(17) = 18, hub(18) none -> stays in the random remainder
      2-hop anchors (larger of hub and hub(hub) by degree): 13 -> B -> hub(B) = H: anchor H;
        14 -> C, hub(C) none: anchor C; 15 -> A -> hub(A) = H: anchor H
      order: 1-hop hubbed first by anchor degree desc [1 (H), 6 (C)], then the m(r) ones [3]
    perm = [0, 2] + [4] + [1, 6, 3] + shuffle([5]) = [0, 2, 4, 1, 6, 3, 5]."""
    pairs = [(0, 1), (0, 2), (0, 20), (0, 21), (0, 22),
             (1, 10), (1, 11), (1, 12),
             (2, 13), (2, 23), (2, 24),
             (3, 14), (3, 25), (3, 26), (3, 27),
             (12, 15), (17, 18)]
    off, adj = _csr(28, pairs)
    deg = np.diff(off.astype(np.int64))
    assert deg[[0, 1, 2, 3, 12]].tolist() == [5, 4, 4, 4, 2]
    sources = np.array([10, 13, 11, 15, 16, 17, 14], dtype=np.uint32)
    perm = planner.groupby(off, adj, sources, group_bits=2, q=3, p_list=(4,), hops=2)
    assert perm.tolist() == [0, 2, 4, 1, 6, 3, 5]
    # hops = 1 (the literal steps): leftovers in bucket order, then degree-0, then the
    # random remainder {3, 5} (seeded order)
    p1 = planner.groupby(off, adj, sources, group_bits=2, q=3, p_list=(4,), hops=1)
    assert p1.tolist()[:5] == [0, 2, 1, 6, 4] and sorted(p1.tolist()[5:]) == [3, 5]
