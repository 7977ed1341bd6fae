"""Pins for the CPU oracle (task rule ③): values the paper prints, closed forms,
brute force (Floyd-Warshall, the APSP baseline the paper names), a third-party
library (scipy.sparse.csgraph), the complete invariant certificate,
and structural identities.  None of these re-types oracle.c's BFS loop."""
from __future__ import annotations

import numpy as np
import pytest

import ibfs_gen
import oracle
from oracle import certify, stats
from golden_io import read_fig1

M64 = (1 << 64) - 1


def floyd_warshall(nv, pairs, directed):
    """Brute-force all-pairs shortest paths with unit weights; INF -> -1."""
    INF = 10 ** 6
    D = np.full((nv, nv), INF, dtype=np.int64)
    np.fill_diagonal(D, 0)
    for u, v in pairs:
        if u != v:
            D[u, v] = min(D[u, v], 1)
            if not directed:
                D[v, u] = min(D[v, u], 1)
    for k in range(nv):
        D = np.minimum(D, D[:, k:k + 1] + D[k:k + 1, :])
    D[D >= INF] = -1
    return D


def random_multigraph(rng, nv, m):
    pairs = [(int(rng.integers(nv)), int(rng.integers(nv))) for _ in range(m)]
    if m and rng.random() < 0.5:  # force multi-edges and self-loops
        pairs.append(pairs[0])
        x = int(rng.integers(nv))
        pairs.append((x, x))
    return pairs


def run_oracle(nv, pairs, sources, directed=False):
    el = ibfs_gen.from_pairs(nv, pairs if pairs else np.zeros((0, 2)), directed)
    g = oracle.OracleGraph.from_edges(el)
    return g, g.bfs(np.asarray(sources, dtype=np.uint32))


@pytest.mark.parametrize("directed", [False, True])
def test_floyd_warshall_random_tiny(directed):
    rng = np.random.default_rng(12345 + directed)
    for trial in range(600):
        nv = int(rng.integers(1, 41))
        m = int(rng.integers(0, 2 * nv + 1))
        pairs = random_multigraph(rng, nv, m)
        fw = floyd_warshall(nv, pairs, directed)
        srcs = np.arange(nv, dtype=np.uint32)
        _, res = run_oracle(nv, pairs, srcs, directed)
        assert res.status == 0
        np.testing.assert_array_equal(res.depths.astype(np.int64), fw, err_msg=f"trial {trial}")


def test_closed_forms():
    n = 50
    # path: d(i, j) = |i - j|
    _, r = run_oracle(n, [(i, i + 1) for i in range(n - 1)], range(n))
    ii, jj = np.meshgrid(np.arange(n), np.arange(n), indexing="ij")
    np.testing.assert_array_equal(r.depths, np.abs(ii - jj))
    # cycle: min(|i-j|, n-|i-j|)
    _, r = run_oracle(n, [(i, (i + 1) % n) for i in range(n)], range(n))
    dd = np.abs(ii - jj)
    np.testing.assert_array_equal(r.depths, np.minimum(dd, n - dd))
    # star with centre 0: 0<->leaf 1, leaf<->leaf 2
    _, r = run_oracle(n, [(0, i) for i in range(1, n)], range(n))
    exp = np.where(ii == jj, 0, np.where((ii == 0) | (jj == 0), 1, 2))
    np.testing.assert_array_equal(r.depths, exp)
    # complete graph: 1 off the diagonal
    k = 12
    _, r = run_oracle(k, [(a, b) for a in range(k) for b in range(a + 1, k)], range(k))
    np.testing.assert_array_equal(r.depths, 1 - np.eye(k, dtype=np.int64))
    # 2-D grid a x b: Manhattan distance
    a, b = 7, 9
    idx = lambda x, y: x * b + y  # noqa: E731
    pairs = [(idx(x, y), idx(x + 1, y)) for x in range(a - 1) for y in range(b)]
    pairs += [(idx(x, y), idx(x, y + 1)) for x in range(a) for y in range(b - 1)]
    _, r = run_oracle(a * b, pairs, range(a * b))
    xy = np.array([(x, y) for x in range(a) for y in range(b)])
    man = np.abs(xy[:, None, 0] - xy[None, :, 0]) + np.abs(xy[:, None, 1] - xy[None, :, 1])
    np.testing.assert_array_equal(r.depths, man)
    # disjoint union of two paths: -1 across components
    pairs = [(i, i + 1) for i in range(9)] + [(10 + i, 11 + i) for i in range(9)]
    _, r = run_oracle(20, pairs, range(20))
    cross = (ii[:20, :20] < 10) != (jj[:20, :20] < 10)
    assert (r.depths[cross] == -1).all()
    # isolated source: row is -1 except 0 at the source
    _, r = run_oracle(5, [(0, 1), (1, 2)], [4])
    np.testing.assert_array_equal(r.depths[0], [-1, -1, -1, -1, 0])
    assert r.m_s[0] == 0 and r.reached[0] == 1 and r.ecc[0] == 0


def test_worked_example_fig1():
    fx = read_fig1()
    g, r = run_oracle(fx["nv"], fx["edges"], fx["sources"])
    np.testing.assert_array_equal(r.depths, fx["depths"])
    # textual constraints of the decoding
    off, adj = g.adjacency()
    nbrs = lambda x: sorted(adj[off[x]:off[x + 1]].tolist())  # noqa: E731
    assert nbrs(0) == [1, 4] and nbrs(7) == [5, 6, 8] and 3 in nbrs(6) and 4 in nbrs(1)


def test_worked_example_frontiers_fig4_fig13():
    fx = read_fig1()
    _, r = run_oracle(fx["nv"], fx["edges"], fx["sources"])
    d = r.depths
    # Fig. 4 JFQ3: vertices with some instance at depth 1 (discovered at our level 1)
    jfq = sorted(np.flatnonzero((d == 1).any(axis=0)).tolist())
    assert jfq == fx["jfq_after_level1"]
    # Fig. 13: BSA after our level 2 = visited bits (depth <= 2), BFS-0 leftmost
    words = ["".join("1" if 0 <= d[j, v] <= 2 else "0" for j in range(4)) for v in range(5, 9)]
    assert words == fx["bsa_v5_v8"]


def test_sharing_degree_fig1_and_lemma1():
    fx = read_fig1()
    _, r = run_oracle(fx["nv"], fx["edges"], fx["sources"])
    lc = stats.level_counts(r.depths, "TTTT")
    # frontier sizes per TD level: 4 sources, 6, 9, 9 and Lemma 1's
    # identity sum_k sum_j |FQ_j(k)| = N*|V| on a connected graph
    assert [x["jfq"] for x in lc] == [4, 6, 9, 9]
    assert sum(x["sum_fq"] for x in lc) == 4 * 9
    assert abs(stats.sharing_degree(r.depths) - 36 / 28) < 1e-12


def test_scipy_cross_check_rmat():
    sp = pytest.importorskip("scipy.sparse")
    csgraph = pytest.importorskip("scipy.sparse.csgraph")
    for scale, abc in ((10, ibfs_gen.RMAT), (12, ibfs_gen.KRONECKER)):
        el = ibfs_gen.rmat(scale, 16, abc, seed=7)
        srcs = ibfs_gen.sample_sources(el, 40, seed=9)
        g = oracle.OracleGraph.from_edges(el)
        r = g.bfs(srcs)
        A = sp.coo_matrix((np.ones(el.m), (el.u, el.v)), shape=(el.nv, el.nv)).tocsr()
        D = csgraph.shortest_path(A, directed=False, unweighted=True, indices=srcs.astype(np.int64))
        D = np.where(np.isinf(D), -1, D).astype(np.int64)
        np.testing.assert_array_equal(r.depths.astype(np.int64), D)


def test_certificate_accepts_oracle_and_rejects_perturbations():
    el = ibfs_gen.rmat(10, 8, ibfs_gen.KRONECKER, seed=3)
    g = oracle.OracleGraph.from_edges(el)
    off, adj = g.adjacency()
    srcs = ibfs_gen.sample_sources(el, 8, seed=4)
    r = g.bfs(srcs)
    assert certify.certify_rows(off, adj, srcs, r.depths) == []
    rng = np.random.default_rng(0)
    rejected = 0
    for t in range(200):
        row = r.depths[t % 8].astype(np.int16).copy()
        v = int(rng.integers(el.nv))
        kind = t % 4
        if kind == 0 and row[v] >= 0:
            row[v] += 1
        elif kind == 1 and row[v] > 0:
            row[v] -= 1
        elif kind == 2:
            row[v] = -1 if row[v] >= 0 else 5
        else:
            row[v] = -2
        if (row == r.depths[t % 8]).all():
            continue
        assert certify.certify_row(off, adj, int(srcs[t % 8]), row) is not None
        rejected += 1
    assert rejected > 100


def test_c_certificate_matches_python_certificate():
    # OracleGraph.certify (C loops, used on config-5 rows) vs certify.py on the same rows:
    # both accept the oracle's rows and reject the same perturbations
    rng = np.random.default_rng(11)
    for trial in range(40):
        nv = int(rng.integers(2, 50))
        m = int(rng.integers(0, 3 * nv + 1))
        pairs = [(int(rng.integers(nv)), int(rng.integers(nv))) for _ in range(m)]
        el = ibfs_gen.from_pairs(nv, pairs if pairs else np.zeros((0, 2)))
        g = oracle.OracleGraph.from_edges(el)
        off, adj = g.adjacency()
        srcs = rng.integers(0, nv, size=4).astype(np.uint32)
        r = g.bfs(srcs)
        for j, s in enumerate(srcs):
            assert g.certify(int(s), r.depths[j]) is None
            for _ in range(10):
                row = r.depths[j].copy()
                v = int(rng.integers(nv))
                row[v] = np.int8(int(rng.choice([-2, -1, 0, 1, 2, 3, 7])))
                py = certify.certify_row(off, adj, int(s), row)
                c = g.certify(int(s), row)
                assert (py is None) == (c is None), (trial, py, c)
    # a closed form it must accept: path 0-1-...-9 from 0
    el = ibfs_gen.from_pairs(10, [(i, i + 1) for i in range(9)])
    g = oracle.OracleGraph.from_edges(el)
    assert g.certify(0, np.arange(10, dtype=np.int8)) is None
    assert g.certify(0, np.r_[np.arange(9), 7].astype(np.int8)) is not None


def test_apsp_symmetry_and_mass():
    el = ibfs_gen.rmat(9, 8, ibfs_gen.KRONECKER, seed=5)
    g = oracle.OracleGraph.from_edges(el)
    r = g.bfs(np.arange(el.nv, dtype=np.uint32))
    np.testing.assert_array_equal(r.depths, r.depths.T)
    # m_s: degrees counted independently from the raw tuples (each tuple adds one entry
    # to each endpoint; a self-loop adds two to its vertex), P:L887 / P:L977
    deg = np.bincount(el.u, minlength=el.nv) + np.bincount(el.v, minlength=el.nv)
    np.testing.assert_array_equal(r.m_s, stats.m_s_from_depths(r.depths, deg))
    np.testing.assert_array_equal(r.reached, (r.depths >= 0).sum(axis=1))
    np.testing.assert_array_equal(r.ecc, r.depths.max(axis=1))


def _splitmix(z):
    z = (z + 0x9E3779B97F4A7C15) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def test_digest_definition():
    fx = read_fig1()
    _, r = run_oracle(fx["nv"], fx["edges"], fx["sources"])
    for row, dg in zip(r.depths, r.digest):
        exp = sum(_splitmix((v << 8) | (int(d) + 1)) for v, d in enumerate(row) if d >= 0) & M64
        assert int(dg) == exp


def test_range_error_on_deep_path():
    n = 200
    _, r = run_oracle(n, [(i, i + 1) for i in range(n - 1)], [0])
    assert r.status == oracle.ORACLE_E_RANGE


def test_thread_count_invariance():
    el = ibfs_gen.rmat(11, 16, ibfs_gen.RMAT, seed=1)
    srcs = ibfs_gen.sample_sources(el, 33, seed=2)
    g = oracle.OracleGraph.from_edges(el)
    a = g.bfs(srcs, threads=1)
    b = g.bfs(srcs, threads=7)
    np.testing.assert_array_equal(a.depths, b.depths)
    np.testing.assert_array_equal(a.digest, b.digest)


# ---- k-hop reachability index (§8.7: "the first k levels BFS") ----------

@pytest.mark.parametrize("directed", [False, True])
def test_khop_floyd_warshall_random_tiny(directed):
    """depth capped at k == the brute-force distance where it is <= k, else -1; m_s and
    reached count exactly the vertices within k hops (degrees from the raw tuples)."""
    rng = np.random.default_rng(777 + directed)
    for trial in range(300):
        nv = int(rng.integers(1, 31))
        m = int(rng.integers(0, 2 * nv + 1))
        pairs = random_multigraph(rng, nv, m)
        fw = floyd_warshall(nv, pairs, directed)
        deg = np.zeros(nv, dtype=np.int64)
        for u, v in pairs:
            deg[u] += 1
            if not directed:
                deg[v] += 1
        k = int(rng.integers(0, 5))
        el = ibfs_gen.from_pairs(nv, pairs if pairs else np.zeros((0, 2)), directed)
        res = oracle.OracleGraph.from_edges(el).bfs(np.arange(nv, dtype=np.uint32), max_depth=k)
        exp = np.where((fw >= 0) & (fw <= k), fw, -1)
        np.testing.assert_array_equal(res.depths.astype(np.int64), exp, err_msg=f"trial {trial} k={k}")
        within = exp >= 0
        np.testing.assert_array_equal(res.reached.astype(np.int64), within.sum(axis=1))
        np.testing.assert_array_equal(res.m_s.astype(np.int64), (within * deg[None, :]).sum(axis=1))


def test_khop_closed_forms():
    """Path graph: d = |i - j| where <= k; k = 0 keeps only the source; k >= the diameter
    is the plain BFS."""
    n = 40
    pairs = [(i, i + 1) for i in range(n - 1)]
    el = ibfs_gen.from_pairs(n, pairs, False)
    g = oracle.OracleGraph.from_edges(el)
    ii, jj = np.meshgrid(np.arange(n), np.arange(n), indexing="ij")
    dd = np.abs(ii - jj)
    for k in (0, 1, 3, 7):
        r = g.bfs(np.arange(n, dtype=np.uint32), max_depth=k)
        np.testing.assert_array_equal(r.depths, np.where(dd <= k, dd, -1))
        assert (r.ecc == np.minimum(k, np.maximum(np.arange(n), n - 1 - np.arange(n)))).all()
    full = g.bfs(np.arange(n, dtype=np.uint32))
    capped = g.bfs(np.arange(n, dtype=np.uint32), max_depth=n - 1)
    np.testing.assert_array_equal(full.depths, capped.depths)
    np.testing.assert_array_equal(full.digest, capped.digest)
    with pytest.raises(ValueError):
        g.bfs(np.arange(2, dtype=np.uint32), max_depth=-1)
