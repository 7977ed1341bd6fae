"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by
element on the same seeded inputs.  Depths are integer results: bit-exact everywhere.
Full BASELINE sizes are checked on sampled rows the oracle computes one by one, plus
the complete invariant certificate and m_s / digest identities."""
from __future__ import annotations

import numpy as np
import pytest

import ibfs_gen
import oracle
from oracle import certify, planner, stats
from golden_io import read_fig1

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_sigmod_liuhh16_b200 as P  # noqa: E402
from paper_conf_sigmod_liuhh16_b200 import _lib  # noqa: E402

SCHEDULES = ["auto", "td", "bu1", "bu2", "alt", "rand"]


def run_kwargs(kind, rng=None):
    if kind == "auto":
        return {}
    if kind == "td":
        return {"direction": "td"}
    if kind == "bu1":
        return {"direction": "bu_from", "bu_from": 1}
    if kind == "bu2":
        return {"direction": "bu_from", "bu_from": 2}
    if kind == "alt":
        return {"schedule": "TB" * 70}
    if kind == "rand":
        r = rng or np.random.default_rng(0)
        return {"schedule": "".join(r.choice(["T", "B"], size=130))}
    raise ValueError(kind)


def gpu_depths(g, src, W, **kw):
    d, st = g.run(src, W, **kw)
    torch.cuda.synchronize()
    return d.cpu().numpy(), st


# --------------------------------------------------------------------- worked example
@pytest.mark.parametrize("W", [32, 64, 128])
@pytest.mark.parametrize("kind", SCHEDULES)
def test_fig1_all_schedules(W, kind):
    fx = read_fig1()
    el = ibfs_gen.from_pairs(fx["nv"], fx["edges"])
    g = P.Graph.from_edgelist(el)
    d, st = gpu_depths(g, fx["sources"], W, want_digest=True, **run_kwargs(kind))
    np.testing.assert_array_equal(d, fx["depths"])
    ref = oracle.bfs(el, fx["sources"])
    np.testing.assert_array_equal(st.per_source_m, ref.m_s)
    np.testing.assert_array_equal(st.per_source_digest, ref.digest)


@pytest.mark.parametrize("W", [32, 128])
@pytest.mark.parametrize("kind", ["bu1", "bu2", "alt", "rand"])
@pytest.mark.parametrize("mod", [1, 2, 3])
def test_fig1_split_levels(W, kind, mod):
    # per-instance split of BU levels (IBFS_SPLIT_FORCE): instances j % mod == 0 run
    # top-down inside every BU level; results never change
    fx = read_fig1()
    el = ibfs_gen.from_pairs(fx["nv"], fx["edges"])
    g = P.Graph.from_edgelist(el)
    d, st = gpu_depths(g, fx["sources"], W, split="force", split_mod=mod, **run_kwargs(kind))
    np.testing.assert_array_equal(d, fx["depths"])
    ref = oracle.bfs(el, fx["sources"])
    np.testing.assert_array_equal(st.per_source_m, ref.m_s)


def test_fig1_trace_frontiers():
    # SURVEY App. A trace (TD, TD, BU, ...): JFQ sizes 4, 6, then all 9 vertices in BU.
    fx = read_fig1()
    g = P.Graph.from_edgelist(ibfs_gen.from_pairs(fx["nv"], fx["edges"]))
    _, st = gpu_depths(g, fx["sources"], 32, schedule="TTBT")
    lv = st.per_level
    assert [x["jfq_td"] for x in lv[:2]] == [4, 6]
    assert lv[2]["bu_groups"] == 1 and lv[2]["jfq_bu"] == 9
    # Lemma 1 style identity on the TD-only run: sum_k sum_j |FQ_j(k)| = N * |V|
    _, st = gpu_depths(g, fx["sources"], 32, direction="td")
    assert st.sd_fq_td == 4 * 9 and st.sd_jfq_td == 28


# ---------------------------------------------------------------- random tiny graphs
def test_random_tiny_multigraphs_forced_schedules():
    rng = np.random.default_rng(2024)
    for trial in range(120):
        nv = int(rng.integers(1, 60))
        m = int(rng.integers(0, 3 * nv + 1))
        pairs = [(int(rng.integers(nv)), int(rng.integers(nv))) for _ in range(m)]
        if m:
            pairs += [pairs[0], (pairs[-1][0], pairs[-1][0])]
        el = ibfs_gen.from_pairs(nv, pairs if pairs else np.zeros((0, 2)))
        n = int(rng.integers(1, 3 * 64))
        src = rng.integers(0, nv, size=n).astype(np.uint32)  # duplicates allowed
        W = int(rng.choice([32, 64, 128]))
        kind = SCHEDULES[trial % len(SCHEDULES)]
        split = ["auto", "off", "force"][trial % 3]
        mod = int(rng.integers(1, 6))
        g = P.Graph.from_edgelist(el)
        d, st = gpu_depths(g, src, W, groups_in_flight=int(rng.integers(0, 4)), split=split, split_mod=mod,
                           **run_kwargs(kind, rng))
        ref = oracle.bfs(el, src)
        np.testing.assert_array_equal(d, ref.depths, err_msg=f"trial {trial} W={W} {kind} split={split}/{mod}")
        np.testing.assert_array_equal(st.per_source_m, ref.m_s)


# ------------------------------------------------------------------------- configs
def _check_full(el, src, W, **kw):
    g = P.Graph.from_edgelist(el)
    d, st = gpu_depths(g, src, W, want_digest=True, **kw)
    ref = oracle.bfs(el, src)
    np.testing.assert_array_equal(d, ref.depths)
    np.testing.assert_array_equal(st.per_source_m, ref.m_s)
    np.testing.assert_array_equal(st.per_source_digest, ref.digest)
    assert st.edges_traversed == int(ref.m_s.sum())
    return g, d, st, ref


@pytest.mark.parametrize("kind", ["auto", "td", "bu2"])
@pytest.mark.parametrize("split", ["auto", "off", "force"])
def test_config1_full(kind, split):
    cfg = ibfs_gen.CONFIGS["c1"]
    el = cfg.edges()
    src = cfg.sources(el)
    g = P.Graph.from_edgelist(el)
    perm = g.plan(src, cfg.group_bits)
    _check_full(el, src[perm], cfg.group_bits, split=split, split_mod=3, **run_kwargs(kind))


@pytest.mark.parametrize("W", [32, 64, 128])
@pytest.mark.parametrize("mode", ["groupby", "random", "identity"])
def test_config2_full(W, mode):
    cfg = ibfs_gen.CONFIGS["c2"]
    el = cfg.edges()
    src = cfg.sources(el)
    g = P.Graph.from_edgelist(el)
    perm = g.plan(src, W, mode=mode)
    s = src[perm]
    d, st = gpu_depths(g, s, W, want_digest=True)
    ref = _oracle_c2(el, s)
    np.testing.assert_array_equal(d, ref.depths)
    np.testing.assert_array_equal(st.per_source_digest, ref.digest)
    np.testing.assert_array_equal(st.per_source_m, ref.m_s)


_C2 = {}


def _oracle_c2(el, s):
    key = s.tobytes()
    if key not in _C2:
        _C2[key] = oracle.bfs(el, s)
    return _C2[key]


def test_config2_td_only_sd_counters_match_oracle():
    cfg = ibfs_gen.CONFIGS["c2"]
    el = cfg.edges()
    src = cfg.sources(el)
    g = P.Graph.from_edgelist(el)
    d, st = gpu_depths(g, src, 128, direction="td")
    ref = _oracle_c2(el, src)
    np.testing.assert_array_equal(d, ref.depths)
    lc = stats.level_counts(ref.depths, "T" * 200)
    assert st.sd_fq_td == sum(x["sum_fq"] for x in lc)
    assert st.sd_jfq_td == sum(x["jfq"] for x in lc)
    assert [x["new_pairs"] for x in st.per_level] == [x["new_pairs"] for x in lc]


@pytest.mark.parametrize("split", ["auto", "off", "force"])
def test_config2_auto_level_counters_match_oracle(split):
    # a split BU level counts as bottom-up in Eq. 1 (reading #23 over all active instances)
    cfg = ibfs_gen.CONFIGS["c2"]
    el = cfg.edges()
    src = cfg.sources(el)
    g = P.Graph.from_edgelist(el)
    d, st = gpu_depths(g, src, 128, split=split, split_mod=2)
    ref = _oracle_c2(el, src)
    np.testing.assert_array_equal(d, ref.depths)
    sched = "".join("T" if x["td_groups"] else "B" for x in st.per_level)
    lc = stats.level_counts(ref.depths, sched)
    for x, y in zip(st.per_level, lc):
        if y["dir"] == "T":
            assert (x["jfq_td"], x["fq_td"]) == (y["jfq"], y["sum_fq"])
        else:
            assert (x["jfq_bu"], x["fq_bu"]) == (y["jfq"], y["sum_fq"])


def test_config4_apsp_subset_and_symmetry():
    cfg = ibfs_gen.CONFIGS["c4"]
    el = cfg.edges()
    g = P.Graph.from_edgelist(el)
    allsrc = cfg.sources(el)
    perm = g.plan(allsrc, 128)
    # 64 groups of the real plan (8,192 sources), run as the bench does (many groups per launch)
    s = allsrc[perm][: 64 * 128]
    d, st = gpu_depths(g, s, 128, want_digest=True)
    ref = oracle.bfs(el, s)
    np.testing.assert_array_equal(d, ref.depths)
    np.testing.assert_array_equal(st.per_source_digest, ref.digest)
    # symmetry d(s,t) = d(t,s) on the sampled block
    pos = {int(v): i for i, v in enumerate(s)}
    idx = np.array([pos[int(v)] for v in s[:500]])
    block = d[idx][:, s[:500]]
    np.testing.assert_array_equal(block, block.T)


@pytest.mark.parametrize("name,rows", [("c3", 12), ("c5", 6)])
def test_full_size_sampled_rows(name, rows):
    cfg = ibfs_gen.CONFIGS[name]
    el = cfg.edges()
    src = cfg.sources(el)
    g = P.Graph.from_edgelist(el)
    perm = g.plan(src, 128)
    s = src[perm][:128]  # one full group, W = 128 as the bench runs it
    d, st = gpu_depths(g, s, 128, want_digest=True)
    pick = np.random.default_rng(5).choice(128, size=rows, replace=False)
    og = oracle.OracleGraph.from_edges(el)
    ref = og.bfs(s[pick])
    np.testing.assert_array_equal(d[pick], ref.depths)
    np.testing.assert_array_equal(st.per_source_digest[pick], ref.digest)
    np.testing.assert_array_equal(st.per_source_m[pick], ref.m_s)
    off, adj = og.adjacency()
    for r in range(0, 128, 32):  # certificate on rows the oracle did not compute
        assert certify.certify_row(off, adj, int(s[r]), d[r]) is None


# ----------------------------------------------------------------------- planner
@pytest.mark.parametrize("W", [32, 64, 128])
def test_planner_matches_oracle_planner(W):
    for cfg in (ibfs_gen.CONFIGS["c1"], ibfs_gen.CONFIGS["c2"], ibfs_gen.CONFIGS["d2"]):
        el = cfg.edges()
        src = cfg.sources(el)
        g = P.Graph.from_edgelist(el)
        og = oracle.OracleGraph.from_edges(el)
        off, adj = og.adjacency()
        np.testing.assert_array_equal(g.plan(src, W), planner.groupby(off, adj, src, W))
        np.testing.assert_array_equal(g.plan(src, W, hops=2), planner.groupby(off, adj, src, W, hops=2))
        np.testing.assert_array_equal(g.plan(src, W, mode="random", seed=9), planner.random_plan(len(src), 9))
        np.testing.assert_array_equal(g.plan(src, W, mode="identity"), np.arange(len(src)))
    el = ibfs_gen.rmat(12, 16, ibfs_gen.KRONECKER, seed=1)
    allv = ibfs_gen.all_vertices(el.nv)
    g = P.Graph.from_edgelist(el)
    off, adj = oracle.OracleGraph.from_edges(el).adjacency()
    np.testing.assert_array_equal(g.plan(allv, W), planner.groupby(off, adj, allv, W))
    np.testing.assert_array_equal(g.plan(allv, W, hops=2), planner.groupby(off, adj, allv, W, hops=2))


def test_csr_build_matches_oracle_adjacency():
    el = ibfs_gen.rmat(12, 8, ibfs_gen.RMAT, seed=4)
    g = P.Graph.from_edgelist(el, hub_first=False)
    off, adj = g.export_csr()
    ooff, oadj = oracle.OracleGraph.from_edges(el).adjacency()
    np.testing.assert_array_equal(off, ooff)
    np.testing.assert_array_equal(adj, oadj)  # tuple order kept within every row
    g2 = P.Graph.from_csr(off, adj)
    assert (g2.nv, g2.ne, g2.max_degree) == (g.nv, g.ne, g.max_degree)
    # hub-first rows: same multiset per row, neighbour degree non-increasing, stable
    g2.sort_rows(True)
    off2, adj2 = g2.export_csr()
    np.testing.assert_array_equal(off2, off)
    deg = np.diff(off.astype(np.int64))
    for v in range(0, el.nv, 7):
        r0, r1 = int(off[v]), int(off[v + 1])
        row, srow = adj[r0:r1], adj2[r0:r1]
        assert sorted(row.tolist()) == sorted(srow.tolist())
        exp = sorted(range(r1 - r0), key=lambda i: (-deg[row[i]], i))
        np.testing.assert_array_equal(srow, row[exp])
    s = np.arange(0, el.nv, 37, dtype=np.uint32)
    d1, _ = g.run(s, 64)
    d2, _ = g2.run(s, 64)
    np.testing.assert_array_equal(d1.cpu().numpy(), d2.cpu().numpy())


# --------------------------------------------------------------------- edge cases
def test_edge_cases():
    el = ibfs_gen.rmat(10, 4, ibfs_gen.KRONECKER, seed=8)
    g = P.Graph.from_edgelist(el)
    deg = np.bincount(el.u, minlength=el.nv) + np.bincount(el.v, minlength=el.nv)
    iso = np.flatnonzero(deg == 0).astype(np.uint32)
    assert iso.size > 0
    # n = 0
    d, st = g.run(np.zeros(0, dtype=np.uint32), 64)
    assert d.shape == (0, el.nv) and st.edges_traversed == 0
    # n = 1 (single-source BFS), isolated sources, duplicates, ragged last group
    for s in (np.array([5], dtype=np.uint32), iso[:3], np.array([7] * 70, dtype=np.uint32),
              np.arange(200, dtype=np.uint32)):
        for W in (32, 128):
            dd, _ = gpu_depths(g, s, W)
            np.testing.assert_array_equal(dd, oracle.bfs(el, s).depths)
    # device-resident sources, host output, no output
    s = np.arange(0, 300, 3, dtype=np.uint32)
    ref = oracle.bfs(el, s)
    dd, _ = g.run(torch.from_numpy(s.astype(np.int32)).cuda(), 64, out="host")
    np.testing.assert_array_equal(dd, ref.depths)
    none, st = g.run(s, 64, out=None, want_digest=True)
    assert none is None
    np.testing.assert_array_equal(st.per_source_digest, ref.digest)
    # invalid source id / group_bits
    with pytest.raises(_lib.IbfsError) as e:
        g.run(np.array([el.nv], dtype=np.uint32), 64)
    assert e.value.code == _lib.IBFS_E_INVALID
    with pytest.raises(_lib.IbfsError):
        g.run(s, 48)


def test_depth_above_127_is_range_error():
    n = 200
    el = ibfs_gen.from_pairs(n, [(i, i + 1) for i in range(n - 1)])
    g = P.Graph.from_edgelist(el)
    with pytest.raises(_lib.IbfsError) as e:
        g.run(np.array([0], dtype=np.uint32), 32)
    assert e.value.code == _lib.IBFS_E_RANGE
    # the failed call left its ring slots dirty (never marked zero): the next call on the
    # same graph clears them first (clean ring) and is exact
    s = np.array([100, 90, 110], dtype=np.uint32)  # max depths 100, 109, 110
    d, _ = gpu_depths(g, s, 32)
    np.testing.assert_array_equal(d, oracle.bfs(el, s).depths)
    # a 128-vertex path has max depth 127: fits
    el = ibfs_gen.from_pairs(128, [(i, i + 1) for i in range(127)])
    g = P.Graph.from_edgelist(el)
    d, _ = gpu_depths(g, np.array([0, 127], dtype=np.uint32), 32)
    np.testing.assert_array_equal(d, oracle.bfs(el, np.array([0, 127], dtype=np.uint32)).depths)


def test_torch_allocator_hook():
    el = ibfs_gen.rmat(10, 8, ibfs_gen.RMAT, seed=2)
    g = P.Graph.from_edgelist(el)
    s = np.arange(100, dtype=np.uint32)
    P.use_torch_allocator(True)
    try:
        d, _ = gpu_depths(g, s, 64)
    finally:
        P.use_torch_allocator(False)
    np.testing.assert_array_equal(d, oracle.bfs(el, s).depths)


# ------------------------------------------------- k-hop reachability index (NEXT #2)
# §8.7: "computes the first k levels BFS for a large amount of selected
# vertices"; Table 1 builds the 3-hop index.  Oracle: the same textbook BFS capped at k.
@pytest.mark.parametrize("k", [1, 2, 3, 5])
@pytest.mark.parametrize("kind", ["auto", "td", "bu1", "rand"])
def test_khop_fig1_and_tiny(k, kind):
    rng = np.random.default_rng(100 + k)
    for trial in range(20):
        nv = int(rng.integers(1, 50))
        m = int(rng.integers(0, 3 * nv + 1))
        pairs = [(int(rng.integers(nv)), int(rng.integers(nv))) for _ in range(m)]
        el = ibfs_gen.from_pairs(nv, pairs if pairs else np.zeros((0, 2)))
        n = int(rng.integers(1, 150))
        src = rng.integers(0, nv, size=n).astype(np.uint32)
        W = int(rng.choice([32, 64, 128]))
        g = P.Graph.from_edgelist(el)
        d, st = gpu_depths(g, src, W, max_depth=k, want_digest=True, **run_kwargs(kind, rng))
        ref = oracle.bfs(el, src, max_depth=k)
        np.testing.assert_array_equal(d, ref.depths, err_msg=f"trial {trial} k={k} {kind} W={W}")
        np.testing.assert_array_equal(st.per_source_m, ref.m_s)
        np.testing.assert_array_equal(st.per_source_digest, ref.digest)
        assert st.max_levels <= k


@pytest.mark.parametrize("k", [1, 2, 3])
def test_khop_config2_full(k):
    cfg = ibfs_gen.CONFIGS["c2"]
    el = cfg.edges()
    src = cfg.sources(el)
    g = P.Graph.from_edgelist(el)
    s = src[g.plan(src, 128)]
    d, st = gpu_depths(g, s, 128, max_depth=k, want_digest=True)
    ref = oracle.bfs(el, s, max_depth=k)
    np.testing.assert_array_equal(d, ref.depths)
    np.testing.assert_array_equal(st.per_source_m, ref.m_s)
    np.testing.assert_array_equal(st.per_source_digest, ref.digest)
    full = _oracle_c2(el, s)
    np.testing.assert_array_equal(d, np.where(full.depths <= k, full.depths, -1))


def test_khop_invalid():
    g = P.Graph.from_edgelist(ibfs_gen.from_pairs(4, [(0, 1)]))
    with pytest.raises(ValueError):
        g.run(np.array([0], dtype=np.uint32), 32, max_depth=0)


# ------------------------------------------------------------ directed graphs (NEXT #1)
# "for directed graphs, we also store the reverse edges" -- top-down expands the
# out-edge rows, bottom-up reads a vertex's parents from the in-edge rows.  The oracle
# runs its textbook BFS over out-edges (oracle.c, pinned by directed Floyd-Warshall).
def _transpose_csr(nv, off, adj):
    src = np.repeat(np.arange(nv, dtype=np.uint32), np.diff(off).astype(np.int64))
    order = np.argsort(adj, kind="stable")
    roff = np.zeros(nv + 1, dtype=np.uint64)
    np.cumsum(np.bincount(adj, minlength=nv), out=roff[1:])
    return roff, src[order]


def test_directed_random_tiny_forced_schedules():
    rng = np.random.default_rng(4242)
    for trial in range(120):
        nv = int(rng.integers(1, 60))
        m = int(rng.integers(0, 4 * nv + 1))
        pairs = [(int(rng.integers(nv)), int(rng.integers(nv))) for _ in range(m)]
        if m:
            pairs += [pairs[0], (pairs[-1][0], pairs[-1][0])]
        el = ibfs_gen.from_pairs(nv, pairs if pairs else np.zeros((0, 2)), directed=True)
        n = int(rng.integers(1, 3 * 64))
        src = rng.integers(0, nv, size=n).astype(np.uint32)
        W = int(rng.choice([32, 64, 128]))
        kind = SCHEDULES[trial % len(SCHEDULES)]
        split = ["auto", "off", "force"][trial % 3]
        g = P.Graph.from_edgelist(el, hub_first=bool(trial % 2))
        d, st = gpu_depths(g, src, W, split=split, split_mod=int(rng.integers(1, 6)), want_digest=True,
                           **run_kwargs(kind, rng))
        ref = oracle.bfs(el, src)
        np.testing.assert_array_equal(d, ref.depths, err_msg=f"trial {trial} W={W} {kind} split={split}")
        np.testing.assert_array_equal(st.per_source_m, ref.m_s)
        np.testing.assert_array_equal(st.per_source_digest, ref.digest)


@pytest.mark.parametrize("W", [32, 64, 128])
@pytest.mark.parametrize("kind", ["auto", "td", "bu2"])
def test_directed_config_full(W, kind):
    cfg = ibfs_gen.CONFIGS["d2"]
    el = cfg.edges()
    assert el.directed
    src = cfg.sources(el)
    g = P.Graph.from_edgelist(el)
    s = src[g.plan(src, W)]
    d, st = gpu_depths(g, s, W, want_digest=True, **run_kwargs(kind))
    key = ("d2", s.tobytes())
    if key not in _C2:
        _C2[key] = oracle.bfs(el, s)
    ref = _C2[key]
    np.testing.assert_array_equal(d, ref.depths)
    np.testing.assert_array_equal(st.per_source_m, ref.m_s)
    np.testing.assert_array_equal(st.per_source_digest, ref.digest)
    # a directed graph is not symmetric: some pair must differ from the undirected BFS
    und = _oracle_c2(ibfs_gen.CONFIGS["c2"].edges(), s) if W == 128 and kind == "auto" else None
    if und is not None:
        assert not np.array_equal(und.depths, d)


def test_directed_from_csr_matches_from_edges_and_khop():
    cfg = ibfs_gen.CONFIGS["d2"]
    el = cfg.edges()
    og = oracle.OracleGraph.from_edges(el)
    off, adj = og.adjacency()
    roff, radj = _transpose_csr(el.nv, off, adj)
    g = P.Graph.from_csr(off, adj, rev_offsets=roff, rev_adj=radj)
    src = cfg.sources(el)[:128]
    d, st = gpu_depths(g, src, 128, want_digest=True)
    ref = og.bfs(src)
    np.testing.assert_array_equal(d, ref.depths)
    np.testing.assert_array_equal(st.per_source_m, ref.m_s)
    d3, _ = gpu_depths(g, src, 128, max_depth=3)
    np.testing.assert_array_equal(d3, og.bfs(src, max_depth=3).depths)
    # the out-edge rows come back unchanged
    eo, ea = g.export_csr()
    np.testing.assert_array_equal(eo, off)
    np.testing.assert_array_equal(ea, adj)
    # a reverse CSR that is not the transpose is rejected
    bad_off = roff.copy()
    bad_off[1:-1] = np.minimum(bad_off[1:-1] + 1, bad_off[-1])
    with pytest.raises(Exception):
        P.Graph.from_csr(off, adj, rev_offsets=bad_off, rev_adj=radj)


# ------------------------------------- byte-JSA joint engine (ablation rung, NEXT #3)
# §4: the Joint Status Array keeps a depth byte per (vertex, instance); the
# same depths, m_s and digests as the oracle (and as the bitwise engine).
@pytest.mark.parametrize("W", [32, 64, 128])
@pytest.mark.parametrize("kind", SCHEDULES)
def test_joint_engine_fig1(W, kind):
    fx = read_fig1()
    el = ibfs_gen.from_pairs(fx["nv"], fx["edges"])
    g = P.Graph.from_edgelist(el)
    d, st = gpu_depths(g, fx["sources"], W, engine="joint", want_digest=True, **run_kwargs(kind))
    np.testing.assert_array_equal(d, fx["depths"])
    ref = oracle.bfs(el, fx["sources"])
    np.testing.assert_array_equal(st.per_source_m, ref.m_s)
    np.testing.assert_array_equal(st.per_source_digest, ref.digest)


def test_joint_engine_random_tiny():
    rng = np.random.default_rng(909)
    for trial in range(60):
        nv = int(rng.integers(1, 60))
        m = int(rng.integers(0, 3 * nv + 1))
        pairs = [(int(rng.integers(nv)), int(rng.integers(nv))) for _ in range(m)]
        directed = bool(trial % 3 == 0)
        el = ibfs_gen.from_pairs(nv, pairs if pairs else np.zeros((0, 2)), directed=directed)
        n = int(rng.integers(1, 200))
        src = rng.integers(0, nv, size=n).astype(np.uint32)
        W = int(rng.choice([32, 64, 128]))
        kind = SCHEDULES[trial % len(SCHEDULES)]
        k = int(rng.integers(1, 4)) if trial % 5 == 0 else None
        g = P.Graph.from_edgelist(el)
        d, st = gpu_depths(g, src, W, engine="joint", want_digest=True, max_depth=k, **run_kwargs(kind, rng))
        ref = oracle.bfs(el, src, max_depth=k)
        np.testing.assert_array_equal(d, ref.depths, err_msg=f"trial {trial} W={W} {kind} dir={directed} k={k}")
        np.testing.assert_array_equal(st.per_source_m, ref.m_s)
        np.testing.assert_array_equal(st.per_source_digest, ref.digest)


@pytest.mark.parametrize("name", ["c1", "c2", "d2"])
def test_joint_engine_configs(name):
    cfg = ibfs_gen.CONFIGS[name]
    el = cfg.edges()
    src = cfg.sources(el)
    g = P.Graph.from_edgelist(el)
    s = src[g.plan(src, cfg.group_bits)]
    d, st = gpu_depths(g, s, cfg.group_bits, engine="joint", want_digest=True)
    db, stb = gpu_depths(g, s, cfg.group_bits, want_digest=True)
    np.testing.assert_array_equal(d, db)  # bitwise and joint engines agree
    ref = oracle.bfs(el, s)
    np.testing.assert_array_equal(d, ref.depths)
    np.testing.assert_array_equal(st.per_source_m, ref.m_s)
    np.testing.assert_array_equal(st.per_source_digest, ref.digest)


# ------------------------------------------ late-list overflow (depth-kernel skipping)
@pytest.mark.parametrize("late_cap", [1, 7, 300])
def test_late_list_overflow_falls_back_to_snapshots(late_cap):
    # sparse-committed levels put their new vertices on a per-group late list instead of
    # having the depth kernel read their snapshot.  A tiny late_cap makes
    # the list overflow: the overflowing level (and every later sparse one) is read from
    # its snapshot instead.  Results never change.  A 100-vertex path beside a 20,000-vertex random component: path sources discover one
    # or two vertices per level, far below the sparse-commit threshold (writes <= nva/128)
    rng = np.random.default_rng(77)
    npath, ncomp = 100, 20000
    pairs = [(i, i + 1) for i in range(npath - 1)]
    pairs += [(npath + int(a), npath + int(b)) for a, b in rng.integers(0, ncomp, size=(3 * ncomp, 2))]
    el = ibfs_gen.from_pairs(npath + ncomp, pairs)
    g = P.Graph.from_edgelist(el)
    src = np.concatenate([np.arange(0, npath, 3), npath + np.arange(0, 40)]).astype(np.uint32)
    ref = oracle.bfs(el, src)
    for W in (32, 128):
        d, st = gpu_depths(g, src, W, late_cap=late_cap, want_digest=True)
        np.testing.assert_array_equal(d, ref.depths)
        np.testing.assert_array_equal(st.per_source_digest, ref.digest)
        # the overflow path ran: fewer skipped snapshots -> more snapshot bytes read
        _, st0 = gpu_depths(g, src, W, want_digest=True)
        if late_cap < 100:
            assert st.depth_bytes > st0.depth_bytes
    cfg = ibfs_gen.CONFIGS["c2"]
    el = cfg.edges()
    s = cfg.sources(el)
    g = P.Graph.from_edgelist(el)
    d, st = gpu_depths(g, s, 128, late_cap=late_cap, want_digest=True)
    ref = _oracle_c2(el, s)
    np.testing.assert_array_equal(d, ref.depths)
    np.testing.assert_array_equal(st.per_source_digest, ref.digest)
