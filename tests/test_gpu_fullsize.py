"""Full-size parity at the launch shape bench.py times.

Each test builds bench.py's own ``Workload`` (GroupBy hops = 2 plan, LPT share, G groups
per ``Graph.run`` call, the library's automatic launch batches, rows materialised in a
device buffer) and runs every step of one cycle through the C ABI.  The expected values
come from the oracle only:

* ``tests/golden/<cfg>_ms_digest.npz`` -- m_s and the order-free row digest of EVERY
  source, keyed by source id in generator order, written by ``tools/make_golden.py``
  (which imports only ``oracle/`` and ``ibfs_gen``);
* full rows of sampled sources recomputed here by the oracle (one textbook BFS each);
* the complete BFS certificate (``OracleGraph.certify``) on more rows.

Depths are integers: every comparison is bit-exact (PAPER.md P:L43-L49 shortest paths,
P:L887 results stored in GPU memory).
"""
from __future__ import annotations

import os

import numpy as np
import pytest

import ibfs_gen
import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import bench  # noqa: E402  (the bench's Workload: the same schedule and options)
import paper_conf_sigmod_liuhh16_b200 as P  # noqa: E402

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def _golden(name):
    path = os.path.join(GOLDEN, f"{name}_ms_digest.npz")
    if not os.path.exists(path):
        pytest.fail(f"missing {path}: run tools/make_golden.py {name}")
    z = np.load(path)
    return {int(s): (int(m), int(d)) for s, m, d in zip(z["sources"], z["m_s"], z["digest"])}, z


def _run_cycle(name, sample_rows=0, seed=5, out_rows_host=None):
    """Every step of one cycle of bench.py's workload on `name`; returns per-source
    (m_s, digest) dicts and the host copies of the sampled rows."""
    args = bench.parse(["--config", name])
    cfg = ibfs_gen.CONFIGS[name]
    el = cfg.edges()
    g = P.Graph.from_edgelist(el)
    wl = bench.Workload(args, g, el)
    sched = wl.sched
    n = len(wl.s_plan)
    pick = set()
    if sample_rows:
        pick = set(int(x) for x in np.random.default_rng(seed).choice(n, size=sample_rows, replace=False))
    out = torch.empty((wl.G * wl.W, g.nv), dtype=torch.int8, device="cuda")
    got_m, got_d, rows_host = {}, {}, {}
    stream = torch.cuda.current_stream()
    for k in range(sched.steps_per_cycle):
        rows = sched.step_rows(k)
        s = wl.s_plan[rows]
        _, st = g.run(s, wl.W, out=out[: len(s)], stream=stream, want_digest=True, **wl.run_kw)
        torch.cuda.synchronize()
        for i, r in enumerate(rows):
            src = int(wl.s_plan[r])
            got_m[src] = int(st.per_source_m[i])
            got_d[src] = int(st.per_source_digest[i])
            if int(r) in pick and int(r) not in rows_host:
                rows_host[int(r)] = out[i].cpu().numpy()
    assert sorted(int(x) for x in got_m) == sorted(int(x) for x in wl.s_plan)  # one cycle covers the plan
    return el, g, wl, got_m, got_d, rows_host


def _compare_golden(name, got_m, got_d):
    gold, _ = _golden(name)
    assert set(gold) == set(got_m)
    bad_m = [s for s in gold if gold[s][0] != got_m[s]]
    bad_d = [s for s in gold if gold[s][1] != got_d[s]]
    assert not bad_m, f"{name}: m_s differs for {len(bad_m)} sources, e.g. {bad_m[:5]}"
    assert not bad_d, f"{name}: digest differs for {len(bad_d)} sources, e.g. {bad_d[:5]}"


def _compare_rows(el, wl, rows_host, certify_extra=()):
    og = oracle.OracleGraph.from_edges(el)
    keys = sorted(rows_host)
    for i in range(0, len(keys), 16):  # oracle rows in chunks (host memory)
        chunk = keys[i:i + 16]
        ref = og.bfs(wl.s_plan[chunk])
        for j, r in enumerate(chunk):
            np.testing.assert_array_equal(rows_host[r], ref.depths[j], err_msg=f"row {r} (source {wl.s_plan[r]})")
    for r, row in certify_extra:
        assert og.certify(int(wl.s_plan[r]), row) is None, f"certificate rejects row {r}"


@pytest.mark.parametrize("name", ["c5"])
def test_c5_bench_shape_all_digests_and_sampled_rows(name):
    # all 4,096 sources: 32 groups, 4 per step (one launch batch), 8 steps -- the bench
    # line's exact shape; 64 sampled rows vs the oracle, 8 more through the certificate
    el, g, wl, got_m, got_d, rows_host = _run_cycle(name, sample_rows=72, seed=26)
    _compare_golden(name, got_m, got_d)
    keys = sorted(rows_host)
    assert len(keys) == 72
    sampled = {r: rows_host[r] for r in keys[:64]}
    extra = [(r, rows_host[r]) for r in keys[64:]]
    _compare_rows(el, wl, sampled, extra)


def test_c3_bench_shape_all_digests_and_sampled_rows():
    # all 1,024 sources: 8 groups in one step (two launch batches of 4), 64 sampled rows
    el, g, wl, got_m, got_d, rows_host = _run_cycle("c3", sample_rows=72, seed=24)
    assert wl.sched.steps_per_cycle == 1
    _compare_golden("c3", got_m, got_d)
    keys = sorted(rows_host)
    _compare_rows(el, wl, {r: rows_host[r] for r in keys[:64]}, [(r, rows_host[r]) for r in keys[64:]])


def test_c4_apsp_bench_shape_all_digests():
    # all 262,144 sources (APSP): 2,048 groups, 256 per step (two launch batches of 128),
    # 8 steps; 256 sampled rows vs the oracle and a symmetry block d(s,t) = d(t,s)
    el, g, wl, got_m, got_d, rows_host = _run_cycle("c4", sample_rows=256, seed=18)
    assert wl.sched.steps_per_cycle == 8
    _compare_golden("c4", got_m, got_d)
    _compare_rows(el, wl, rows_host)
    src = {int(wl.s_plan[r]): rows_host[r] for r in rows_host}
    ids = sorted(src)[:200]
    block = np.array([[src[a][b] for b in ids] for a in ids])
    np.testing.assert_array_equal(block, block.T)


def test_golden_files_are_oracle_written():
    # the golden recipe names the generator config and the oracle; Σ m_s is the TEPS
    # numerator of a whole cycle (each source once)
    for name in ("c3", "c4", "c5"):
        _, z = _golden(name)
        assert "oracle/oracle.c" in str(z["recipe"])
        cfg = ibfs_gen.CONFIGS[name]
        assert int(z["nv"]) == 1 << cfg.scale and int(z["tuples"]) == cfg.ef << cfg.scale
        assert len(z["sources"]) == (cfg.n_sources or (1 << cfg.scale))


# ------------------------------------------------------------ the plain ibfs_run call
def test_plain_ibfs_run_host_and_device_outputs():
    # ibfs_run (north_star's entry point: sources, n, group_bits, out_depths) with a host
    # and a device output buffer, on config 2 (all 128 sources, W = 32/128, ragged n)
    cfg = ibfs_gen.CONFIGS["c2"]
    el = cfg.edges()
    src = cfg.sources(el)
    g = P.Graph.from_edgelist(el)
    ref = oracle.bfs(el, src)
    for W in (32, 128):
        host = np.full((len(src), g.nv), 77, dtype=np.int8)
        g.run_plain(src, W, host)
        np.testing.assert_array_equal(host, ref.depths)
        dev = torch.full((len(src) - 5, g.nv), 77, dtype=torch.int8, device="cuda")
        g.run_plain(src[:-5], W, dev)
        np.testing.assert_array_equal(dev.cpu().numpy(), ref.depths[:-5])
    g.run_plain(src[:3], 64, None)  # no output: rows stay in device scratch


# --------------------------------------------------- the multi-rank bench, one GPU
def test_bench_two_ranks_gloo_partition(tmp_path):
    # bench.py --gpus 2 relaunches itself as 2 ranks (torch.distributed.run); here both
    # share the one GPU over gloo.  The ranks' groups partition the plan, the reported
    # rate is the summed edges over the max rank time, and Σ m_s of the first runs equals
    # the oracle's over every source.
    import json
    import subprocess
    import sys
    out = tmp_path / "b.json"
    cmd = [sys.executable, os.path.join(os.path.dirname(GOLDEN), "..", "bench.py"), "--gpus", "2",
           "--dist-backend", "gloo", "--config", "c2", "--group-bits", "32", "--groups-per-rank", "2",
           "--steps", "3", "--warmup", "3", "--no-e2e", "--no-cpu-baseline", "--no-clocks", "--json-out", str(out)]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    line = json.loads(out.read_text())
    assert line["n_gpus"] == 2
    ranks = line["shards"]["ranks"]
    groups = sorted(g for rk in ranks for g in rk["groups"])
    assert groups == list(range(4))  # c2: 128 sources / 32 = 4 groups, disjoint shares
    max_ms = max(rk["ms"] for rk in ranks)
    edges = sum(rk["edges"] for rk in ranks)
    assert abs(line["value"] - edges / (max_ms * 1e-3) / 1e9) <= 1e-3 * line["value"]
    cfg = ibfs_gen.CONFIGS["c2"]
    el = cfg.edges()
    ref = oracle.bfs(el, cfg.sources(el), want_depths=False)
    assert line["shards"]["sum_m_s_first_runs"] == int(ref.m_s.sum())
