"""The seeded input generator (ibfs_gen): determinism, counts, and the R-MAT recipe."""
from __future__ import annotations

import numpy as np

import ibfs_gen


def test_determinism_and_thread_invariance():
    a = ibfs_gen.rmat(12, 16, ibfs_gen.KRONECKER, seed=11, threads=1)
    b = ibfs_gen.rmat(12, 16, ibfs_gen.KRONECKER, seed=11, threads=5)
    c = ibfs_gen.rmat(12, 16, ibfs_gen.KRONECKER, seed=12, threads=5)
    np.testing.assert_array_equal(a.u, b.u)
    np.testing.assert_array_equal(a.v, b.v)
    assert not np.array_equal(a.u, c.u)
    assert a.m == 16 << 12 and a.nv == 1 << 12
    assert int(a.u.max()) < a.nv and int(a.v.max()) < a.nv


def test_quadrant_probabilities_unrelabeled():
    # Without relabeling, bit b of (u, v) picks quadrant (ii, jj) with probabilities
    # A, B, C, D.  Check the top bit's empirical frequencies.
    scale = 14
    A, B, C = ibfs_gen.KRONECKER
    el = ibfs_gen.rmat(scale, 16, (A, B, C), seed=3, relabel=False)
    top = scale - 1
    ii = (el.u >> top) & 1
    jj = (el.v >> top) & 1
    m = el.m
    freq = [np.mean((ii == a) & (jj == b)) for a, b in ((0, 0), (0, 1), (1, 0), (1, 1))]
    exp = [A, B, C, 1 - A - B - C]
    for f, e in zip(freq, exp):
        assert abs(f - e) < 5 * np.sqrt(e * (1 - e) / m)


def test_relabel_is_permutation_of_unrelabeled():
    raw = ibfs_gen.rmat(10, 4, ibfs_gen.RMAT, seed=5, relabel=False)
    lab = ibfs_gen.rmat(10, 4, ibfs_gen.RMAT, seed=5, relabel=True)
    perm = ibfs_gen.permutation(1 << 10, 5)
    assert sorted(perm.tolist()) == list(range(1 << 10))
    np.testing.assert_array_equal(perm[raw.u], lab.u)
    np.testing.assert_array_equal(perm[raw.v], lab.v)


def test_skew_sanity_graph500():
    # Graph500 s16 ef16 has ~29 % isolated vertices and max degree ~2.6e4.
    el = ibfs_gen.rmat(16, 16, ibfs_gen.KRONECKER, seed=1)
    deg = np.bincount(el.u, minlength=el.nv) + np.bincount(el.v, minlength=el.nv)
    iso = np.mean(deg == 0)
    assert 0.2 < iso < 0.4
    assert 5_000 < deg.max() < 100_000


def test_sources_distinct_touched():
    el = ibfs_gen.rmat(12, 16, ibfs_gen.KRONECKER, seed=1)
    s = ibfs_gen.sample_sources(el, 500, seed=2)
    deg = np.bincount(el.u, minlength=el.nv) + np.bincount(el.v, minlength=el.nv)
    assert len(s) == 500 and len(set(s.tolist())) == 500
    assert (deg[s] > 0).all()
    np.testing.assert_array_equal(s, ibfs_gen.sample_sources(el, 500, seed=2))
