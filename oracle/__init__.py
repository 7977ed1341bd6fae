"""CPU oracle for the iBFS hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
(``paper_conf_sigmod_liuhh16_b200``) never imports it, and the two share no code: the
only common dependency is the seeded input generator ``ibfs_gen``.

Contents
--------
* ``OracleGraph`` / ``bfs``  -- plain C textbook BFS per source (``oracle.c``): depth rows,
  m_s (TEPS numerator), digests.  Follows PAPER.md P:L171-L175 (BFS levels) and reaches the
  shortest-path definition of P:L43-L49 exactly.
* ``planner.groupby``        -- the outdegree-based GroupBy rules of §5.2 (P:L567-L619,
  P:L661), step by step in the paper's order (parity *unpinned* beyond invariants and a
  hand-built example: the depths do not depend on it).
* ``stats``                  -- sharing degree (Eq. 1) and per-level frontier
  sizes, computed from depth rows.
* ``certify``                -- the complete BFS-depth certificate;
  ``OracleGraph.certify`` is the same certificate as C loops for full-size rows.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")
_lib = None

ORACLE_E_RANGE = -4


def build(force: bool = False) -> str:
    """Compile oracle.c (plain C, -O3, pthreads) -> liboracle.so."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O3", "-march=x86-64-v2", "-fPIC", "-shared", "-pthread",
                               "-o", _SO, _SRC])
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        P = ctypes.c_void_p
        lib.oracle_graph_new.restype = P
        lib.oracle_graph_new.argtypes = [ctypes.c_uint64, ctypes.c_uint64, P, P, ctypes.c_int, ctypes.c_int]
        lib.oracle_graph_free.restype = None
        lib.oracle_graph_free.argtypes = [P]
        lib.oracle_graph_nv.restype = ctypes.c_uint64
        lib.oracle_graph_nv.argtypes = [P]
        lib.oracle_graph_ne.restype = ctypes.c_uint64
        lib.oracle_graph_ne.argtypes = [P]
        lib.oracle_graph_export.restype = None
        lib.oracle_graph_export.argtypes = [P, P, P]
        lib.oracle_bfs.restype = ctypes.c_int
        lib.oracle_bfs.argtypes = [P, P, ctypes.c_uint64, P, P, P, P, P, ctypes.c_int]
        lib.oracle_bfs_k.restype = ctypes.c_int
        lib.oracle_bfs_k.argtypes = [P, P, ctypes.c_uint64, ctypes.c_int32, P, P, P, P, P, ctypes.c_int]
        lib.oracle_certify.restype = ctypes.c_int
        lib.oracle_certify.argtypes = [P, ctypes.c_uint32, P]
        _lib = lib
    return _lib


class OracleResult:
    def __init__(self, n):
        self.depths = None
        self.m_s = np.zeros(n, dtype=np.uint64)
        self.digest = np.zeros(n, dtype=np.uint64)
        self.ecc = np.zeros(n, dtype=np.int32)
        self.reached = np.zeros(n, dtype=np.uint64)
        self.status = 0


class OracleGraph:
    """Adjacency lists built from the raw tuples (never from the GPU path's CSR)."""

    def __init__(self, nv: int, u: np.ndarray, v: np.ndarray, directed: bool = False,
                 threads: int | None = None):
        lib = _load()
        self._u = np.ascontiguousarray(u, dtype=np.uint32)
        self._v = np.ascontiguousarray(v, dtype=np.uint32)
        self.nv = int(nv)
        self.directed = bool(directed)
        self._h = lib.oracle_graph_new(self.nv, int(self._u.shape[0]), self._u.ctypes.data,
                                       self._v.ctypes.data, 1 if directed else 0,
                                       int(threads or os.cpu_count() or 1))
        if not self._h:
            raise ValueError("oracle_graph_new failed (bad vertex id or out of memory)")
        del self._u, self._v
        self._csr = None

    @classmethod
    def from_edges(cls, el) -> "OracleGraph":
        return cls(el.nv, el.u, el.v, getattr(el, "directed", False))

    def __del__(self):
        h = getattr(self, "_h", None)
        if h and _lib is not None:
            _lib.oracle_graph_free(h)
            self._h = None

    @property
    def ne(self) -> int:
        return int(_load().oracle_graph_ne(self._h))

    def adjacency(self):
        """(offsets u64[nv+1], adj u32[ne]) of the oracle's own adjacency lists."""
        if self._csr is None:
            off = np.empty(self.nv + 1, dtype=np.uint64)
            adj = np.empty(max(self.ne, 1), dtype=np.uint32)
            _load().oracle_graph_export(self._h, off.ctypes.data, adj.ctypes.data)
            self._csr = (off, adj[: self.ne])
        return self._csr

    def degrees(self) -> np.ndarray:
        off, _ = self.adjacency()
        return np.diff(off).astype(np.uint64)

    def bfs(self, sources, want_depths: bool = True, threads: int | None = None,
            max_depth: int | None = None) -> OracleResult:
        """One textbook BFS per source.  depths: int8 [n][nv], row r <-> sources[r].

        max_depth = k caps every search at its first k levels -- the k-hop reachability
        index of §8.7 ("computes the first k levels BFS"): vertices farther
        than k hops are -1, and m_s / digest / reached count the vertices within k hops."""
        lib = _load()
        src = np.ascontiguousarray(np.asarray(sources, dtype=np.uint32))
        n = int(src.shape[0])
        res = OracleResult(n)
        out_ptr = None
        if want_depths:
            res.depths = np.empty((n, self.nv), dtype=np.int8)
            out_ptr = res.depths.ctypes.data
        t = threads or os.cpu_count() or 1
        k = -1 if max_depth is None else int(max_depth)
        if max_depth is not None and k < 0:
            raise ValueError("max_depth must be >= 0")
        res.status = lib.oracle_bfs_k(self._h, src.ctypes.data if n else None, n, k, out_ptr,
                                    res.m_s.ctypes.data, res.digest.ctypes.data, res.ecc.ctypes.data,
                                    res.reached.ctypes.data, int(t))
        if res.status not in (0, ORACLE_E_RANGE):
            raise ValueError(f"oracle_bfs failed: {res.status}")
        return res


    CERTIFY_REASONS = {1: "(o) value < -1", 2: "(i) d(s) != 0", 3: "(ii) reachability differs across an edge",
                       4: "(ii) |d(u)-d(v)| > 1 across an edge", 5: "(iii) a vertex other than s has depth 0",
                       6: "(iii) a reached vertex has no neighbour one level closer"}

    def certify(self, s: int, row) -> str | None:
        """The complete certificate (certify.py's conditions, C loops; undirected graphs):
        None if `row` is the exact BFS depth row from s, else the violated condition."""
        if self.directed:
            raise ValueError("the certificate is for undirected graphs")
        d = np.ascontiguousarray(np.asarray(row), dtype=np.int8)
        if d.shape != (self.nv,):
            raise ValueError("row must have nv entries")
        rc = _load().oracle_certify(self._h, int(s), d.ctypes.data)
        if rc < 0:
            raise ValueError("bad source")
        return None if rc == 0 else self.CERTIFY_REASONS[rc]


def bfs(el, sources, want_depths=True, threads=None, max_depth=None) -> OracleResult:
    return OracleGraph.from_edges(el).bfs(sources, want_depths, threads, max_depth)


from . import planner, stats, certify  # noqa: E402,F401
