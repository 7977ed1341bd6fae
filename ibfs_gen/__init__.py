"""Seeded synthetic input generator shared by the oracle and the CUDA path.

This module is the ONLY code both sides use (task rule ③).  It holds none of the
method's arithmetic: it draws R-MAT / Kronecker edge tuples (PAPER.md P:L975 for the
(A, B, C) values), a seeded vertex relabeling, and a seeded source sample.  The recipe
is stated in ``gen.c``'s header and in DESIGN.md §3.

The C code is compiled to ``libibfs_gen.so`` next to this file by
``__graft_entry__.build()`` (or lazily on first use with gcc).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libibfs_gen.so")
_SRC = os.path.join(_HERE, "gen.c")
_lib = None

# (A, B, C) per PAPER.md P:L975: Graph500 "KG" graphs and the GTgraph "RM" graph.
KRONECKER = (0.57, 0.19, 0.19)
RMAT = (0.45, 0.15, 0.15)


def build(force: bool = False) -> str:
    """Compile gen.c -> libibfs_gen.so (plain C, -O3, pthreads)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O3", "-march=x86-64-v2", "-fPIC", "-shared", "-pthread",
                               "-o", _SO, _SRC])
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        lib.ibfs_gen_rmat.restype = ctypes.c_int
        lib.ibfs_gen_rmat.argtypes = [ctypes.c_int, ctypes.c_uint32, ctypes.c_double, ctypes.c_double,
                                      ctypes.c_double, ctypes.c_uint64, ctypes.c_int, ctypes.c_int,
                                      ctypes.c_void_p, ctypes.c_void_p]
        lib.ibfs_gen_permutation.restype = None
        lib.ibfs_gen_permutation.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p]
        lib.ibfs_gen_sources.restype = ctypes.c_uint64
        lib.ibfs_gen_sources.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p,
                                         ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p]
        _lib = lib
    return _lib


@dataclass
class EdgeList:
    """Undirected tuple list (u[e], v[e]); duplicates and self-loops kept."""
    nv: int
    u: np.ndarray  # uint32 [m]
    v: np.ndarray  # uint32 [m]
    directed: bool = False

    @property
    def m(self) -> int:
        return int(self.u.shape[0])


def rmat(scale: int, ef: int, abc=RMAT, seed: int = 1, relabel: bool = True,
         threads: int | None = None) -> EdgeList:
    """R-MAT / Kronecker tuples: M = ef * 2^scale, recursion of SURVEY.md §8(d)."""
    lib = _load()
    m = int(ef) << int(scale)
    u = np.empty(m, dtype=np.uint32)
    v = np.empty(m, dtype=np.uint32)
    a, b, c = abc
    t = threads or min(os.cpu_count() or 1, 256)
    rc = lib.ibfs_gen_rmat(int(scale), int(ef), float(a), float(b), float(c), int(seed),
                           1 if relabel else 0, int(t), u.ctypes.data, v.ctypes.data)
    if rc != 0:
        raise ValueError("ibfs_gen_rmat: bad arguments")
    return EdgeList(1 << int(scale), u, v)


def permutation(n: int, seed: int) -> np.ndarray:
    lib = _load()
    out = np.empty(n, dtype=np.uint32)
    lib.ibfs_gen_permutation(int(n), int(seed), out.ctypes.data)
    return out


def sample_sources(el: EdgeList, count: int, seed: int = 2) -> np.ndarray:
    """First `count` of a seeded Fisher-Yates shuffle of the touched (deg > 0) vertices."""
    lib = _load()
    out = np.empty(max(int(count), 1), dtype=np.uint32)
    u = np.ascontiguousarray(el.u, dtype=np.uint32)
    v = np.ascontiguousarray(el.v, dtype=np.uint32)
    w = lib.ibfs_gen_sources(int(el.nv), int(el.m), u.ctypes.data, v.ctypes.data,
                             int(count), int(seed), out.ctypes.data)
    return out[:int(w)].copy()


def all_vertices(nv: int) -> np.ndarray:
    """APSP source list: every vertex in id order."""
    return np.arange(nv, dtype=np.uint32)


def from_pairs(nv: int, pairs, directed: bool = False) -> EdgeList:
    """Hand-built fixture graphs (tests)."""
    arr = np.asarray(list(pairs), dtype=np.uint32).reshape(-1, 2)
    return EdgeList(int(nv), arr[:, 0].copy(), arr[:, 1].copy(), directed)


@dataclass(frozen=True)
class Config:
    """One BASELINE.json config, as a synthetic input recipe."""
    name: str
    abc: tuple
    scale: int
    ef: int
    n_sources: int  # 0 = all vertices (APSP)
    group_bits: int
    graph_seed: int = 1
    source_seed: int = 2
    directed: bool = False  # tuple (u, v) = the edge u->v only

    def edges(self, threads=None) -> EdgeList:
        el = rmat(self.scale, self.ef, self.abc, self.graph_seed, True, threads)
        el.directed = self.directed
        return el

    def sources(self, el: EdgeList) -> np.ndarray:
        if self.n_sources == 0:
            return all_vertices(el.nv)
        return sample_sources(el, self.n_sources, self.source_seed)


CONFIGS = {
    "c1": Config("c1: R-MAT s10 ef16, i=64", RMAT, 10, 16, 64, 64),
    "c2": Config("c2: Kronecker s20 ef16, i=128", KRONECKER, 20, 16, 128, 128),
    "c3": Config("c3: R-MAT s24 ef32, i=1024", RMAT, 24, 32, 1024, 128),
    "c4": Config("c4: Kronecker s18 ef16, APSP i=|V|", KRONECKER, 18, 16, 0, 128),
    "c5": Config("c5: Kronecker s26 ef16, i=4096", KRONECKER, 26, 16, 4096, 128),
    # directed parity case (NEXT #1): config 2's tuples read as directed edges u->v
    "d2": Config("d2: directed Kronecker s20 ef16, i=128", KRONECKER, 20, 16, 128, 128, directed=True),
}
