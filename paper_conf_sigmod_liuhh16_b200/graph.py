"""Python binding of include/ibfs.h -- argument marshalling only.

Every step of the traversal runs in libibfs.so's sm_100a kernels; this module turns
numpy arrays / torch tensors into pointers, fills the option structs, and returns the
statistics.  Names follow the C ABI: ``Graph.from_csr`` -> ``ibfs_load_csr``,
``Graph.from_edges`` -> ``ibfs_load_edges``, ``Graph.plan`` -> ``ibfs_plan_groups``,
``Graph.run`` -> ``ibfs_run_ex``.
"""
from __future__ import annotations

import ctypes as C
from dataclasses import dataclass, field

import numpy as np

from . import _lib
from ._lib import check

_STAT_FIELDS = tuple(f for f, _ in _lib.Stats._fields_
                     if f not in ("per_source_m", "per_source_digest", "level_cap", "per_level"))
_DIRS = {"auto": _lib.DIR_AUTO, "td": _lib.DIR_TD_ONLY, "bu_from": _lib.DIR_BU_FROM,
         "schedule": _lib.DIR_SCHEDULE}
_PLAN_MODES = {"groupby": 0, "random": 1, "identity": 2}


def _ptr(x):
    """(pointer, keepalive) for numpy arrays, torch tensors or None."""
    if x is None:
        return None, None
    if isinstance(x, np.ndarray):
        if not x.flags["C_CONTIGUOUS"]:
            x = np.ascontiguousarray(x)
        return x.ctypes.data, x
    try:
        import torch
        if isinstance(x, torch.Tensor):
            if not x.is_contiguous():
                raise ValueError("tensor must be contiguous")
            return x.data_ptr(), x
    except ImportError:
        pass
    raise TypeError(f"unsupported buffer type {type(x)}")


def _u32(x):
    """uint32 view of a source list (numpy or torch int32/uint32), keeping device tensors."""
    if isinstance(x, np.ndarray):
        return np.ascontiguousarray(x, dtype=np.uint32)
    try:
        import torch
        if isinstance(x, torch.Tensor):
            if x.dtype not in (torch.int32, torch.uint32):
                x = x.to(torch.int32)
            return x.contiguous()
    except ImportError:
        pass
    return np.ascontiguousarray(np.asarray(x), dtype=np.uint32)


def _len(x) -> int:
    return int(x.shape[0])


@dataclass
class RunStats:
    traverse_ms: float
    finalize_ms: float
    copyout_ms: float
    edges_traversed: int
    edges_inspected: int
    bytes_algorithmic: int
    sd_fq_td: int
    sd_jfq_td: int
    sd_fq_bu: int
    sd_jfq_bu: int
    n_groups: int
    max_levels: int
    levels_td: int
    levels_bu: int
    n_launches: int
    level_ms: float
    expand_ms: float
    commit_ms: float
    init_ms: float
    depth_ms: float
    level_launches: int
    init_launches: int
    depth_launches: int
    expand_bytes: int
    commit_bytes: int
    init_bytes: int
    depth_bytes: int
    level_gap_ms: float
    commit_bytes_moved: int
    depth_rows_bytes: int
    ms_bytes: int
    ms_ms: float
    ms_launches: int
    level_launches_live: int
    words_gathered: int
    host_setup_ms: float
    host_wait_ms: float
    host_total_ms: float
    clean_ms: float
    clean_launches: int
    clean_bytes: int
    per_source_m: np.ndarray | None = None
    per_source_digest: np.ndarray | None = None
    per_level: list = field(default_factory=list)

    @property
    def gteps(self) -> float:
        return self.edges_traversed / (self.traverse_ms * 1e-3) / 1e9 if self.traverse_ms > 0 else 0.0

    @property
    def sd_td(self) -> float:
        return self.sd_fq_td / self.sd_jfq_td if self.sd_jfq_td else 0.0

    @property
    def sd_bu(self) -> float:
        return self.sd_fq_bu / self.sd_jfq_bu if self.sd_jfq_bu else 0.0


class Graph:
    """A CSR graph resident on one GPU (ibfs_graph)."""

    def __init__(self, handle, device: int):
        self._h = handle
        self.device = device
        lib = _lib.load()
        nv, ne, md, dev = C.c_uint32(), C.c_uint64(), C.c_uint32(), C.c_int()
        check(lib.ibfs_graph_info(self._h, C.byref(nv), C.byref(ne), C.byref(md), C.byref(dev)))
        self.nv, self.ne, self.max_degree = int(nv.value), int(ne.value), int(md.value)

    # ---- loading -------------------------------------------------------------------
    def sort_rows(self, hub_first: bool = True) -> "Graph":
        """ibfs_graph_sort_rows: neighbour lists by outdegree, descending (results unchanged)."""
        check(_lib.load().ibfs_graph_sort_rows(self._h, _lib.ROWS_HUB_FIRST if hub_first else _lib.ROWS_KEEP))
        return self

    @classmethod
    def from_csr(cls, offsets, adj, device: int = 0, rev_offsets=None, rev_adj=None) -> "Graph":
        """ibfs_load_csr.  Directed graphs also pass the in-edge CSR (rev_offsets, rev_adj)."""
        lib = _lib.load()
        if isinstance(offsets, np.ndarray):
            offsets = np.ascontiguousarray(offsets, dtype=np.uint64)
            adj = np.ascontiguousarray(adj, dtype=np.uint32)
        if isinstance(rev_offsets, np.ndarray):
            rev_offsets = np.ascontiguousarray(rev_offsets, dtype=np.uint64)
            rev_adj = np.ascontiguousarray(rev_adj, dtype=np.uint32)
        po, ko = _ptr(offsets)
        pa, ka = _ptr(adj)
        pro, kro = _ptr(rev_offsets)
        pra, kra = _ptr(rev_adj)
        nv = _len(offsets) - 1
        ne = _len(adj)
        h = C.c_void_p()
        check(lib.ibfs_load_csr(int(device), nv, ne, po, pa if ne else None, pro,
                                pra if (ne and pro) else None, C.byref(h)))
        return cls(h, device)

    @classmethod
    def from_edges(cls, nv: int, u, v, device: int = 0, directed: bool = False) -> "Graph":
        lib = _lib.load()
        if isinstance(u, np.ndarray):
            u = np.ascontiguousarray(u, dtype=np.uint32)
            v = np.ascontiguousarray(v, dtype=np.uint32)
        pu, ku = _ptr(u)
        pv, kv = _ptr(v)
        m = _len(u)
        h = C.c_void_p()
        check(lib.ibfs_load_edges(int(device), int(nv), m, pu if m else None, pv if m else None,
                                  1 if directed else 0, C.byref(h)))
        return cls(h, device)

    @classmethod
    def from_edgelist(cls, el, device: int = 0, hub_first: bool = True) -> "Graph":
        g = cls.from_edges(el.nv, el.u, el.v, device, getattr(el, "directed", False))
        return g.sort_rows(True) if hub_first else g

    def close(self):
        if getattr(self, "_h", None):
            _lib.load().ibfs_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def export_csr(self):
        off = np.empty(self.nv + 1, dtype=np.uint64)
        adj = np.empty(max(self.ne, 1), dtype=np.uint32)
        check(_lib.load().ibfs_graph_export_csr(self._h, off.ctypes.data, adj.ctypes.data))
        return off, adj[: self.ne]

    # ---- planning ------------------------------------------------------------------
    def plan(self, sources, group_bits: int = 128, mode: str = "groupby", q: int = 128,
             p=(4, 16, 64, 128), seed: int = 3, hops: int = 1) -> np.ndarray:
        lib = _lib.load()
        src = _u32(sources)
        ps, ks = _ptr(src)
        n = _len(src)
        pp = _lib.PlanParams()
        lib.ibfs_plan_params_default(C.byref(pp))
        pp.mode = _PLAN_MODES[mode]
        pp.q = int(q)
        pp.n_p = len(p)
        for i, x in enumerate(p):
            pp.p[i] = int(x)
        pp.hops = int(hops)
        pp.seed = int(seed)
        perm = np.empty(max(n, 1), dtype=np.uint32)
        ng = C.c_uint32()
        check(lib.ibfs_plan_groups(self._h, ps if n else None, n, int(group_bits), C.byref(pp),
                                   perm.ctypes.data, C.byref(ng)))
        return perm[:n]

    # ---- traversal -----------------------------------------------------------------
    def run(self, sources, group_bits: int = 128, out="device", direction: str = "auto",
            schedule: str | None = None, bu_from: int = 2, alpha: float = 3.0, beta: float = 24.0,
            groups_in_flight: int = 0, stream=None, timing: bool = False, want_m: bool = True,
            want_digest: bool = False, level_cap: int = 130, split: str = "auto",
            split_mod: int = 2, split_div: float = 512.0, max_depth: int | None = None,
            engine: str = "bitwise", late_cap: int = 0):
        """n concurrent BFS instances; returns (depths, RunStats).

        engine: "bitwise" (the product path) or "joint" (the byte-JSA joint traversal of §4,
        kept for the ablation ladder; same results).
        max_depth = k >= 1: k-hop mode, the first k levels only (the reachability index of
        §8.7); vertices farther than k hops are -1.  None = plain BFS.

        split: "auto" | "off" | "force" -- per-instance direction inside a bottom-up level
        (include/ibfs.h IBFS_SPLIT_*); never changes results.

        out: "device" (allocate a torch int8 [n, nv] CUDA tensor), "host" (numpy), None
        (no rows returned; they are still materialised on the device), or a caller buffer
        (torch tensor on the device or host, or numpy) of int8 [n, nv].
        """
        lib = _lib.load()
        src = _u32(sources)
        n = _len(src)
        if isinstance(out, str):
            if out == "device":
                import torch
                out = torch.empty((n, self.nv), dtype=torch.int8, device=f"cuda:{self.device}")
            elif out == "host":
                out = np.empty((n, self.nv), dtype=np.int8)
            else:
                raise ValueError(out)
        ps, ks = _ptr(src)
        po, ko = _ptr(out)
        opts = _lib.RunOpts()
        lib.ibfs_run_opts_default(C.byref(opts))
        sched_buf = None
        if schedule is not None:
            direction = "schedule"
            sched_buf = (C.c_uint8 * max(len(schedule), 1))(*[ord(c) for c in schedule])
            opts.schedule = C.cast(sched_buf, C.c_void_p)
            opts.schedule_len = len(schedule)
        opts.direction = _DIRS[direction]
        opts.bu_from = int(bu_from)
        opts.alpha = float(alpha)
        opts.beta = float(beta)
        opts.groups_in_flight = int(groups_in_flight)
        if stream is None:
            try:
                import torch
                if torch.cuda.is_available():
                    stream = torch.cuda.current_stream(self.device)
            except ImportError:
                stream = None
        opts.cuda_stream = getattr(stream, "cuda_stream", stream) or None
        opts.timing = 1 if timing else 0
        opts.split = {"auto": 0, "off": 1, "force": 2}[split]
        opts.split_mod = int(split_mod)
        opts.split_div = float(split_div)
        if max_depth is not None:
            if int(max_depth) < 1:
                raise ValueError("max_depth must be >= 1 (None = unbounded)")
            opts.max_depth = int(max_depth)
        opts.engine = {"bitwise": 0, "joint": 1}[engine]
        opts.late_cap = int(late_cap)
        st = _lib.Stats()
        m_arr = np.zeros(max(n, 1), dtype=np.uint64) if want_m else None
        d_arr = np.zeros(max(n, 1), dtype=np.uint64) if want_digest else None
        lv = (_lib.LevelStats * level_cap)()
        st.per_source_m = m_arr.ctypes.data if want_m else None
        st.per_source_digest = d_arr.ctypes.data if want_digest else None
        st.level_cap = level_cap
        st.per_level = C.cast(lv, C.c_void_p)
        check(lib.ibfs_run_ex(self._h, ps if n else None, n, int(group_bits), po, C.byref(opts),
                              C.byref(st)))
        rs = RunStats(**{f: getattr(st, f) for f in _STAT_FIELDS})
        rs.per_source_m = m_arr[:n] if want_m else None
        rs.per_source_digest = d_arr[:n] if want_digest else None
        rs.per_level = [
            {f: getattr(lv[i], f) for f, _ in _lib.LevelStats._fields_}
            for i in range(min(level_cap, st.max_levels))
        ]
        return out, rs

    def run_plain(self, sources, group_bits: int = 128, out=None):
        """ibfs_run: the plain entry point north_star names (no options, no statistics; the
        legacy default stream; returns after the work completes).  out: int8 [n, nv] host
        (numpy / torch CPU) or device (torch CUDA) buffer, or None."""
        lib = _lib.load()
        src = _u32(sources)
        n = _len(src)
        ps, ks = _ptr(src)
        po, ko = _ptr(out)
        check(lib.ibfs_run(self._h, ps if n else None, n, int(group_bits), po))
        return out


def use_torch_allocator(enable: bool = True) -> None:
    """Route libibfs device scratch through torch's caching allocator (ibfs_set_allocator)."""
    lib = _lib.load()
    if not enable:
        check(lib.ibfs_set_allocator(None, None, None))
        _ALLOC_KEEP.clear()
        return
    import torch

    def _alloc(nbytes, dev, ctx):
        try:
            return torch.cuda.caching_allocator_alloc(int(nbytes), int(dev))
        except Exception:
            return None

    def _release(ptr, dev, ctx):
        torch.cuda.caching_allocator_delete(ptr)

    a, r = _lib.ALLOC_FN(_alloc), _lib.RELEASE_FN(_release)
    _ALLOC_KEEP[:] = [a, r]
    check(lib.ibfs_set_allocator(C.cast(a, C.c_void_p), C.cast(r, C.c_void_p), None))


_ALLOC_KEEP: list = []
