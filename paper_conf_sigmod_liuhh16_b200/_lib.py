"""ctypes declarations of include/ibfs.h (argument marshalling only).

The shared library is loaded from this package directory; if it is missing the import of
the product API fails loudly -- there is no CPU fallback anywhere in this package.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
SO = os.environ.get("IBFS_LIB") or os.path.join(HERE, "libibfs.so")  # IBFS_LIB: A/B builds

IBFS_OK = 0
IBFS_E_INVALID = -1
IBFS_E_NOMEM = -2
IBFS_E_CUDA = -3
IBFS_E_RANGE = -4
IBFS_E_UNSUPPORTED = -5

DIR_AUTO, DIR_TD_ONLY, DIR_BU_FROM, DIR_SCHEDULE = 0, 1, 2, 3

EXPORTS = [
    "ibfs_version", "ibfs_last_error", "ibfs_load_csr", "ibfs_load_edges", "ibfs_graph_info",
    "ibfs_graph_export_csr", "ibfs_free", "ibfs_plan_params_default", "ibfs_plan_groups",
    "ibfs_run", "ibfs_run_opts_default", "ibfs_run_ex", "ibfs_set_allocator", "ibfs_graph_sort_rows",
]
ROWS_KEEP, ROWS_HUB_FIRST = 0, 1


class PlanParams(C.Structure):
    _fields_ = [("mode", C.c_uint32), ("q", C.c_uint32), ("n_p", C.c_uint32), ("p", C.c_uint32 * 8),
                ("hops", C.c_uint32), ("seed", C.c_uint64)]


class RunOpts(C.Structure):
    _fields_ = [("direction", C.c_uint32), ("bu_from", C.c_uint32), ("schedule", C.c_void_p),
                ("schedule_len", C.c_uint32), ("alpha", C.c_float), ("beta", C.c_float),
                ("groups_in_flight", C.c_uint32), ("cuda_stream", C.c_void_p), ("timing", C.c_uint32),
                ("split", C.c_uint32), ("split_mod", C.c_uint32), ("split_div", C.c_float),
                ("max_depth", C.c_uint32), ("engine", C.c_uint32), ("late_cap", C.c_uint32),
                ("reserved", C.c_uint32)]


class LevelStats(C.Structure):
    _fields_ = [("td_groups", C.c_uint32), ("bu_groups", C.c_uint32), ("jfq_td", C.c_uint64),
                ("fq_td", C.c_uint64), ("jfq_bu", C.c_uint64), ("fq_bu", C.c_uint64),
                ("inspected", C.c_uint64), ("new_pairs", C.c_uint64), ("gathered", C.c_uint64),
                ("expand_ms", C.c_double), ("commit_ms", C.c_double)]


class Stats(C.Structure):
    _fields_ = [("traverse_ms", C.c_double), ("finalize_ms", C.c_double), ("copyout_ms", C.c_double),
                ("edges_traversed", C.c_uint64), ("edges_inspected", C.c_uint64),
                ("bytes_algorithmic", C.c_uint64),
                ("sd_fq_td", C.c_uint64), ("sd_jfq_td", C.c_uint64), ("sd_fq_bu", C.c_uint64),
                ("sd_jfq_bu", C.c_uint64),
                ("n_groups", C.c_uint32), ("max_levels", C.c_uint32), ("levels_td", C.c_uint32),
                ("levels_bu", C.c_uint32), ("n_launches", C.c_uint64),
                ("level_ms", C.c_double), ("expand_ms", C.c_double), ("commit_ms", C.c_double),
                ("init_ms", C.c_double), ("depth_ms", C.c_double),
                ("level_launches", C.c_uint64), ("init_launches", C.c_uint64), ("depth_launches", C.c_uint64),
                ("expand_bytes", C.c_uint64), ("commit_bytes", C.c_uint64), ("init_bytes", C.c_uint64),
                ("depth_bytes", C.c_uint64), ("level_gap_ms", C.c_double),
                ("commit_bytes_moved", C.c_uint64), ("depth_rows_bytes", C.c_uint64), ("ms_bytes", C.c_uint64),
                ("ms_ms", C.c_double), ("ms_launches", C.c_uint64), ("level_launches_live", C.c_uint64),
                ("words_gathered", C.c_uint64), ("host_setup_ms", C.c_double), ("host_wait_ms", C.c_double),
                ("host_total_ms", C.c_double),
                ("clean_ms", C.c_double), ("clean_launches", C.c_uint64), ("clean_bytes", C.c_uint64),
                ("per_source_m", C.c_void_p), ("per_source_digest", C.c_void_p),
                ("level_cap", C.c_uint32), ("per_level", C.c_void_p)]


ALLOC_FN = C.CFUNCTYPE(C.c_void_p, C.c_size_t, C.c_int, C.c_void_p)
RELEASE_FN = C.CFUNCTYPE(None, C.c_void_p, C.c_int, C.c_void_p)

_lib = None


def load(path: str | None = None):
    """Load libibfs.so and declare every entry point of include/ibfs.h."""
    global _lib
    if _lib is not None and path is None:
        return _lib
    p = path or SO
    if not os.path.exists(p):
        raise ImportError(f"libibfs.so not built at {p}: run __graft_entry__.build() "
                          "(there is no CPU fallback)")
    lib = C.CDLL(p)
    P = C.c_void_p
    lib.ibfs_version.restype = C.c_int
    lib.ibfs_version.argtypes = []
    lib.ibfs_last_error.restype = C.c_char_p
    lib.ibfs_last_error.argtypes = []
    lib.ibfs_load_csr.restype = C.c_int
    lib.ibfs_load_csr.argtypes = [C.c_int, C.c_uint32, C.c_uint64, P, P, P, P, C.POINTER(P)]
    lib.ibfs_load_edges.restype = C.c_int
    lib.ibfs_load_edges.argtypes = [C.c_int, C.c_uint32, C.c_uint64, P, P, C.c_int, C.POINTER(P)]
    lib.ibfs_graph_info.restype = C.c_int
    lib.ibfs_graph_info.argtypes = [P, C.POINTER(C.c_uint32), C.POINTER(C.c_uint64),
                                    C.POINTER(C.c_uint32), C.POINTER(C.c_int)]
    lib.ibfs_graph_sort_rows.restype = C.c_int
    lib.ibfs_graph_sort_rows.argtypes = [P, C.c_int]
    lib.ibfs_graph_export_csr.restype = C.c_int
    lib.ibfs_graph_export_csr.argtypes = [P, P, P]
    lib.ibfs_free.restype = None
    lib.ibfs_free.argtypes = [P]
    lib.ibfs_plan_params_default.restype = None
    lib.ibfs_plan_params_default.argtypes = [C.POINTER(PlanParams)]
    lib.ibfs_plan_groups.restype = C.c_int
    lib.ibfs_plan_groups.argtypes = [P, P, C.c_uint32, C.c_uint32, C.POINTER(PlanParams), P,
                                     C.POINTER(C.c_uint32)]
    lib.ibfs_run.restype = C.c_int
    lib.ibfs_run.argtypes = [P, P, C.c_uint32, C.c_uint32, P]
    lib.ibfs_run_opts_default.restype = None
    lib.ibfs_run_opts_default.argtypes = [C.POINTER(RunOpts)]
    lib.ibfs_run_ex.restype = C.c_int
    lib.ibfs_run_ex.argtypes = [P, P, C.c_uint32, C.c_uint32, P, C.POINTER(RunOpts), C.POINTER(Stats)]
    lib.ibfs_set_allocator.restype = C.c_int
    lib.ibfs_set_allocator.argtypes = [P, P, P]
    if path is None:
        _lib = lib
    return lib


class IbfsError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"ibfs error {code}: {msg}")
        self.code = code


def check(rc: int) -> None:
    if rc != IBFS_OK:
        msg = load().ibfs_last_error()
        raise IbfsError(rc, msg.decode() if msg else "")
