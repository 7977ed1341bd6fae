"""CPU checks of the C-ABI boundary: the library builds, loads, exports every symbol
include/ibfs.h declares, the ctypes mirrors match the C struct layouts, and argument
validation fails the documented way (no compute calls without a GPU)."""
from __future__ import annotations

import ctypes as C
import os
import re
import subprocess

import numpy as np
import pytest

import paper_conf_sigmod_liuhh16_b200 as P
from paper_conf_sigmod_liuhh16_b200 import _lib
from conftest import ROOT, gpu_available

HEADER = os.path.join(ROOT, "include", "ibfs.h")


@pytest.fixture(scope="module")
def lib():
    P.build()
    return _lib.load()


def declared_functions():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(ibfs_[a-z_]+)\s*\(", text)))


def test_exports_every_declared_symbol(lib):
    names = declared_functions()
    assert len(names) >= 13
    assert set(names) == set(_lib.EXPORTS)
    out = subprocess.check_output(["nm", "-D", "--defined-only", _lib.SO]).decode()
    exported = set(re.findall(r" T (ibfs_\w+)", out))
    missing = [n for n in names if n not in exported]
    assert not missing, missing
    for n in names:
        assert hasattr(lib, n)


def test_struct_layouts_match_c(tmp_path):
    src = tmp_path / "layout.c"
    src.write_text(r'''
#include <stdio.h>
#include <stddef.h>
#include "ibfs.h"
int main(void) {
  printf("%zu %zu %zu %zu\n", sizeof(ibfs_plan_params), sizeof(ibfs_run_opts),
         sizeof(ibfs_level_stats), sizeof(ibfs_stats));
  printf("%zu %zu %zu %zu\n", offsetof(ibfs_plan_params, seed), offsetof(ibfs_run_opts, cuda_stream),
         offsetof(ibfs_stats, per_source_m), offsetof(ibfs_stats, per_level));
  return 0;
}
''')
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), "-o", str(exe), str(src)])
    a, b = subprocess.check_output([str(exe)]).decode().split("\n")[:2]
    sizes = [int(x) for x in a.split()]
    offs = [int(x) for x in b.split()]
    assert sizes == [C.sizeof(_lib.PlanParams), C.sizeof(_lib.RunOpts), C.sizeof(_lib.LevelStats),
                     C.sizeof(_lib.Stats)]
    assert offs == [_lib.PlanParams.seed.offset, _lib.RunOpts.cuda_stream.offset,
                    _lib.Stats.per_source_m.offset, _lib.Stats.per_level.offset]


def test_defaults(lib):
    pp = _lib.PlanParams()
    lib.ibfs_plan_params_default(C.byref(pp))
    assert (pp.mode, pp.q, pp.n_p, list(pp.p)[:4], pp.hops) == (0, 128, 4, [4, 16, 64, 128], 1)
    o = _lib.RunOpts()
    lib.ibfs_run_opts_default(C.byref(o))
    assert o.direction == 0 and o.alpha > 0 and o.beta > 0
    assert lib.ibfs_version() >= 10000


def test_validation_before_device_work(lib):
    h = C.c_void_p()
    off = np.array([0, 1, 2], dtype=np.uint64)
    adj = np.array([1, 0], dtype=np.uint32)
    assert lib.ibfs_load_csr(0, 2, 2, off.ctypes.data, adj.ctypes.data, None, None, None) == _lib.IBFS_E_INVALID
    assert lib.ibfs_load_csr(0, 0, 0, off.ctypes.data, None, None, None, C.byref(h)) == _lib.IBFS_E_INVALID
    # directed: the in-edge CSR comes as a pair
    assert lib.ibfs_load_csr(0, 2, 2, off.ctypes.data, adj.ctypes.data, off.ctypes.data, None,
                             C.byref(h)) == _lib.IBFS_E_INVALID
    assert lib.ibfs_load_edges(0, 2, 1, None, None, 0, C.byref(h)) == _lib.IBFS_E_INVALID
    assert lib.ibfs_load_edges(0, 2, 1, None, None, 1, C.byref(h)) == _lib.IBFS_E_INVALID
    src = np.zeros(4, dtype=np.uint32)
    assert lib.ibfs_run(None, src.ctypes.data, 4, 64, None) == _lib.IBFS_E_INVALID
    assert lib.ibfs_run_ex(None, src.ctypes.data, 4, 64, None, None, None) == _lib.IBFS_E_INVALID
    assert lib.ibfs_plan_groups(None, src.ctypes.data, 4, 64, None, src.ctypes.data, None) == _lib.IBFS_E_INVALID
    assert lib.ibfs_set_allocator(C.c_void_p(1), None, None) == _lib.IBFS_E_INVALID
    assert lib.ibfs_last_error()  # message of the last failure on this thread
    lib.ibfs_free(None)  # NULL-safe


@pytest.mark.skipif(gpu_available(), reason="checks the no-GPU behaviour")
def test_no_cpu_fallback_without_gpu(lib):
    h = C.c_void_p()
    off = np.array([0, 1, 2], dtype=np.uint64)
    adj = np.array([1, 0], dtype=np.uint32)
    rc = lib.ibfs_load_csr(0, 2, 2, off.ctypes.data, adj.ctypes.data, None, None, C.byref(h))
    assert rc == _lib.IBFS_E_CUDA
    assert b"no CUDA device" in lib.ibfs_last_error()
    with pytest.raises(_lib.IbfsError):
        P.Graph.from_csr(off, adj)


def test_product_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_sigmod_liuhh16_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".cpp", ".h")):
                text = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"\boracle\b\s*(import|\.)|import\s+oracle|from\s+oracle", text), f
                assert "liboracle" not in text, f
