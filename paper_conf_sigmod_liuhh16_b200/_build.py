"""In-tree build of libibfs.so for sm_100a (nvcc cross-compiles without a GPU)."""
from __future__ import annotations

import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
INCLUDE = os.path.join(os.path.dirname(HERE), "include")
SO = os.path.join(HERE, "libibfs.so")
SOURCES = ["ibfs.cu", "plan.cpp"]
import glob as _glob


def _headers():
    """Every header the sources include (csrc/*.cuh, csrc/*.h), so an edit to any of
    them rebuilds the library."""
    return sorted(os.path.basename(p) for p in _glob.glob(os.path.join(CSRC, "*.cuh")) +
                  _glob.glob(os.path.join(CSRC, "*.h")))

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC", "-shared",
]


def _stale() -> bool:
    if not os.path.exists(SO):
        return True
    t = os.path.getmtime(SO)
    deps = [os.path.join(CSRC, f) for f in SOURCES + _headers()] + [os.path.join(INCLUDE, "ibfs.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    if force or _stale():
        nvcc = os.environ.get("NVCC", "nvcc")
        cmd = [nvcc, *NVCC_FLAGS, "-o", SO] + [os.path.join(CSRC, f) for f in SOURCES]
        if verbose:
            cmd.insert(1, "-Xptxas=-v")
        subprocess.check_call(cmd, cwd=CSRC)
    return SO


def build_variant(name: str, defines: dict) -> str:
    """A/B build (tuning experiments): build/libibfs_<name>.so with -D overrides of the
    compile-time knobs (IBFS_EXPAND_MINB, IBFS_BU_U); select it with IBFS_LIB=<path>."""
    out_dir = os.path.join(os.path.dirname(HERE), "build")
    os.makedirs(out_dir, exist_ok=True)
    out = os.path.join(out_dir, f"libibfs_{name}.so")
    nvcc = os.environ.get("NVCC", "nvcc")
    cmd = [nvcc, *NVCC_FLAGS, *[f"-D{k}={v}" for k, v in defines.items()], "-o", out] + \
        [os.path.join(CSRC, f) for f in SOURCES]
    subprocess.check_call(cmd, cwd=CSRC)
    return out
