#!/usr/bin/env python
"""Write oracle-computed goldens for the full-size parity tests -- calls only ``oracle/``.

    python tools/make_golden.py c3 c4 c5 [--threads T]

For each config: the seeded graph and sources from ``ibfs_gen`` (the shared input
generator), one textbook BFS per source in ``oracle/oracle.c`` (the
shortest-path definition of, depths in GPU memory P:L887), and per
source, keyed by source id in GENERATOR order (no planner involved):

    m_s     = sum over reached v of deg(v)                     (TEPS numerator)
    digest  = sum over reached v of splitmix64((v<<8)|(d+1))
    ecc     = max depth,  reached = number of reached vertices

-> ``tests/golden/<cfg>_ms_digest.npz`` (sources, m_s, digest, ecc, reached, plus the
graph's nv / tuple count / the generator recipe as a guard).  Nothing here comes from the
CUDA path.  Work is checkpointed per chunk under ``gpurun_out/golden_ckpt/`` so a long c5
run (about 8.8e12 neighbour visits) can resume.
"""
from __future__ import annotations

import argparse
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import ibfs_gen  # noqa: E402
import oracle  # noqa: E402

GOLDEN = os.path.join(ROOT, "tests", "golden")
CKPT = os.path.join(ROOT, "gpurun_out", "golden_ckpt")  # --ckpt overrides


def make(name: str, threads: int, chunk: int, reverse: bool = False, extra_ckpt=(),
         assemble_only: bool = False) -> str:
    cfg = ibfs_gen.CONFIGS[name]
    t0 = time.time()
    el = cfg.edges(threads=threads)
    src = cfg.sources(el)
    og = oracle.OracleGraph.from_edges(el)
    m_tuples = el.m
    del el
    print(f"[{name}] graph nv={og.nv} ne={og.ne} sources={len(src)} built in {time.time() - t0:.1f}s",
          flush=True)
    n = len(src)
    m_s = np.zeros(n, dtype=np.uint64)
    dig = np.zeros(n, dtype=np.uint64)
    ecc = np.zeros(n, dtype=np.int32)
    reached = np.zeros(n, dtype=np.uint64)
    os.makedirs(CKPT, exist_ok=True)
    starts = list(range(0, n, chunk))
    if reverse:
        starts = starts[::-1]
    missing = 0
    for lo in starts:
        hi = min(n, lo + chunk)
        got = False
        for d in [CKPT] + list(extra_ckpt):
            ck = os.path.join(d, f"{name}_{lo}_{hi}.npz")
            if os.path.exists(ck):
                z = np.load(ck)
                if np.array_equal(z["sources"], src[lo:hi]):
                    m_s[lo:hi], dig[lo:hi], ecc[lo:hi], reached[lo:hi] = z["m_s"], z["digest"], z["ecc"], z["reached"]
                    got = True
                    break
        if got:
            continue
        if assemble_only:
            missing += 1
            continue
        ck = os.path.join(CKPT, f"{name}_{lo}_{hi}.npz")
        t1 = time.time()
        r = og.bfs(src[lo:hi], want_depths=False, threads=threads)
        if r.status != 0:
            raise RuntimeError(f"oracle status {r.status} on {name} [{lo}, {hi})")
        m_s[lo:hi], dig[lo:hi], ecc[lo:hi], reached[lo:hi] = r.m_s, r.digest, r.ecc, r.reached
        np.savez(ck, sources=src[lo:hi], m_s=r.m_s, digest=r.digest, ecc=r.ecc, reached=r.reached)
        dt = time.time() - t1
        print(f"[{name}] sources [{lo}, {hi}) in {dt:.1f}s  ({float(r.m_s.sum()) / dt / 1e9:.3f} GTEPS)",
              flush=True)
    if missing:
        print(f"[{name}] {missing} chunks missing: no golden written", flush=True)
        return ""
    out = os.path.join(GOLDEN, f"{name}_ms_digest.npz")
    np.savez_compressed(
        out, sources=src, m_s=m_s, digest=dig, ecc=ecc, reached=reached,
        nv=np.uint64(og.nv), ne=np.uint64(og.ne), tuples=np.uint64(m_tuples),
        recipe=np.array(f"{cfg.name}; abc={cfg.abc}; graph_seed={cfg.graph_seed}; "
                        f"source_seed={cfg.source_seed}; oracle/oracle.c textbook BFS per source"))
    print(f"[{name}] wrote {out} in {time.time() - t0:.1f}s; sum m_s = {int(m_s.sum())}", flush=True)
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="+")
    ap.add_argument("--threads", type=int, default=os.cpu_count() or 1)
    ap.add_argument("--chunk", type=int, default=0, help="sources per checkpoint (0 = per config)")
    ap.add_argument("--ckpt", default=None, help="checkpoint directory (default gpurun_out/golden_ckpt)")
    ap.add_argument("--extra-ckpt", action="append", default=[], help="more checkpoint directories to read")
    ap.add_argument("--reverse", action="store_true", help="compute the chunks from the last one down")
    ap.add_argument("--assemble", action="store_true", help="only assemble existing chunks")
    a = ap.parse_args()
    if a.ckpt:
        global CKPT
        CKPT = os.path.abspath(a.ckpt)
    for name in a.configs:
        chunk = a.chunk or {"c5": 64, "c3": 128, "c4": 16384}.get(name, 1 << 30)
        make(name, a.threads, chunk, a.reverse, a.extra_ckpt, a.assemble)


if __name__ == "__main__":
    main()
