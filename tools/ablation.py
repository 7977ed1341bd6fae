"""Ablation ladder on a synthetic config (Fig. 15 P:L959-L987,
Fig. 20): the same sources traversed
  (1) sequentially -- one BFS instance per call (W = 32 word, one active bit), the
      "sequential concurrent BFS" of P:L217 on this library's kernels;
  (2) joint traversal with the byte-per-instance Joint Status Array (§4, engine "joint"),
      random grouping;
  (3) bitwise joint traversal, random grouping (plan mode "random");
  (4) bitwise joint traversal + outdegree-based GroupBy (§5.2).
GTEPS = sum of m_s / device time (CUDA events).  usage: ablation.py [config] [n_sources]"""
import os
import sys
import json

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import ibfs_gen
import paper_conf_sigmod_liuhh16_b200 as P

name = sys.argv[1] if len(sys.argv) > 1 else "c2"
nsrc = int(sys.argv[2]) if len(sys.argv) > 2 else 512
cfg = ibfs_gen.CONFIGS[name]
el = cfg.edges(threads=os.cpu_count())
g = P.Graph.from_edgelist(el)
src = ibfs_gen.sample_sources(el, nsrc, cfg.source_seed) if cfg.n_sources else ibfs_gen.all_vertices(el.nv)[:nsrc]
W = 128
out = torch.empty((max(len(src), W), g.nv), dtype=torch.int8, device="cuda")
stream = torch.cuda.current_stream()


def timed(fn):
    fn()  # warm-up
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    edges = fn()
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    return {"ms": round(ms, 3), "edges": int(edges), "gteps": round(edges / (ms * 1e-3) / 1e9, 2)}


def sequential():
    k = min(len(src), 64)  # bounded sample; GTEPS is a rate
    e = 0
    for s in src[:k]:
        _, st = g.run(np.array([s], dtype=np.uint32), 32, out=out[:1], stream=stream)
        e += st.edges_traversed
    return e


def joint(mode, engine="bitwise"):
    perm = g.plan(src, W, mode=mode)
    s = src[perm]

    def f():
        _, st = g.run(s, W, out=out[: len(s)], stream=stream, engine=engine)
        return st.edges_traversed
    return f


res = {"config": cfg.name, "sources": int(len(src)),
       "sequential (1 instance per call, 64-source sample)": timed(sequential),
       "joint byte-JSA (§4), random grouping": timed(joint("random", "joint")),
       "bitwise, random grouping": timed(joint("random")),
       "bitwise + GroupBy": timed(joint("groupby"))}
print(json.dumps(res, indent=1))
