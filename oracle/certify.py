"""Complete BFS-depth certificate -- TEST INFRASTRUCTURE ONLY.

SURVEY.md Appendix C, C4: a row d is the BFS depth row of source s on an undirected
graph iff
  (o)   every d(v) in {-1, 0, 1, 2, ...}
  (i)   d(s) = 0
  (ii)  for every edge {u, v}: d(u) = -1 <=> d(v) = -1, otherwise |d(u) - d(v)| <= 1
  (iii) every v != s with d(v) >= 0 has d(v) >= 1 and a neighbour u with d(u) = d(v) - 1.
(iii) + following predecessors gives dist <= d; (ii) along a shortest path gives
d <= dist; an unreachable v with d(v) >= 0 would contradict (iii).  North_star's
invariants (source depth 0, |d(u)-d(v)| <= 1 across every edge, unreachable = -1) are
(i)-(ii).  This checks ANY output at any size, including sampled GPU rows.
"""
from __future__ import annotations

import numpy as np


def certify_row(off: np.ndarray, adj: np.ndarray, s: int, d: np.ndarray) -> str | None:
    """None if d is the exact BFS depth row from s, else a reason string."""
    d = np.asarray(d).astype(np.int32)
    nv = d.shape[0]
    if (d < -1).any():
        return "(o) value < -1"
    if d[s] != 0:
        return "(i) d(s) != 0"
    deg = np.diff(off.astype(np.int64))
    src = np.repeat(np.arange(nv, dtype=np.int64), deg)
    du = d[src]
    dv = d[adj.astype(np.int64)]
    if ((du == -1) != (dv == -1)).any():
        return "(ii) reachability differs across an edge"
    both = (du >= 0) & (dv >= 0)
    if (np.abs(du - dv)[both] > 1).any():
        return "(ii) |d(u)-d(v)| > 1 across an edge"
    zero = np.flatnonzero(d == 0)
    if zero.shape[0] != 1 or zero[0] != s:
        return "(iii) a vertex other than s has depth 0"
    has_pred = np.zeros(nv, dtype=bool)
    pred_edge = (du >= 0) & (dv == du - 1)
    has_pred[src[pred_edge]] = True
    need = (d >= 1)
    if (need & ~has_pred).any():
        return "(iii) a reached vertex has no neighbour one level closer"
    return None


def certify_rows(off, adj, sources, depths) -> list[tuple[int, str]]:
    bad = []
    for r, s in enumerate(np.asarray(sources)):
        why = certify_row(off, adj, int(s), depths[r])
        if why:
            bad.append((r, why))
    return bad
