"""Frontier statistics from depth rows -- TEST INFRASTRUCTURE ONLY.

Sharing degree, Eq. 1:
    SD_A = sum_k sum_j |FQ_j(k)|  /  sum_k |JFQ_A(k)|
with, in our level numbering (level l expands depth l-1 and discovers depth l; DESIGN.md
reading #20) and reading #23:
  * top-down level l:   FQ_j = {v : d_j(v) = l-1},  JFQ = union_j FQ_j
  * bottom-up level l:  FQ_j = {v : d_j(v) = -1 or d_j(v) >= l}, restricted to the
                        instances still active (some vertex at depth l-1), JFQ = union
                        (reading #24).
Everything is computed from plain depth rows of one group (int8 [w][nv]).
"""
from __future__ import annotations

import numpy as np


def level_counts(depths: np.ndarray, schedule) -> list[dict]:
    """Per-level (dir, sum_fq, jfq, new_pairs) for one group.

    depths: int8 [w][nv] rows of one group; schedule: list of 'T'/'B' per level 1..L
    (levels beyond the list are treated as 'T').  Levels run until no instance is
    active, i.e. L = max depth + 1 (the last level discovers nothing).
    """
    d = depths.astype(np.int16)
    w = d.shape[0]
    maxd = int(d.max(initial=-1))
    out = []
    for lvl in range(1, maxd + 2):
        dirc = schedule[lvl - 1] if lvl - 1 < len(schedule) else "T"
        active = (d == lvl - 1).any(axis=1)  # instance j discovered something at l-1
        if dirc == "T":
            fq = (d == lvl - 1)
        else:
            fq = ((d == -1) | (d >= lvl)) & active[:, None]
        out.append({
            "dir": dirc,
            "sum_fq": int(fq.sum()),
            "jfq": int(fq.any(axis=0).sum()),
            "new_pairs": int((d == lvl).sum()),
            "active": int(active.sum()) if w else 0,
        })
    return out


def sharing_degree(depths: np.ndarray, schedule=()) -> float:
    """Eq. 1 for one group (TD-only unless a schedule is given)."""
    lc = level_counts(depths, schedule)
    num = sum(x["sum_fq"] for x in lc)
    den = sum(x["jfq"] for x in lc)
    return num / den if den else 0.0


def m_s_from_depths(depths: np.ndarray, deg: np.ndarray) -> np.ndarray:
    """m_s = sum over reached v of deg(v) (reading #11)."""
    reached = depths >= 0
    return (reached.astype(np.uint64) * deg.astype(np.uint64)[None, :]).sum(axis=1).astype(np.uint64)
