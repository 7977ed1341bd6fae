"""Reader for tests/golden/*.txt fixtures (paper-printed values with citations)."""
from __future__ import annotations

import os

import numpy as np

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def read_fig1():
    rows, fields = [], {}
    with open(os.path.join(GOLDEN, "fig1.txt")) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            key, val = line.split(":", 1)
            if key == "row":
                rows.append([int(x) for x in val.split()])
            else:
                fields[key] = val.split()
    cols = [int(x) for x in fields["columns"]]
    sources = [int(x) for x in fields["sources"]]
    edges = [tuple(int(y) for y in e.split("-")) for e in fields["edges"]]
    nv = 9
    depths = np.full((len(rows), nv), -2, dtype=np.int8)
    for r, row in enumerate(rows):
        for c, val in zip(cols, row):
            depths[r, c] = val - 1  # paper depth (source = 1) -> ours (source = 0), reading #1
    return {
        "nv": nv,
        "sources": np.asarray(sources, dtype=np.uint32),
        "edges": edges,
        "depths": depths,
        "jfq_after_level1": [int(x) for x in fields["jfq_after_level1"]],
        "bsa_v5_v8": fields["bsa_after_level2_v5_v8"],
    }
