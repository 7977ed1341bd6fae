#!/usr/bin/env python
"""Config 2 as BASELINE.json words it: "Graph500 Kronecker scale 20, edgefactor 16, i=128
sources: GroupBy vs random grouping, top-down/bottom-up switch".

For W = 32 / 64 / 128 and planner GroupBy (hops 1 and 2) / random / identity, and direction
auto / TD-only: the Eq. 1 sharing degrees SD_TD and SD_BU (reading #23),
inspections, GTEPS (device time, best of 5 runs after a warm-up) and the per-level
direction of each group.  Writes a markdown report (default profiles/r02/c2_report.md).

    python tools/c2_report.py [--out profiles/r02/c2_report.md]
"""
from __future__ import annotations

import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import ibfs_gen  # noqa: E402
import paper_conf_sigmod_liuhh16_b200 as P  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r02", "c2_report.md"))
    ap.add_argument("--reps", type=int, default=5)
    a = ap.parse_args()
    import torch
    cfg = ibfs_gen.CONFIGS["c2"]
    el = cfg.edges()
    src = cfg.sources(el)
    g = P.Graph.from_edgelist(el)
    out = torch.empty((len(src), g.nv), dtype=torch.int8, device="cuda")
    lines = ["# Config 2: GroupBy vs random grouping, direction switch (B200)", "",
             f"Kronecker s20 ef16 (|V| = {g.nv:,}, CSR entries = {g.ne:,}), i = {len(src)} sources "
             "(seeded, deg > 0).  SD = sum_j |FQ_j| / |JFQ| per direction (Eq. 1, reading #23); "
             "GTEPS = sum_s m_s / device traversal time (best of %d runs); 'dirs' = per-level "
             "direction over the groups (T = all top-down, B = all bottom-up, M = mixed).  "
             "Written by tools/c2_report.py." % a.reps, "",
             "| W | groups | planner | direction | SD_TD | SD_BU | inspections | GTEPS | ms | dirs |",
             "|---|---|---|---|---|---|---|---|---|---|"]
    for W in (32, 64, 128):
        for plan, kw in (("GroupBy hops=1", dict(mode="groupby", hops=1)), ("GroupBy hops=2", dict(mode="groupby", hops=2)),
                         ("random", dict(mode="random", seed=3)), ("identity", dict(mode="identity"))):
            s = src[g.plan(src, W, **kw)]
            for direction in ("auto", "td"):
                best = None
                for _ in range(a.reps + 1):
                    _, st = g.run(s, W, out=out[: len(s)], direction=direction, timing=True, groups_in_flight=1)
                    torch.cuda.synchronize()
                    if best is None or st.traverse_ms < best.traverse_ms:
                        best = st
                st = best
                dirs = "".join("T" if x["td_groups"] and not x["bu_groups"] else ("B" if x["bu_groups"] and not x["td_groups"] else "M")
                               for x in st.per_level)
                lines.append(f"| {W} | {st.n_groups} | {plan} | {direction} | {st.sd_td:.2f} | {st.sd_bu:.2f} | "
                             f"{st.edges_inspected:,} | {st.gteps:,.0f} | {st.traverse_ms:.3f} | {dirs} |")
                print(lines[-1], flush=True)
    lines += ["", "Per-level 'dirs' is over all groups of the run: T = every group top-down, B = every group "
              "bottom-up, M = mixed.  Groups run one per launch (groups_in_flight = 1) so the GroupBy vs "
              "random comparison is per group, as in P:L1015."]
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out, "w") as f:
        f.write("\n".join(lines) + "\n")
    print("wrote", a.out)


if __name__ == "__main__":
    main()
