"""Per-call timing breakdown of Graph.run on a config (diagnostics, not the bench)."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import ibfs_gen
import paper_conf_sigmod_liuhh16_b200 as P

name = sys.argv[1] if len(sys.argv) > 1 else "c5"
G = int(sys.argv[2]) if len(sys.argv) > 2 else 1
extra = dict(a.split("=") for a in sys.argv[3:])
cfg = ibfs_gen.CONFIGS[name]
el = cfg.edges(threads=os.cpu_count())
g = P.Graph.from_edgelist(el)
src = cfg.sources(el)
s = src[g.plan(src, 128, hops=int(os.environ.get("PROBE_HOPS", 1)))]
out = torch.empty((G * 128, g.nv), dtype=torch.int8, device="cuda")
kw = {}
for k, v in extra.items():
    kw[k] = float(v) if k in ("alpha", "beta") else (int(v) if v.isdigit() else v)
iters = int(os.environ.get("PROBE_ITERS", 4))
g0s = [int(x) for x in os.environ.get("PROBE_GROUPS", "").split(",") if x]
for it in range(len(g0s) or iters):
    g0 = g0s[it] if g0s else it * G
    ss = s[(g0 * 128) % len(s):][: G * 128]
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    _, st = g.run(ss, 128, out=out[: len(ss)], timing=True, **kw)
    t1 = time.perf_counter()
    print(f"{name} it{it} g0={g0}: wall {1e3*(t1-t0):.1f} ms traverse {st.traverse_ms:.1f} finalize {st.finalize_ms:.1f} "
          f"level {st.level_ms:.1f} (expand {st.expand_ms:.1f} commit {st.commit_ms:.1f}) depth {st.depth_ms:.1f} init {st.init_ms:.1f} "
          f"levels {st.max_levels} td {st.levels_td} bu {st.levels_bu} gteps {st.gteps:.0f} launches {st.n_launches}")
    for i, L in enumerate(st.per_level):
        print("   L%d td%d bu%d jfq_td %d jfq_bu %d insp %d new %d  exp %.2f ms com %.2f ms" % (i + 1, L["td_groups"], L["bu_groups"], L["jfq_td"], L["jfq_bu"], L["inspected"], L["new_pairs"], L["expand_ms"], L["commit_ms"]))
