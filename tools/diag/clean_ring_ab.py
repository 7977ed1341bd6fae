"""Diagnostic: per-source digests of one config under the current IBFS_CLEAN_RING /
IBFS_FUSED_CLEAN setting (run once per setting in separate processes; compare the .npz)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import ibfs_gen
import paper_conf_sigmod_liuhh16_b200 as P

name, out = sys.argv[1], sys.argv[2]
ngroups = int(sys.argv[3]) if len(sys.argv) > 3 else 8
cfg = ibfs_gen.CONFIGS[name]
el = cfg.edges(threads=os.cpu_count())
g = P.Graph.from_edgelist(el)
src = cfg.sources(el)
s = src[g.plan(src, 128, hops=2)][: ngroups * 128]
rows = torch.empty((len(s), g.nv), dtype=torch.int8, device="cuda")
res = {}
for rep in range(2):
    _, st = g.run(s, 128, out=rows, want_digest=True)
    torch.cuda.synchronize()
    res[f"d{rep}"] = st.per_source_digest.copy()
    res[f"m{rep}"] = st.per_source_m.copy()
# per-level depth histogram of row 0 and a few rows, for locating a difference
res["hist"] = np.stack([np.bincount(rows[i].cpu().numpy().astype(np.int16) + 1, minlength=130) for i in range(0, len(s), 64)])
np.savez(out, sources=s, **res)
print(name, os.environ.get("IBFS_CLEAN_RING"), os.environ.get("IBFS_FUSED_CLEAN"), "digest[0..3]", res["d0"][:3],
      "rep-equal", bool(np.array_equal(res["d0"], res["d1"])))
