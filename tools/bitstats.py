"""Per-instance frontier statistics of one group from its depth rows (diagnostics).
usage: PROBE_GROUPS=0,31 python tools/bitstats.py c5"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import ibfs_gen
import paper_conf_sigmod_liuhh16_b200 as P

name = sys.argv[1] if len(sys.argv) > 1 else "c5"
cfg = ibfs_gen.CONFIGS[name]
el = cfg.edges(threads=os.cpu_count())
g = P.Graph.from_edgelist(el)
off = g.export_csr()[0]
deg = torch.from_numpy(np.diff(off).astype(np.int64)).cuda()
ne = int(off[-1])
src = cfg.sources(el)
s = src[g.plan(src, 128)]
out = torch.empty((128, g.nv), dtype=torch.int8, device="cuda")
for g0 in [int(x) for x in os.environ.get("PROBE_GROUPS", "0").split(",")]:
    ss = s[g0 * 128:(g0 + 1) * 128]
    _, st = g.run(ss, 128, out=out[: len(ss)], timing=True, split="off")
    torch.cuda.synchronize()
    print(f"== {name} group {g0}: sources deg min/med/max {np.diff(off)[ss].min()}/{int(np.median(np.diff(off)[ss]))}/{np.diff(off)[ss].max()}")
    cum = torch.zeros(128, dtype=torch.float64, device="cuda")
    for lvl in range(st.max_levels + 1):
        nf = torch.zeros(128, dtype=torch.float64, device="cuda")
        mf = torch.zeros(128, dtype=torch.float64, device="cuda")
        for r0 in range(0, 128, 4):
            m = (out[r0:r0 + 4] == lvl)
            nf[r0:r0 + 4] = m.sum(1).double()
            mf[r0:r0 + 4] = (m.to(torch.int64) * deg[None, :]).sum(1).double()
        cum += mf
        mu = (ne - cum).clamp(min=1.0)
        r = mf / mu
        L = st.per_level[lvl] if lvl < len(st.per_level) else None
        dirs = ("T" if L and L["td_groups"] else "B") if L else "-"
        qs = lambda x: "/".join(f"{v:.2g}" for v in torch.quantile(x, torch.tensor([0.0, 0.1, 0.5, 0.9, 1.0], dtype=torch.float64, device=x.device)).tolist())
        nxt = f"next L{lvl+1} {dirs} insp {L['inspected']:.3g} ms {L['expand_ms']:.2f}" if L else ""
        print(f" depth {lvl}: n_f q0/10/50/90/100 {qs(nf)}  m_f/ne {qs(mf / ne)}  #m_f<ne/1024 {(mf < ne / 1024).sum().item()}  r=m_f/m_u {qs(r)} #r<1/16 {(r < 1/16).sum().item()} #r<1/64 {(r < 1/64).sum().item()}  {nxt}")
