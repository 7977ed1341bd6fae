"""Instructions executed per CUDA source line (diagnostics). usage: ncu_inst.py rep [skip] [top]"""
import csv, io, subprocess, sys
from collections import defaultdict
rep = sys.argv[1]; skip = sys.argv[2] if len(sys.argv) > 2 else "0"; top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "--launch-skip", skip, "--launch-count", "1"], capture_output=True, text=True).stdout
rd = list(csv.reader(io.StringIO(out)))
hdr = None; cur = ""; agg = defaultdict(float); text = {}
for r in rd:
    if not r: continue
    if r[0] in ("File Name", "File Path"): cur = r[1].split("/")[-1]; continue
    if r[0] == "Line No": hdr = r; continue
    if hdr is None or not r[0].isdigit(): continue
    d = dict(zip(hdr, r))
    try: x = float(d.get("Instructions Executed", 0) or 0)
    except ValueError: continue
    key = (cur, int(r[0])); text[key] = r[1].strip(); agg[key] += x
tot = sum(agg.values())
print(f"total warp instructions {tot:.4g}")
for k, v in sorted(agg.items(), key=lambda kv: -kv[1])[:top]:
    print(f"{100*v/tot:5.1f}% {v:10.4g}  {k[0]}:{k[1]}  {text[k][:100]}")
