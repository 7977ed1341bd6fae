"""Stall-reason breakdown per CUDA source line (diagnostics). usage: ncu_stalls.py rep [skip] [top]"""
import csv, io, subprocess, sys
from collections import defaultdict
rep = sys.argv[1]; skip = sys.argv[2] if len(sys.argv) > 2 else "0"; top = int(sys.argv[3]) if len(sys.argv) > 3 else 12
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "--launch-skip", skip, "--launch-count", "1"], capture_output=True, text=True).stdout
rd = list(csv.reader(io.StringIO(out)))
hdr = None; cur = ""; agg = defaultdict(lambda: defaultdict(float)); text = {}
tot = defaultdict(float)
for r in rd:
    if not r: continue
    if r[0] == "File Path": cur = r[1].split("/")[-1]; continue
    if r[0] == "Line No": hdr = r; continue
    if hdr is None or not r[0].isdigit() or len(r) < len(hdr): continue
    d = dict(zip(hdr, r)); key = (cur, int(r[0])); text[key] = r[1].strip()
    for c in hdr:
        if c.startswith("stall_") and "Not Issued" not in c:
            try: x = float(d[c] or 0)
            except ValueError: continue
            agg[key][c] += x; tot[c] += x
T = sum(tot.values()) or 1
print("overall:", ", ".join(f"{k[6:]} {v/T*100:.1f}%" for k, v in sorted(tot.items(), key=lambda kv: -kv[1])[:8]))
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1].values()))[:top]:
    s = sum(v.values())
    print(f"{s/T*100:5.1f}% {k[0]}:{k[1]:<5} " + ", ".join(f"{c[6:]} {x/s*100:.0f}%" for c, x in sorted(v.items(), key=lambda kv: -kv[1])[:3]) + f"   | {text[k][:60]}")
