"""Per-source-line L2 sector requests and stall samples from an ncu report (diagnostics).
usage: ncu_lines.py report.ncu-rep [launch_skip] [top]"""
import csv, io, subprocess, sys
from collections import defaultdict
rep = sys.argv[1]; skip = sys.argv[2] if len(sys.argv) > 2 else "0"; top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "--launch-skip", skip, "--launch-count", "1"], capture_output=True, text=True).stdout
rd = list(csv.reader(io.StringIO(out)))
hdr = None; cur = ""; agg = defaultdict(lambda: [0.0, 0.0, 0.0]); text = {}
for r in rd:
    if not r: continue
    if r[0] == "File Path": cur = r[1].split("/")[-1]; continue
    if r[0] == "Line No": hdr = r; continue
    if hdr is None or not r[0].isdigit() or len(r) < len(hdr): continue
    d = dict(zip(hdr, r))
    # cuda rows: Line No, Source(cuda) ... ; we aggregate per cuda line
    key = (cur, int(r[0])); text[key] = r[1].strip()
    for i, c in enumerate(("L2 Theoretical Sectors Global", "L2 Theoretical Sectors Global Ideal", "Warp Stall Sampling (All Samples)")):
        try: agg[key][i] += float(d.get(c, "0") or 0)
        except ValueError: pass
tot = sum(v[0] for v in agg.values()) or 1; tots = sum(v[2] for v in agg.values()) or 1
print(f"total L2 sectors {tot:.3e} ({tot*32/1e9:.2f} GB), stall samples {tots:.0f}")
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    print(f"{v[0]/tot*100:5.1f}% sect ({v[0]*32/1e9:6.3f} GB, ideal {v[1]*32/1e9:6.3f})  {v[2]/tots*100:5.1f}% stall  {k[0]}:{k[1]:<5} {text[k][:80]}")
