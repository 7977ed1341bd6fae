"""Top CUDA source lines by warp-stall samples from an ncu report (diagnostics).
usage: ncu_hot.py report.ncu-rep [launch_skip] [top]"""
import csv, io, subprocess, sys
from collections import defaultdict
rep = sys.argv[1]
skip = sys.argv[2] if len(sys.argv) > 2 else "0"
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "--launch-skip", skip, "--launch-count", "1"], capture_output=True, text=True).stdout
rd = list(csv.reader(io.StringIO(out)))
agg = defaultdict(float)
text = {}
col = None
cur_file = ""
for r in rd:
    if not r:
        continue
    if r[0] == "File Path":
        cur_file = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        col = r.index("Warp Stall Sampling (All Samples)")
        continue
    if col is None or len(r) <= col or not r[0].isdigit():
        continue
    try:
        x = float(r[col])
    except ValueError:
        continue
    key = (cur_file, int(r[0]))
    agg[key] += x
    text[key] = r[1].strip()
tot = sum(agg.values())
print("total samples", tot)
for k, v in sorted(agg.items(), key=lambda kv: -kv[1])[:top]:
    print(f"{v / tot * 100:5.1f}%  {k[0]}:{k[1]:<5} {text[k][:100]}")
