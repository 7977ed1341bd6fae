#!/bin/bash
# Copy a gpu_final.sh run (gpurun_out/TAG) into profiles/r01/final and regenerate the summaries.
set -eu
TAG=$1; SRC=gpurun_out/$TAG; DST=${2:-profiles/r01/final}
mkdir -p "$DST"
cp "$SRC"/bench_c5.json "$SRC"/bench_c4.json "$SRC"/bench_c3.json "$SRC"/bench_c5_3hop.json "$SRC"/bench_ref_c5.log \
   "$SRC"/pytest_gpu.log "$SRC"/smoke.log "$SRC"/info.txt "$DST"/
if [ -f "$SRC/launches_c5.csv" ]; then
  cp "$SRC/launches_c5.csv" "$DST/ncu_launches_c5.csv"
  python tools/ncu_launch_traffic.py "$DST/ncu_launches_c5.csv" c5 'level_kernel=level' 'depth_kernel=depth' \
    --json profiles/ncu_traffic.json > "$DST/launches_c5_summary.md"
  python - <<'PY'
import json
p = "profiles/ncu_traffic.json"; j = json.load(open(p))
for k in j.get("c5", {}).values():
    k["source"] = "profiles/r01/final/ncu_launches_c5.csv"
json.dump(j, open(p, "w"), indent=1)
PY
fi
python tools/ncu_summary.py full "$SRC/level_kernel_c5.ncu-rep" "$SRC/depth_kernel_c5.ncu-rep" > "$DST/ncu_full_c5.md"
for s in 0 1 2; do echo "### level_kernel, heavy launch $s (stall reasons by source line)"; echo '```'
  python tools/ncu_stalls.py "$SRC/level_kernel_c5.ncu-rep" $s 10; echo '```'; done > "$DST/ncu_level_stalls.md" 2>&1
(echo "### depth_kernel"; echo '```'; python tools/ncu_stalls.py "$SRC/depth_kernel_c5.ncu-rep" 0 10; echo '```') > "$DST/ncu_depth_stalls.md" 2>&1
echo collected "$SRC" into "$DST"
