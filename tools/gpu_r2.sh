#!/bin/bash
# new-feature GPU tests + per-group probe of c5 + ncu full captures (level, depth)
set -u
OUT=gpurun_out/${1:-r01c}; mkdir -p "$OUT"
timeout 900 python -m pytest tests -m gpu -x -q -k "khop or directed or planner" > "$OUT/pytest_new.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_new.log"
PROBE_GROUPS=$(seq -s, 0 31) timeout 600 python tools/probe.py c5 1 > "$OUT/probe_c5_all.txt" 2>&1
echo "rc=$?" >> "$OUT/probe_c5_all.txt"
B="python bench.py --config c5 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --groups-per-rank 4"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:level_kernel -s 1 -c 3 -o "$OUT/level_kernel_c5" $B > "$OUT/ncu_level.log" 2>&1
echo "rc=$?" >> "$OUT/ncu_level.log"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:depth_kernel -s 0 -c 1 -o "$OUT/depth_kernel_c5" $B > "$OUT/ncu_depth.log" 2>&1
echo "rc=$?" >> "$OUT/ncu_depth.log"
echo done > "$OUT/DONE"
