#!/bin/bash
set -u
OUT=gpurun_out/${1:-r01h}; mkdir -p "$OUT"
timeout 900 python -m pytest tests -m gpu -x -q -k "joint" > "$OUT/pytest_joint.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_joint.log"
for i in 1 2; do
  for c in "" "--no-clocks"; do
    tag=c4$(echo "$c" | tr -d ' -')_$i
    timeout 600 python bench.py --config c4 $c --no-e2e --no-cpu-baseline --json-out "$OUT/bench_$tag.json" > "$OUT/bench_$tag.log" 2>&1
  done
done
PROBE_GROUPS=0,100,200,1000 timeout 600 python tools/probe.py c4 64 > "$OUT/probe_c4.txt" 2>&1
timeout 900 python tools/ablation.py c2 512 > "$OUT/ablation_c2.json" 2> "$OUT/ablation_c2.err"
timeout 900 python tools/ablation.py c4 2048 > "$OUT/ablation_c4.json" 2> "$OUT/ablation_c4.err"
echo done > "$OUT/DONE"
