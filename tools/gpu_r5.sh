#!/bin/bash
set -u
OUT=gpurun_out/${1:-r01f}; mkdir -p "$OUT"
timeout 1500 python -m pytest tests -m gpu -x -q > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
PROBE_GROUPS=0,5,23,31 timeout 600 python tools/probe.py c5 1 > "$OUT/probe_c5.txt" 2>&1
for v in "c5:" "c5:--groups-in-flight 4" "c5:--split-div 16" "c5:--split-div 256" "c3:" "c4:"; do
  c=${v%%:*}; extra=${v#*:}; tag=$(echo "$c$extra" | tr -d ' -')
  timeout 600 python bench.py --config $c $extra --no-e2e --no-cpu-baseline --json-out "$OUT/bench_$tag.json" > "$OUT/bench_$tag.log" 2>&1
done
timeout 600 python tools/ablation.py c2 512 > "$OUT/ablation_c2.json" 2> "$OUT/ablation_c2.err"
echo done > "$OUT/DONE"
