#!/bin/bash
# parity + bench lines (no e2e / cpu baseline) after a change
set -u
OUT=gpurun_out/${1:-check}; shift; mkdir -p "$OUT"
timeout 1500 python -m pytest tests -m gpu -x -q > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
for c in ${CFGS:-c5 c4 c3}; do
  timeout 600 python bench.py --config $c --no-e2e --no-cpu-baseline --json-out "$OUT/bench_$c.json" > "$OUT/bench_$c.log" 2>&1
done
echo done > "$OUT/DONE"
