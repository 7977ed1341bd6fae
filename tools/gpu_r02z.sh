#!/bin/bash
# direction-rule re-check after the round-2 kernels: alpha (TD -> BU) and beta (BU -> TD) on c5 / c3
set -u
OUT=gpurun_out/${1:-r02z}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
B="timeout 900 python bench.py --no-e2e --no-cpu-baseline --no-clocks"
for c in c5 c3; do
  for al in 3 6; do $B --config $c --alpha $al --json-out "$OUT/bench_${c}_a$al.json" > "$OUT/bench_${c}_a$al.log" 2>&1; done
  for be in 12 48; do $B --config $c --beta $be --json-out "$OUT/bench_${c}_b$be.json" > "$OUT/bench_${c}_b$be.log" 2>&1; done
  $B --config $c --json-out "$OUT/bench_${c}_base.json" > "$OUT/bench_${c}_base.log" 2>&1
done
echo done > "$OUT/DONE"
