#!/bin/bash
# split_div re-check at alpha = 3 (c5 / c3)
set -u
OUT=gpurun_out/${1:-r02ab}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
B="timeout 600 python bench.py --no-e2e --no-cpu-baseline --no-clocks"
for c in c5 c3; do
  for sd in 256 512 1024; do $B --config $c --split-div $sd --json-out "$OUT/bench_${c}_sd$sd.json" > "$OUT/bench_${c}_sd$sd.log" 2>&1; done
done
echo done > "$OUT/DONE"
