#!/bin/bash
# alpha (TD -> BU switch) around 3 on c3 / c4 / c5
set -u
OUT=gpurun_out/${1:-r02aa}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
B="timeout 900 python bench.py --no-e2e --no-cpu-baseline --no-clocks"
for al in 2.5 3 3.5 4; do $B --config c4 --alpha $al --json-out "$OUT/bench_c4_a$al.json" > "$OUT/bench_c4_a$al.log" 2>&1; done
for al in 2.5 3.5; do $B --config c3 --alpha $al --json-out "$OUT/bench_c3_a$al.json" > "$OUT/bench_c3_a$al.log" 2>&1; done
for al in 2.5 3.5; do $B --config c5 --alpha $al --json-out "$OUT/bench_c5_a$al.json" > "$OUT/bench_c5_a$al.log" 2>&1; done
echo done > "$OUT/DONE"
