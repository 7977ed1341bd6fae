#!/bin/bash
# c5 launch-batch width A/B: 4 groups per step (default) vs 8 groups in one launch batch
set -u
OUT=gpurun_out/${1:-r02y}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
B="timeout 900 python bench.py --config c5 --no-e2e --no-cpu-baseline"
$B --json-out "$OUT/bench_c5_g4.json" > "$OUT/bench_c5_g4.log" 2>&1
$B --groups-per-rank 8 --groups-in-flight 8 --steps 4 --json-out "$OUT/bench_c5_g8.json" > "$OUT/bench_c5_g8.log" 2>&1
$B --groups-per-rank 8 --steps 4 --json-out "$OUT/bench_c5_g8x4.json" > "$OUT/bench_c5_g8x4.log" 2>&1
$B --groups-per-rank 2 --groups-in-flight 2 --steps 16 --json-out "$OUT/bench_c5_g2.json" > "$OUT/bench_c5_g2.log" 2>&1
echo done > "$OUT/DONE"
