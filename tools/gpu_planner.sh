#!/bin/bash
set -u
OUT=gpurun_out/${1:-r01k}; mkdir -p "$OUT"
timeout 900 python -m pytest tests -m gpu -x -q -k "planner" > "$OUT/pytest_planner.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_planner.log"
timeout 600 python bench.py --config c5 --plan-hops 2 --no-e2e --no-cpu-baseline --json-out "$OUT/bench_c5_hops2.json" > "$OUT/bench_c5_hops2.log" 2>&1
timeout 600 python bench.py --config c3 --plan-hops 2 --no-e2e --no-cpu-baseline --json-out "$OUT/bench_c3_hops2.json" > "$OUT/bench_c3_hops2.log" 2>&1
timeout 600 python bench.py --config c4 --plan-hops 2 --no-e2e --no-cpu-baseline --json-out "$OUT/bench_c4_hops2.json" > "$OUT/bench_c4_hops2.log" 2>&1
PROBE_HOPS=2 PROBE_GROUPS=$(seq -s, 0 31) timeout 600 python tools/probe.py c5 1 > "$OUT/probe_c5_hops2.txt" 2>&1
echo done > "$OUT/DONE"
