#!/bin/bash
# A/B: fused clean ring (consumer-side zero stores) and the relative split (IBFS_SPLIT_REL);
# per-level probe of c5; c5 golden chunks in the background
set -u
OUT=gpurun_out/${1:-r02p}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
GOLDEN_THREADS=${GOLDEN_THREADS:-12} source tools/box_golden.sh
B="timeout 900 python bench.py --no-e2e --no-cpu-baseline"
for c in c5 c3; do
  for fc in 1 0; do
    IBFS_FUSED_CLEAN=$fc $B --config $c --json-out "$OUT/bench_${c}_fc$fc.json" > "$OUT/bench_${c}_fc$fc.log" 2>&1
  done
  for sr in 8 32 128; do
    IBFS_SPLIT_REL=$sr $B --config $c --json-out "$OUT/bench_${c}_sr$sr.json" > "$OUT/bench_${c}_sr$sr.log" 2>&1
  done
done
for sr in 0 32; do
  IBFS_SPLIT_REL=$sr $B --config c4 --json-out "$OUT/bench_c4_sr$sr.json" > "$OUT/bench_c4_sr$sr.log" 2>&1
done
PROBE_HOPS=2 PROBE_ITERS=32 timeout 900 python tools/probe.py c5 > "$OUT/probe_c5.txt" 2>&1
sleep ${GOLDEN_EXTRA:-0}
kill $GOLDEN_PID 2>/dev/null
echo done > "$OUT/DONE"
