#!/bin/bash
# A/B of compile-time knobs: bench lines per variant library (IBFS_LIB) on the given configs
set -u
OUT=gpurun_out/${1:-ab}; shift; mkdir -p "$OUT"
CFGS=${CFGS:-c5}
for v in "$@"; do
  lib=""; [ "$v" != "default" ] && lib="build/libibfs_$v.so"
  for c in $CFGS; do
    IBFS_LIB=$lib timeout 600 python bench.py --config $c --no-e2e --no-cpu-baseline --json-out "$OUT/bench_${c}_$v.json" > "$OUT/bench_${c}_$v.log" 2>&1
  done
done
echo done > "$OUT/DONE"
