#!/bin/bash
# A/B of whole library builds (IBFS_LIB), interleaved twice, plus a launch list of the depth flush kernels
set -u
OUT=gpurun_out/${1:-ab2}; shift; mkdir -p "$OUT"
CFGS=${CFGS:-c5 c3}
for rep in 1 2; do
for v in "$@"; do
  lib=""; [ "$v" != "default" ] && lib="build/libibfs_$v.so"
  for c in $CFGS; do
    IBFS_LIB=$lib timeout 600 python bench.py --config $c --no-e2e --no-cpu-baseline --json-out "$OUT/bench_${c}_${v}_$rep.json" > "$OUT/bench_${c}_${v}_$rep.log" 2>&1
  done
done
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'depth_kernel|late_fix|ms_kernel|iso_fix' --csv --log-file "$OUT/launches_depth_c5.csv" \
  python bench.py --config c5 --steps 2 --warmup 0 --no-e2e --no-cpu-baseline > "$OUT/launches.log" 2>&1
echo done > "$OUT/DONE"
