#!/bin/bash
# ncu --set full captures of the heavy launches of one config + a per-level probe.
# usage: bash tools/gpu_prof.sh TAG CONFIG [kernel:skip:count ...]
set -u
TAG=$1; CFG=${2:-c5}; shift 2 || true
SPECS=${*:-"level_kernel:1:3 depth_kernel:0:1"}
OUT=gpurun_out/$TAG; mkdir -p "$OUT"
B="python bench.py --config $CFG --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
timeout 600 python tools/probe.py $CFG 1 > "$OUT/probe_$CFG.txt" 2>&1
for spec in $SPECS; do
  IFS=: read k s c <<< "$spec"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s $s -c $c \
    -o "$OUT/${k}_$CFG" $B > "$OUT/ncu_${k}_$CFG.log" 2>&1
  echo "rc=$?" >> "$OUT/ncu_${k}_$CFG.log"
done
echo done > "$OUT/DONE"
