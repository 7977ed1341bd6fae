#!/bin/bash
# ncu --set full captures of the c5 level kernel (levels 2-5 of the first batch) and depth kernel
set -u
OUT=gpurun_out/${1:-r02u}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
B="python bench.py --config c5 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-clocks"
for spec in level_kernel:1:4 depth_tma_kernel:0:1 ms_kernel:0:1; do
  IFS=: read k s c <<< "$spec"
  timeout 1500 ncu --set full --clock-control none --import-source on -k regex:$k -s $s -c $c \
    -o "$OUT/full_${k}_c5" $B > "$OUT/full_${k}_c5.log" 2>&1
  echo "rc=$?" >> "$OUT/full_${k}_c5.log"
done
echo done > "$OUT/DONE"
