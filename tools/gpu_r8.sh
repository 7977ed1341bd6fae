#!/bin/bash
set -u
OUT=gpurun_out/${1:-r01i}; mkdir -p "$OUT"
timeout 1500 python -m pytest tests -m gpu -x -q > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
for i in 1 2; do for c in c5 c4 c3; do
  timeout 600 python bench.py --config $c --no-e2e --no-cpu-baseline --json-out "$OUT/bench_${c}_$i.json" > "$OUT/bench_${c}_$i.log" 2>&1
done; done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -k regex:'level_kernel|depth_kernel|init_|ms_kernel|iso_fix' --csv --log-file "$OUT/launches_c5.csv" \
  python bench.py --config c5 --steps 8 --warmup 0 --no-e2e --no-cpu-baseline > "$OUT/launches_c5.log" 2>&1
echo "rc=$?" >> "$OUT/launches_c5.log"
echo done > "$OUT/DONE"
