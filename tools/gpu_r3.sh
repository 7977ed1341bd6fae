#!/bin/bash
# GPU tests + c5 probe + bench + ncu of the depth kernel
set -u
OUT=gpurun_out/${1:-r01d}; mkdir -p "$OUT"
timeout 1500 python -m pytest tests -m gpu -x -q > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
PROBE_GROUPS=0,5,23,31 timeout 600 python tools/probe.py c5 1 > "$OUT/probe_c5.txt" 2>&1
timeout 900 python bench.py --config c5 --json-out "$OUT/bench_c5.json" > "$OUT/bench_c5.log" 2>&1
B="python bench.py --config c5 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --groups-per-rank 4"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:'depth_kernel|ms_kernel' -s 0 -c 2 -o "$OUT/depth_ms_c5" $B > "$OUT/ncu_depth.log" 2>&1
echo "rc=$?" >> "$OUT/ncu_depth.log"
echo done > "$OUT/DONE"
