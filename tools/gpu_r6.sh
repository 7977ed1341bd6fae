#!/bin/bash
set -u
OUT=gpurun_out/${1:-r01g}; mkdir -p "$OUT"
CFGS="c5 c4 c3" bash tools/gpu_ab.sh ${1:-r01g} default d5m3 d3m4
timeout 900 python -m pytest tests -m gpu -x -q -k "config or edge or tiny or fig1 or khop or directed" > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
echo done > "$OUT/DONE"
