#!/bin/bash
set -u
OUT=gpurun_out/${1:-r01e}; mkdir -p "$OUT"
timeout 1500 python -m pytest tests -m gpu -x -q > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
PROBE_GROUPS=0,5,23,31 timeout 600 python tools/probe.py c5 1 > "$OUT/probe_c5.txt" 2>&1
CFGS="c5 c3" bash tools/gpu_ab.sh ${1:-r01e} default m4 u8 m4u8
