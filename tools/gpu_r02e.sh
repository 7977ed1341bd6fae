#!/bin/bash
# Round-2 GPU call: build, parity subset, bench c5/c3 (commit L2 prefetch, depth E_k),
# ncu of a mixed group's big bottom-up level, c2 report.
set -u
OUT=gpurun_out/${1:-r02e}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
timeout 1500 python -m pytest tests -m gpu -x -q -k "${PYTEST_K:-test_gpu_parity}" > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
for c in c5 c3 c4; do
  timeout 900 python bench.py --config $c --no-e2e --no-cpu-baseline --json-out "$OUT/bench_$c.json" > "$OUT/bench_$c.log" 2>&1
done
PROBE_HOPS=2 PROBE_GROUPS=25 timeout 600 ncu --set full --clock-control none --import-source on -k regex:level_kernel -s 2 -c 1 \
  -o "$OUT/level_g25_l3" python tools/probe.py c5 1 > "$OUT/ncu_g25.log" 2>&1
timeout 900 python tools/c2_report.py --out "$OUT/c2_report.md" > "$OUT/c2_report.log" 2>&1
echo done > "$OUT/DONE"
