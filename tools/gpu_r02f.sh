#!/bin/bash
set -u
OUT=gpurun_out/${1:-r02f}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
timeout 1500 python -m pytest tests -m gpu -x -q -k "${PYTEST_K:-test_gpu_parity}" > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
for c in ${CONFIGS:-c5 c3}; do
  timeout 900 python bench.py --config $c --no-e2e --no-cpu-baseline --json-out "$OUT/bench_$c.json" > "$OUT/bench_$c.log" 2>&1
done
PROBE_HOPS=2 PROBE_ITERS=32 timeout 600 python tools/probe.py c5 1 > "$OUT/probe_c5.txt" 2>&1
${EXTRA:-true}
echo done > "$OUT/DONE"
