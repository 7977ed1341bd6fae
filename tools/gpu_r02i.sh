#!/bin/bash
# Round-2 re-entry check: build, GPU tests (c5 golden pending), smoke, c5/c3/c4 bench lines.
set -u
OUT=gpurun_out/${1:-r02i}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
(nvidia-smi; nproc; lscpu | head -20) > "$OUT/info.txt" 2>&1
timeout 2400 python -m pytest tests -m gpu -q ${PYTEST_ARGS:-} > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > "$OUT/smoke.log" 2>&1; echo "smoke rc=$?" >> "$OUT/smoke.log"
for c in c5 c3 c4; do
  timeout 900 python bench.py --config $c --json-out "$OUT/bench_$c.json" > "$OUT/bench_$c.log" 2>&1
  echo "bench $c rc=$?" >> "$OUT/bench_$c.log"
done
echo done > "$OUT/DONE"
