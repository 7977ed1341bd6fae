#!/bin/bash
# m_s pass returns the ring to zero (IBFS_MS_CLEAN): GPU parity + A/B bench; stmatrix layout probe
set -u
OUT=gpurun_out/${1:-r02w}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
./tools/diag/stmatrix_probe > "$OUT/stmatrix_probe.txt" 2>&1
timeout 2400 python -m pytest tests -m gpu -q ${PYTEST_EXTRA:-} > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
B="timeout 900 python bench.py --no-e2e --no-cpu-baseline"
for c in c5 c3 c4; do
  for mc in 1 0; do
    IBFS_MS_CLEAN=$mc $B --config $c --json-out "$OUT/bench_${c}_mc$mc.json" > "$OUT/bench_${c}_mc$mc.log" 2>&1
  done
done
echo done > "$OUT/DONE"
