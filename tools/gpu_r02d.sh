#!/bin/bash
# A/B of the bottom-up frontier-bitmap probe policy (IBFS_BU_PROBE 0/1/2) and per-group probes.
set -u
OUT=gpurun_out/${1:-r02d}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
for p in 1 0 2; do
  for c in c5 c3; do
    IBFS_BU_PROBE=$p timeout 900 python bench.py --config $c --no-e2e --no-cpu-baseline --json-out "$OUT/bench_${c}_p$p.json" > "$OUT/bench_${c}_p$p.log" 2>&1
  done
done
for p in 1 0; do
  IBFS_BU_PROBE=$p PROBE_HOPS=2 PROBE_ITERS=32 timeout 600 python tools/probe.py c5 1 > "$OUT/probe_c5_p$p.txt" 2>&1
done
if [ -n "${PYTEST_K:-}" ]; then
  timeout 1800 python -m pytest tests -m gpu -x -q -k "$PYTEST_K" > "$OUT/pytest_gpu.log" 2>&1; echo "rc=$?" >> "$OUT/pytest_gpu.log"
fi
echo done > "$OUT/DONE"
