#!/bin/bash
# A/B IBFS_TD_SCHECK; full default bench line (e2e + CPU oracle), smoke, reference arm
set -u
OUT=gpurun_out/${1:-r02v}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
B="timeout 900 python bench.py --no-e2e --no-cpu-baseline"
for c in c5 c3 c4; do
  for sc in 0 1; do
    IBFS_TD_SCHECK=$sc $B --config $c --json-out "$OUT/bench_${c}_sc$sc.json" > "$OUT/bench_${c}_sc$sc.log" 2>&1
  done
done
IBFS_TD_SCHECK=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "fig1_all or random_tiny or config1 or config2_full or directed_config" > "$OUT/pytest_sc1.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_sc1.log"
timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > "$OUT/smoke.log" 2>&1; echo "smoke rc=$?" >> "$OUT/smoke.log"
timeout 1200 python bench.py --json-out "$OUT/bench_default.json" > "$OUT/bench_default.log" 2>&1
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > "$OUT/bench_reference.log" 2>&1
echo done > "$OUT/DONE"
