#!/bin/bash
# GPU parity (all -m gpu tests but the c5 golden one until it exists) + bench lines; c5 golden in the background
set -u
OUT=gpurun_out/${1:-r02q}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
[ -n "${GOLDEN_THREADS:-}" ] && source tools/box_golden.sh; GOLDEN_PID=${GOLDEN_PID:-}
DESEL=""
if [ ! -f tests/golden/c5_ms_digest.npz ]; then
  DESEL="--deselect tests/test_gpu_fullsize.py::test_c5_bench_shape_all_digests_and_sampled_rows --deselect tests/test_gpu_fullsize.py::test_golden_files_are_oracle_written"
fi
timeout 2400 python -m pytest tests -m gpu -q $DESEL > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
for c in ${CONFIGS:-c5 c3 c4}; do
  timeout 900 python bench.py --config $c --no-e2e --no-cpu-baseline --json-out "$OUT/bench_$c.json" > "$OUT/bench_$c.log" 2>&1
done
PROBE_HOPS=2 PROBE_ITERS=8 timeout 900 python tools/probe.py c5 > "$OUT/probe_c5.txt" 2>&1
sleep ${GOLDEN_EXTRA:-0}
[ -n "$GOLDEN_PID" ] && kill $GOLDEN_PID 2>/dev/null
echo done > "$OUT/DONE"
