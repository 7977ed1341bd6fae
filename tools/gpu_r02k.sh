#!/bin/bash
# fused clean ring: GPU parity (IBFS_CHECK_RING=1 via conftest), bench A/B, c5 per-level probe;
# the c5 golden in the background on the box's host cores
set -u
OUT=gpurun_out/${1:-r02k}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
GOLDEN_THREADS=${GOLDEN_THREADS:-12} source tools/box_golden.sh
DESEL=""
if [ ! -f tests/golden/c5_ms_digest.npz ]; then  # c5 golden still being written
  DESEL="--deselect tests/test_gpu_fullsize.py::test_c5_bench_shape_all_digests_and_sampled_rows --deselect tests/test_gpu_fullsize.py::test_golden_files_are_oracle_written"
fi
timeout 2400 python -m pytest tests -m gpu -q -x $DESEL > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
for c in c5 c4 c3; do
  for v in ${VARIANTS:-1_1 1_0 0_1}; do
    set -- ${v/_/ }
    IBFS_CLEAN_RING=$1 IBFS_FUSED_CLEAN=$2 timeout 900 python bench.py --config $c --no-e2e --no-cpu-baseline --json-out "$OUT/bench_${c}_cr$1_fc$2.json" > "$OUT/bench_${c}_cr$1_fc$2.log" 2>&1
  done
done
PROBE_HOPS=2 PROBE_ITERS=32 timeout 900 python tools/probe.py c5 > "$OUT/probe_c5.txt" 2>&1
wait_golden() { sleep ${GOLDEN_EXTRA:-0}; }
wait_golden
kill $GOLDEN_PID 2>/dev/null
echo done > "$OUT/DONE"
