#!/bin/bash
# clean ring: GPU parity (IBFS_CHECK_RING=1 via conftest), bench A/B (IBFS_CLEAN_RING=0/1)
set -u
OUT=gpurun_out/${1:-r02j}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
source tools/box_golden.sh
if [ ! -f tests/golden/c5_ms_digest.npz ]; then  # c5 golden still being written
  PYTEST_ARGS="${PYTEST_ARGS:-} --deselect tests/test_gpu_fullsize.py::test_c5_bench_shape_all_digests_and_sampled_rows[c5] --deselect tests/test_gpu_fullsize.py::test_golden_files_are_oracle_written"
fi
timeout 2400 python -m pytest tests -m gpu -q -x ${PYTEST_ARGS:-} > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
for c in c5 c3 c4; do
  for cr in 1 0; do
    IBFS_CLEAN_RING=$cr timeout 900 python bench.py --config $c --no-e2e --no-cpu-baseline --json-out "$OUT/bench_${c}_cr$cr.json" > "$OUT/bench_${c}_cr$cr.log" 2>&1
  done
done
kill $GOLDEN_PID 2>/dev/null
echo done > "$OUT/DONE"
