#!/bin/bash
# Round-2 GPU call: build, GPU parity, bench lines (+ A/B of the depth kernel), ncu captures.
set -u
OUT=gpurun_out/${1:-r02b}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { echo build failed; cat "$OUT/build.log"; exit 1; }
timeout 1800 python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
for c in ${CONFIGS:-c5 c4 c3}; do
  timeout 900 python bench.py --config $c --json-out "$OUT/bench_$c.json" > "$OUT/bench_$c.log" 2>&1
done
if [ -n "${AB:-}" ]; then
  IBFS_DEPTH_TMA=0 timeout 900 python bench.py --config c5 --no-e2e --no-cpu-baseline --json-out "$OUT/bench_c5_notma.json" > "$OUT/bench_c5_notma.log" 2>&1
fi
echo done > "$OUT/DONE"
if [ -n "${NCU:-}" ]; then
  B="python bench.py --config c5 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-clocks"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:depth_tma_kernel -c 1 -o "$OUT/depth_tma_c5" $B > "$OUT/ncu_depth.log" 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:level_kernel -s 1 -c 4 -o "$OUT/level_c5" $B > "$OUT/ncu_level.log" 2>&1
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    -k regex:'level_kernel|depth|init_|ms_kernel|late_fix|iso_fix' --csv --log-file "$OUT/launches_c5.csv" \
    python bench.py --config c5 --steps 8 --warmup 0 --no-e2e --no-cpu-baseline --no-clocks > "$OUT/launches_c5.log" 2>&1
fi
echo done2 > "$OUT/DONE2"
