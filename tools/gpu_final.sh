#!/bin/bash
# Round-end evidence: GPU parity, smoke, bench lines (full contract), k-hop line, reference arm,
# ncu --set full captures of the heavy level launches and the depth kernel (c5).
set -u
OUT=gpurun_out/${1:-final}; mkdir -p "$OUT"
(nvidia-smi; nproc; lscpu | head -20) > "$OUT/info.txt" 2>&1
if [ -z "${SKIP_PYTEST:-}" ]; then  # SKIP_PYTEST=1: the same tree's GPU parity log comes from another call
  timeout 1500 python -m pytest tests -m gpu -x -q > "$OUT/pytest_gpu.log" 2>&1
  echo "rc=$?" >> "$OUT/pytest_gpu.log"
fi
timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > "$OUT/smoke.log" 2>&1
echo "rc=$?" >> "$OUT/smoke.log"
for c in c5 c4 c3; do
  timeout 900 python bench.py --config $c --json-out "$OUT/bench_$c.json" > "$OUT/bench_$c.log" 2>&1
done
timeout 600 python bench.py --config c5 --max-depth 3 --no-e2e --json-out "$OUT/bench_c5_3hop.json" > "$OUT/bench_c5_3hop.log" 2>&1
timeout 600 python bench.py --impl reference --config c5 --steps 2 --warmup 1 > "$OUT/bench_ref_c5.log" 2>&1
B="python bench.py --config c5 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:level_kernel -s 1 -c 3 -o "$OUT/level_kernel_c5" $B > "$OUT/ncu_level.log" 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:depth_kernel -s 0 -c 1 -o "$OUT/depth_kernel_c5" $B > "$OUT/ncu_depth.log" 2>&1
echo done > "$OUT/DONE"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -k regex:'level_kernel|depth_kernel|init_|ms_kernel|iso_fix' --csv --log-file "$OUT/launches_c5.csv" \
  python bench.py --config c5 --steps 8 --warmup 0 --no-e2e --no-cpu-baseline > "$OUT/launches_c5.log" 2>&1
echo done2 > "$OUT/DONE2"
