#!/bin/bash
# Round-2 final evidence at the committed tree: GPU parity, smoke, default bench (e2e + CPU
# oracle), c3/c4 lines, IBFS_TD_SCHECK=2 A/B, ncu launch list (DRAM bytes per launch)
set -u
OUT=gpurun_out/${1:-r02x}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
(nvidia-smi; nproc; lscpu | head -20) > "$OUT/info.txt" 2>&1
timeout 2400 python -m pytest tests -m gpu -q > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > "$OUT/smoke.log" 2>&1; echo "smoke rc=$?" >> "$OUT/smoke.log"
timeout 1200 python bench.py --json-out "$OUT/bench_c5.json" > "$OUT/bench_c5.log" 2>&1
for c in c3 c4; do
  timeout 900 python bench.py --config $c --json-out "$OUT/bench_$c.json" > "$OUT/bench_$c.log" 2>&1
done
for c in ; do
  IBFS_TD_SCHECK=2 timeout 900 python bench.py --config $c --no-e2e --no-cpu-baseline --json-out "$OUT/bench_${c}_sc2.json" > "$OUT/bench_${c}_sc2.log" 2>&1
done
# timeout 900 python bench.py --config c5 --max-depth 3 --no-e2e --json-out "$OUT/bench_c5_3hop.json" > "$OUT/bench_c5_3hop.log" 2>&1
timeout 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -k regex:'level_kernel|depth_|init_|ms_kernel|iso_fix|late_fix|ring_clean|digest_kernel' --csv --log-file "$OUT/launches_c5.csv" \
  python bench.py --config c5 --steps 8 --warmup 3 --no-e2e --no-cpu-baseline > "$OUT/launches_c5.log" 2>&1
echo "rc=$?" >> "$OUT/launches_c5.log"
echo done > "$OUT/DONE"
