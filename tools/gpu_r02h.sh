#!/bin/bash
set -u
OUT=gpurun_out/${1:-r02h}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
timeout 1500 python -m pytest tests -m gpu -x -q -k "${PYTEST_K:-test_gpu_parity}" > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
timeout 900 python bench.py --config c4 --no-e2e --no-cpu-baseline --json-out "$OUT/bench_c4.json" > "$OUT/bench_c4.log" 2>&1
for sd in 128 256 512 1024 4096; do
  timeout 600 python bench.py --config c5 --no-e2e --no-cpu-baseline --no-clocks --split-div $sd --json-out "$OUT/bench_c5_s${sd}.json" > "$OUT/bench_c5_s${sd}.log" 2>&1
done
for sd in 64 256 1024; do
  timeout 600 python bench.py --config c3 --no-e2e --no-cpu-baseline --no-clocks --split-div $sd --json-out "$OUT/bench_c3_s${sd}.json" > "$OUT/bench_c3_s${sd}.log" 2>&1
  timeout 600 python bench.py --config c4 --no-e2e --no-cpu-baseline --no-clocks --split-div $sd --json-out "$OUT/bench_c4_s${sd}.json" > "$OUT/bench_c4_s${sd}.log" 2>&1
done
echo done > "$OUT/DONE"
