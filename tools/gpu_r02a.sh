#!/bin/bash
# Round-2 first GPU call: build, memory ceilings, GPU parity, bench lines.
set -u
OUT=gpurun_out/${1:-r02a}; mkdir -p "$OUT"
(nvidia-smi; nproc; free -g; lscpu | head -20) > "$OUT/info.txt" 2>&1
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/randbench tools/randbench.cu >> "$OUT/build.log" 2>&1
timeout 300 ./tools/randbench > "$OUT/randbench.json" 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} > "$OUT/pytest_gpu.log" 2>&1
echo "rc=$?" >> "$OUT/pytest_gpu.log"
for c in ${CONFIGS:-c5 c4 c3}; do
  timeout 900 python bench.py --config $c --json-out "$OUT/bench_$c.json" > "$OUT/bench_$c.log" 2>&1
done
echo done > "$OUT/DONE"
