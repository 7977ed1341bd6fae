#!/bin/bash
# c4 host-gap diagnosis + alpha / split_div sweep on c5
set -u
OUT=gpurun_out/${1:-r02g}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
timeout 900 python bench.py --config c4 --no-e2e --no-cpu-baseline --json-out "$OUT/bench_c4.json" > "$OUT/bench_c4.log" 2>&1
for al in 2 4 8; do for sd in 16 64 256; do
  timeout 600 python bench.py --config c5 --no-e2e --no-cpu-baseline --no-clocks --alpha $al --split-div $sd --json-out "$OUT/bench_c5_a${al}_s${sd}.json" > "$OUT/bench_c5_a${al}_s${sd}.log" 2>&1
done; done
echo done > "$OUT/DONE"
