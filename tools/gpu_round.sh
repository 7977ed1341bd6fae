#!/bin/bash
# One gpurun call: GPU parity tests, bench lines, ncu launch list + one full capture.
# usage (from the repo root, under gpurun): bash tools/gpu_round.sh [tag] [steps...]
# steps: info tests smoke bench_c5 bench_c3 bench_c4 launches full   (default: all)
set -u
TAG=${1:-r01}
shift || true
STEPS=${*:-"info tests smoke bench_c5 bench_c3 bench_c4 launches full"}
OUT=gpurun_out/$TAG
mkdir -p "$OUT"
has() { [[ " $STEPS " == *" $1 "* ]]; }
if has info; then
  (nvidia-smi; nproc; free -g; lscpu | head -20) > "$OUT/info.txt" 2>&1
fi
if has tests; then
  timeout 1500 python -m pytest tests -m gpu -x -q > "$OUT/pytest_gpu.log" 2>&1
  echo "pytest rc=$?" >> "$OUT/pytest_gpu.log"
fi
if has smoke; then
  timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > "$OUT/smoke.log" 2>&1
  echo "smoke rc=$?" >> "$OUT/smoke.log"
fi
for c in c5 c3 c4 c2; do
  if has bench_$c; then
    timeout 900 python bench.py --config $c --json-out "$OUT/bench_$c.json" > "$OUT/bench_$c.log" 2>&1
    echo "bench $c rc=$?" >> "$OUT/bench_$c.log"
  fi
done
NCU_CFG=${NCU_CFG:-c5}
if has launches; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none \
    -k regex:'level_kernel|depth_kernel|init_|ms_kernel|iso_fix|digest_kernel' \
    --csv --log-file "$OUT/launches_$NCU_CFG.csv" \
    python bench.py --config $NCU_CFG --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > "$OUT/launches_$NCU_CFG.log" 2>&1
  echo "launches rc=$?" >> "$OUT/launches_$NCU_CFG.log"
fi
if has full; then
  timeout 1200 ncu --set full --clock-control none --import-source on \
    -k regex:${NCU_KREGEX:-level_kernel} -s ${NCU_SKIP:-6} -c ${NCU_COUNT:-3} -o "$OUT/full_${NCU_KREGEX:-level_kernel}_$NCU_CFG" \
    python bench.py --config $NCU_CFG --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > "$OUT/full_$NCU_CFG.log" 2>&1
  echo "full rc=$?" >> "$OUT/full_$NCU_CFG.log"
fi
echo done > "$OUT/DONE"
