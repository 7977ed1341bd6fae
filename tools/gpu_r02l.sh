#!/bin/bash
# Round-2 evidence: ncu launch list (time + DRAM bytes) of an 8-step c5 bench, ncu --set full
# captures of the level kernel (levels 2-5 of the first batch) and the depth kernel, probe.
set -u
OUT=gpurun_out/${1:-r02l}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
[ -n "${GOLDEN_THREADS:-}" ] && source tools/box_golden.sh; GOLDEN_PID=${GOLDEN_PID:-}
CFG=${CFG:-c5}
timeout 900 python bench.py --config $CFG --no-e2e --no-cpu-baseline --json-out "$OUT/bench_$CFG.json" > "$OUT/bench_$CFG.log" 2>&1
timeout 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -k regex:'level_kernel|depth_|init_|ms_kernel|iso_fix|late_fix|ring_clean|digest_kernel' --csv --log-file "$OUT/launches_$CFG.csv" \
  python bench.py --config $CFG --steps 8 --warmup 3 --no-e2e --no-cpu-baseline > "$OUT/launches_$CFG.log" 2>&1
echo "rc=$?" >> "$OUT/launches_$CFG.log"
B="python bench.py --config $CFG --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-clocks"
for spec in ${SPECS:-level_kernel:1:4 depth_tma_kernel:0:1}; do
  IFS=: read k s c <<< "$spec"
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:$k -s $s -c $c \
    -o "$OUT/full_${k}_$CFG" $B > "$OUT/full_${k}_$CFG.log" 2>&1
  echo "rc=$?" >> "$OUT/full_${k}_$CFG.log"
done
# c4 APSP as one call per step (all 2,048 groups): the per-call host return amortised
timeout 900 python bench.py --config c4 --groups-per-rank 2048 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline \
  --json-out "$OUT/bench_c4_onecall.json" > "$OUT/bench_c4_onecall.log" 2>&1
sleep ${GOLDEN_EXTRA:-0}
[ -n "$GOLDEN_PID" ] && kill $GOLDEN_PID 2>/dev/null
echo done > "$OUT/DONE"
