#!/bin/bash
# clean-ring A/B parity diagnosis: digests per env setting on c2 / c3, targeted parity tests
set -u
OUT=gpurun_out/${1:-r02m}; mkdir -p "$OUT"
python -c "import __graft_entry__ as e; e.build()" > "$OUT/build.log" 2>&1 || { cat "$OUT/build.log"; exit 1; }
for c in c2 c3; do
  for v in "0 0" "1 0" "1 1"; do
    set -- $v
    IBFS_VERBOSE=1 IBFS_CLEAN_RING=$1 IBFS_FUSED_CLEAN=$2 timeout 600 python tools/diag/clean_ring_ab.py $c "$OUT/dig_${c}_cr$1_fc$2.npz" 8 > "$OUT/dig_${c}_cr$1_fc$2.log" 2>&1
  done
done
for v in "1 0" "1 1"; do
  set -- $v
  IBFS_CLEAN_RING=$1 IBFS_FUSED_CLEAN=$2 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q \
    -k "fig1_all or random_tiny or config1 or config2_full or late_list or range_error or directed_config" > "$OUT/pytest_cr$1_fc$2.log" 2>&1
  echo "rc=$?" >> "$OUT/pytest_cr$1_fc$2.log"
done
echo done > "$OUT/DONE"
