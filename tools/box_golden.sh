#!/bin/bash
# Background c5 golden chunks on the GPU box's spare host cores (tools/make_golden.py, oracle
# only), from the last chunk down; the chunks come back under gpurun_out/golden_ckpt_box/ and
# tools/make_golden.py --assemble joins them with the local ones.  usage: source this file.
mkdir -p gpurun_out/golden_ckpt_box
nice -n 19 python tools/make_golden.py c5 --threads ${GOLDEN_THREADS:-10} --reverse \
  --ckpt gpurun_out/golden_ckpt_box --extra-ckpt tests/golden/c5_ckpt > gpurun_out/golden_box.log 2>&1 &
GOLDEN_PID=$!
