mkdir -p gpurun_out/r01h
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r01h/pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r01h/pytest.log
PROBE_GROUPS=16,28 timeout 900 python tools/bitstats.py c5 > gpurun_out/r01h/bitstats_c5.txt 2>&1
PROBE_GROUPS=0,6 timeout 900 python tools/bitstats.py c3 > gpurun_out/r01h/bitstats_c3.txt 2>&1
for sd in 16 64 256; do PROBE_GROUPS=0,16,28,31 timeout 600 python tools/probe.py c5 1 split_div=$sd > gpurun_out/r01h/probe_c5_sd$sd.txt 2>&1; done
for sd in 16 64 256; do PROBE_GROUPS=0,6 timeout 600 python tools/probe.py c3 1 split_div=$sd > gpurun_out/r01h/probe_c3_sd$sd.txt 2>&1; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:depth_kernel -c 1 -o gpurun_out/r01h/depth_c5 python tools/probe.py c5 1 > gpurun_out/r01h/ncu_depth.log 2>&1
