#!/bin/bash
# compile check of libibfs with ptxas resource usage for the main kernels (CPU only)
cd "$(dirname "$0")/.." && nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC \
  -c paper_conf_sigmod_liuhh16_b200/csrc/ibfs.cu -o /tmp/ibfs_ck.o -Xptxas -v 2>&1 | \
  grep -E "error|Compiling entry function '_ZN4ibfs1[0-9](expand|commit|depth|level)[a-z_]*IN" -A2 | grep -E "error|Compiling|Used|spill" | sed 's/ptxas info    : //'
