#!/bin/bash
# ncu --set full (source counters) of one K5 k_merge_tile launch at k = 12 (tools/merge_bench.py)
# usage: bash tools/ncu_k5.sh <tag> [lib.so]
mkdir -p gpurun_out
K="--set full --clock-control none --import-source on --kernel-name-base demangled"
HSORT_LIB=${2:-} timeout 600 ncu $K -k "regex:k_merge_tile" -s 2 -c 1 -o gpurun_out/${1}_k5 python tools/merge_bench.py 30 12 > gpurun_out/${1}_k5_ncu.log 2>&1
echo "ncu k5 exit $?"
