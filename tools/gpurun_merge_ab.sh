#!/bin/bash
# interleaved K4/K5 A/B of merge.cu builds: bash tools/gpurun_merge_ab.sh <tag> a.so b.so ...
tag=$1; shift
for r in 1 2; do for so in "$@"; do HSORT_LIB=$so timeout 300 python tools/merge_bench.py 30 2,4,8,12,32,128 | sed "s#^#{\"lib\": \"$so\", \"round\": $r} #"; done; done > gpurun_out/${tag}_merge_ab.txt 2>&1
