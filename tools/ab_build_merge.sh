#!/bin/bash
# Build a copy of libhsort.so with merge.cu compiled under $EXTRA: paper_conf_ipps_gowanlockk18a_b200/ab/<name>.so
set -e
name=$1
d=paper_conf_ipps_gowanlockk18a_b200
mkdir -p $d/ab $d/build/ab
nvcc -O3 -lineinfo -std=c++17 $EXTRA -gencode arch=compute_100a,code=sm_100a -Xcompiler -fPIC -c $d/csrc/merge.cu -o $d/build/ab/merge_$name.o
nvcc -shared -gencode arch=compute_100a,code=sm_100a -cudart static -o $d/ab/$name.so $d/build/radix.o $d/build/ab/merge_$name.o $d/build/codec.o $d/build/msd.o $d/build/api.o $d/build/pool.o $d/build/host_merge.o -lpthread
echo built $d/ab/$name.so
