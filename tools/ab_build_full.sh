#!/bin/bash
# build a full libhsort variant with $EXTRA defines: paper_conf_ipps_gowanlockk18a_b200/ab/<name>.so
set -e
name=$1; d=paper_conf_ipps_gowanlockk18a_b200; o=$d/build/ab/$name; mkdir -p $o $d/ab
for f in radix merge codec msd; do nvcc -O3 -lineinfo -std=c++17 $EXTRA -gencode arch=compute_100a,code=sm_100a -Xcompiler -fPIC -c $d/csrc/$f.cu -o $o/$f.o & done
for f in api pool host_merge; do g++ -O3 -std=c++17 -fPIC -pthread $EXTRA -I/usr/local/cuda/include -c $d/csrc/$f.cpp -o $o/$f.o & done
wait
nvcc -shared -gencode arch=compute_100a,code=sm_100a -cudart static -o $d/ab/$name.so $o/*.o -lpthread
echo built $d/ab/$name.so
