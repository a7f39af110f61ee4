#!/bin/bash
# ncu --set full of one random-digit K3 pass for each given .so (source counters)
mkdir -p gpurun_out
K="--set full --clock-control none --import-source on --kernel-name-base demangled"
for so in "$@"; do
  nm=$(basename $so .so)
  HSORT_AB_NO_DDE=1 timeout 600 ncu $K -k "regex:k_onesweep_ws<\(int\)576, \(int\)15, \(bool\)0, \(bool\)0, \(int\)0" -s 12 -c 1 -o gpurun_out/r03d_${nm}_k3 python tools/bench_lib.py $so > gpurun_out/r03d_${nm}_ncu.log 2>&1
  echo "$nm exit $?"
done
