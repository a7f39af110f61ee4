#!/bin/bash
# One --set full capture each of the dominant onesweep pass and the K1 histogram, inside the bench's
# device arm (2^30 keys): onesweep launch 18 = step 3 pass 2 (raw-key variant), hist launch 3.
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 17 -c 1 -o gpurun_out/r01_onesweep_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hist -s 2 -c 1 -o gpurun_out/r01_hist_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_full2.log 2>&1
