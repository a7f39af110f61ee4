#!/bin/bash
# Interleaved A/B timing of libhsort builds on one box: [AB_DISTS="uniform normal"] tools/ab_run.sh a.so b.so ... (2 rounds)
for r in 1 2; do for d in ${AB_DISTS:-uniform}; do for so in "$@"; do timeout 120 python tools/bench_lib.py $so $d 2>&1 | grep -E "pass_ms|Error|error"; done; done; done
