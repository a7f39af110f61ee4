#!/bin/bash
# Interleaved A/B timing of libhsort builds on one box: tools/ab_run.sh a.so b.so ... (2 rounds)
for r in 1 2; do for so in "$@"; do timeout 120 python tools/bench_lib.py $so 2>&1 | grep -E "pass_ms|Error|error"; done; done
