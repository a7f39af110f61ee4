#!/bin/bash
# One B200 check: GPU tests, smoke, one bench run.  usage: bash tools/gpurun_check.sh <tag> [pytest args]
tag=${1:-r02}; shift
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > gpurun_out/${tag}_smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q ${@} > gpurun_out/${tag}_pytest_gpu.txt 2>&1
echo "pytest exit $?" >> gpurun_out/${tag}_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.txt 2>&1
echo "smoke exit $?" >> gpurun_out/${tag}_smoke.txt
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
echo "bench exit $?" >> gpurun_out/${tag}_bench.err
tail -2 gpurun_out/${tag}_pytest_gpu.txt; tail -1 gpurun_out/${tag}_smoke.txt; tail -3 gpurun_out/${tag}_bench.err
