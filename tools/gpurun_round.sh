#!/bin/bash
# Full round check on one B200: GPU tests, smoke, bench x2, ncu launch list, ncu --set full of K3 + K1.
# usage (from the repo root, via gpurun): bash tools/gpurun_round.sh <tag>
tag=${1:-r01}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > gpurun_out/${tag}_smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/${tag}_pytest_gpu.txt 2>&1
echo "pytest exit $?" >> gpurun_out/${tag}_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.txt 2>&1
for i in 1 2; do timeout 400 python bench.py > gpurun_out/${tag}_bench_$i.json 2> gpurun_out/${tag}_bench_$i.err; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${tag}_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/${tag}_ncu_list.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 17 -c 1 -o gpurun_out/${tag}_onesweep_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/${tag}_ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hist -s 2 -c 1 -o gpurun_out/${tag}_hist_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/${tag}_ncu_full2.log 2>&1
tail -3 gpurun_out/${tag}_pytest_gpu.txt
cat gpurun_out/${tag}_bench_1.json
