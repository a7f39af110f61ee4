#!/bin/bash
# Round profile on one B200: GPU tests, smoke, bench, ncu launch list of the bench command, and
# one ncu --set full capture each of K3 (device arm), K5 (a merge chunk of the host->host arm)
# and K1.  usage (repo root, via gpurun): bash tools/gpurun_profile.sh <tag> [skip-tests]
tag=${1:-r02}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > gpurun_out/${tag}_smi.txt 2>&1
if [ "$2" != "skip-tests" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/${tag}_pytest_gpu.txt 2>&1
  echo "pytest exit $?" >> gpurun_out/${tag}_pytest_gpu.txt
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.txt 2>&1
  echo "smoke exit $?" >> gpurun_out/${tag}_smoke.txt
fi
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err
echo "bench exit $?" >> gpurun_out/${tag}_bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 5000 --csv --log-file gpurun_out/${tag}_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-extras > gpurun_out/${tag}_ncu_list.log 2>&1
K="--set full --clock-control none --import-source on --kernel-name-base demangled"
timeout 900 ncu $K -k "regex:k_onesweep_ws<\(int\)576, \(int\)15, \(bool\)0, \(bool\)0, \(int\)0" -s 10 -c 1 -o gpurun_out/${tag}_onesweep_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-extras --device-only --no-dde > gpurun_out/${tag}_ncu_full1.log 2>&1
timeout 900 ncu $K -k "regex:k_merge_tile" -s 20 -c 1 -o gpurun_out/${tag}_merge_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-extras > gpurun_out/${tag}_ncu_full2.log 2>&1
timeout 900 ncu $K -k "regex:k_hist3" -s 2 -c 1 -o gpurun_out/${tag}_hist_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-extras --device-only > gpurun_out/${tag}_ncu_full3.log 2>&1
ls -la gpurun_out/${tag}_* | tail -20
tail -2 gpurun_out/${tag}_pytest_gpu.txt 2>/dev/null; tail -1 gpurun_out/${tag}_smoke.txt 2>/dev/null; tail -2 gpurun_out/${tag}_bench.err
