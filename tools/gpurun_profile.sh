mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_radix.py -q -x -k "lookback or above_2p30" > gpurun_out/t_lb.txt 2>&1
for i in 1 2; do timeout 300 python bench.py > gpurun_out/bench_s32_$i.json 2> gpurun_out/bench_s32_$i.err; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r01_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_list.log 2>&1
tail -2 gpurun_out/t_lb.txt
