# GPU merge check: parity tests of K4/K5 + tools/merge_bench.py, A/B libraries in ab/m_*.so;
# optional ncu capture (NCU=1).  usage: bash tools/gpurun_merge.sh <tag>
tag=${1:-m}
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_merge_api.py -x -q > gpurun_out/${tag}_pytest.txt 2>&1; echo "exit $?" >> gpurun_out/${tag}_pytest.txt
timeout 300 python tools/merge_bench.py 30 2,4,8,12,32,128 > gpurun_out/${tag}_bench.jsonl 2>&1
timeout 300 python tools/merge_bench.py 30 12 normal >> gpurun_out/${tag}_bench.jsonl 2>&1
timeout 300 python tools/merge_bench.py 30 12 zipf_dup >> gpurun_out/${tag}_bench.jsonl 2>&1
for lib in $(ls paper_conf_ipps_gowanlockk18a_b200/ab/m_*.so 2>/dev/null); do
  echo "== $lib" >> gpurun_out/${tag}_bench.jsonl
  HSORT_LIB=$lib timeout 300 python tools/merge_bench.py 30 2,8,12,128 >> gpurun_out/${tag}_bench.jsonl 2>&1
done
if [ -n "$NCU" ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:merge_tile -s 3 -c 1 -o gpurun_out/${tag}_k5_full python tools/merge_bench.py 28 12 > gpurun_out/${tag}_ncu_k5.log 2>&1
fi
tail -2 gpurun_out/${tag}_pytest.txt; cat gpurun_out/${tag}_bench.jsonl
