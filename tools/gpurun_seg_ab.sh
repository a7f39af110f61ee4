mkdir -p gpurun_out; o=gpurun_out/r01s_seg2.jsonl; : > $o
timeout 600 python -m pytest tests/test_gpu_merge_api.py tests/test_gpu_radix.py -x -q > gpurun_out/r01s_seg2_pytest.txt 2>&1; echo "exit $?" >> gpurun_out/r01s_seg2_pytest.txt
for r in 1 2; do
for lib in seg2 paper_conf_ipps_gowanlockk18a_b200/ab/m_noseg2.so; do
  echo "== $lib round $r" >> $o
  if [ $lib = seg2 ]; then unset HSORT_LIB; else export HSORT_LIB=$lib; fi
  timeout 300 python tools/merge_bench.py 30 12,17,24,32 >> $o 2>&1
  timeout 300 python tools/merge_bench.py 30 32 zipf_dup >> $o 2>&1
done; done
