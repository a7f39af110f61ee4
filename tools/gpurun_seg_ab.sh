mkdir -p gpurun_out; o=gpurun_out/r01t_ilp.jsonl; : > $o
timeout 600 python -m pytest tests/test_gpu_merge_api.py tests/test_gpu_radix.py -x -q > gpurun_out/r01t_ilp_pytest.txt 2>&1; echo "exit $?" >> gpurun_out/r01t_ilp_pytest.txt
for r in 1 2; do
for lib in ilp paper_conf_ipps_gowanlockk18a_b200/ab/m_noilp.so; do
  echo "== $lib round $r" >> $o
  if [ $lib = ilp ]; then unset HSORT_LIB; else export HSORT_LIB=$lib; fi
  timeout 300 python tools/merge_bench.py 30 4,8,12,16,48,64,128 >> $o 2>&1
  timeout 300 python tools/merge_bench.py 30 12,128 zipf_dup >> $o 2>&1
done; done
