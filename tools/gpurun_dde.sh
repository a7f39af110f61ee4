# DDE check: tests + per-pass A/B (current lib: dde on/off; ab/pre.so: the build before the elision)
mkdir -p gpurun_out
tag=${1:-dde}
timeout 600 python -m pytest tests/test_gpu_dde.py -x -q > gpurun_out/${tag}_pytest.txt 2>&1; echo "exit $?" >> gpurun_out/${tag}_pytest.txt
tail -3 gpurun_out/${tag}_pytest.txt
timeout 300 python tools/dde_ab.py > gpurun_out/${tag}_ab.txt 2>&1
[ -f paper_conf_ipps_gowanlockk18a_b200/ab/pre.so ] && HSORT_LIB=paper_conf_ipps_gowanlockk18a_b200/ab/pre.so timeout 300 python tools/dde_ab.py >> gpurun_out/${tag}_ab.txt 2>&1
cat gpurun_out/${tag}_ab.txt
