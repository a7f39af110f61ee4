# compute-sanitizer over tools/sanitize_run.py (each tool under its own timeout)
mkdir -p gpurun_out
tag=${1:-san}
timeout 120 python tools/sanitize_run.py > gpurun_out/${tag}_plain.txt 2>&1; echo "exit $?" >> gpurun_out/${tag}_plain.txt
for tool in memcheck synccheck initcheck racecheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python tools/sanitize_run.py > gpurun_out/${tag}_$tool.txt 2>&1
  echo "exit $?" >> gpurun_out/${tag}_$tool.txt
done
for f in gpurun_out/${tag}_*.txt; do echo "== $f"; tail -4 $f; done
