# compute-sanitizer memcheck / racecheck / synccheck / initcheck on the hot paths (logs -> gpurun_out/)
export PYTHONUNBUFFERED=1
for tool in memcheck synccheck racecheck initcheck; do
  for c in ${CASES:-c1_small c1_grid tc simt def42 def42_direct}; do
    echo "== $tool $c" >> gpurun_out/sanitize.log
    timeout 900 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 python scratch/sanitize_case.py $c > gpurun_out/san_${tool}_${c}.log 2>&1
    echo "rc=$?" >> gpurun_out/sanitize.log
    tail -3 gpurun_out/san_${tool}_${c}.log >> gpurun_out/sanitize.log
  done
done
