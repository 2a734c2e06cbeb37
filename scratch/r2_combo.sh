timeout 900 compute-sanitizer --tool racecheck --print-limit 20 --error-exitcode 9 python scratch/sanitize_case.py c1_small > gpurun_out/san_racecheck_c1_small_fixed.log 2>&1; echo "racecheck c1_small fixed rc=$?" > gpurun_out/combo.log
VARS=d10 bash scratch/r2_var.sh
