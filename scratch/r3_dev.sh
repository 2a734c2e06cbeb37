# dev loop: TC parity checks + C3 per-iteration timings + the parity/path GPU tests
EGGSYNC_TC_DEBUG=1 BIG=1 timeout 300 python scratch/tc2check.py > gpurun_out/dev_check.log 2>&1; echo check $?
timeout 200 python scratch/iterbench.py C3 3 > gpurun_out/dev_iter.log 2>&1; echo iter $?
timeout 120 python scratch/iterbench.py C4-d10 2 >> gpurun_out/dev_iter.log 2>&1; echo iter2 $?
timeout 900 python -m pytest tests -m gpu -x -q -k "(paths or parity) and not C3" > gpurun_out/dev_tests.log 2>&1; echo tests $?
if [ -f scratch/variants/lib_d10p.so ]; then EGGSYNC_LIB=/root/repo/scratch/variants/lib_d10p.so timeout 120 python scratch/iterbench.py C3 1 > gpurun_out/dev_prof.log 2>&1; echo prof $?; fi
