BIG=1 timeout 300 python scratch/tc2check.py > gpurun_out/var_check.log 2>&1; echo check $?
timeout 200 python scratch/iterbench.py C3 3 > gpurun_out/var_iter.log 2>&1; echo iter $?
bash scratch/r3_profile.sh
