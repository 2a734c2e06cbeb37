BIG=1 timeout 300 python scratch/tc2check.py > gpurun_out/var_check.log 2>&1; echo check $?
timeout 200 python scratch/iterbench.py C3 3 > gpurun_out/var_iter.log 2>&1; echo iter $?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_tree_agg -c 8 --csv --log-file gpurun_out/agg.csv python scratch/tcprof.py C3 > /dev/null 2>&1; echo ncu $?
