export EGGSYNC_LIB=/root/repo/scratch/variants/lib_d10.so
BIG=1 timeout 300 python scratch/tc2check.py 2>&1 | grep -v "^\[tc" > gpurun_out/dev_plan.log
timeout 200 python scratch/iterbench.py C3 2 2>&1 | tail -1 >> gpurun_out/dev_plan.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/dev_plan_launch.csv python scratch/tcprof.py C3 > /dev/null 2>&1
