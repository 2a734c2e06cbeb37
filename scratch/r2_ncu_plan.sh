export EGGSYNC_LIB=/root/repo/scratch/variants/lib_d10.so
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_tc_plan -c 2 -o gpurun_out/ncu_plan -f python scratch/tcprof.py C3 > gpurun_out/ncu_plan.log 2>&1; echo $?
