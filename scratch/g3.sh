cd $GRAFT_REPO_ROOT
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/launches_tc.csv python scratch/tcprof.py C3 > gpurun_out/g3a.log 2>&1; echo a $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_update_tc -c 1 -o gpurun_out/tc_c3 python scratch/tcprof.py C3 > gpurun_out/g3b.log 2>&1; echo b $?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_tc_plan -c 1 -o gpurun_out/plan_c3 python scratch/tcprof.py C3 > gpurun_out/g3c.log 2>&1; echo c $?
