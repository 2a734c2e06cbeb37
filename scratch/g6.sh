# round-1 measurement: bench line, launch list of the same command, full captures of the update kernels
timeout 400 python bench.py > gpurun_out/bench_r1b.log 2>&1; echo bench $?
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1b.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/ncu_bench.log 2>&1; echo launches $?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_update_tc -c 4 -o gpurun_out/tc_full python scratch/tcprof.py C3 > gpurun_out/ncu_tc.log 2>&1; echo tcfull $?
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_tc_plan -c 1 -o gpurun_out/plan_full python scratch/tcprof.py C3 > gpurun_out/ncu_plan.log 2>&1; echo planfull $?
