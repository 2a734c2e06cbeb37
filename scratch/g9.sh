# final round-1 measurement: tests, bench line, per-stage times, launch list, full captures
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/f_tests.log 2>&1; echo tests $?
timeout 400 python bench.py > gpurun_out/f_bench.log 2>&1; echo bench $?
timeout 300 python scratch/stagebench.py C1 C2 C3 C4-d2 C4-d5 C4-d10 C4-d16 C4-d20 > gpurun_out/f_stages.log 2>&1; echo stages $?
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/f_launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu > gpurun_out/f_ncu_bench.log 2>&1; echo launches $?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_update_tc -c 4 -o gpurun_out/f_tc_full python scratch/tcprof.py C3 > gpurun_out/f_ncu_tc.log 2>&1; echo tcfull $?
