# round-2 (late) evidence: full ncu capture of the 4 k_update_tc launches of one C3 clustering
# (summarised on the box: raw metrics + per-SASS source page as CSV; the report itself is too
# big to bring back), the plan / tree / cell kernels, and the launch list of the bench command
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:k_update_tc -c 4 -o /tmp/ncu_tc_r2c -f python scratch/tcprof.py C3 > gpurun_out/ncu_tc_r2c.log 2>&1; echo full $?
ncu -i /tmp/ncu_tc_r2c.ncu-rep --page raw --csv > gpurun_out/ncu_tc_r2c_raw.csv 2>/dev/null
ncu -i /tmp/ncu_tc_r2c.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_tc_r2c_sass.csv 2>/dev/null
gzip -f gpurun_out/ncu_tc_r2c_sass.csv
# (build-kernel capture: see profiles/ncu_build_r2b.txt)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches_r2c.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-direct > gpurun_out/launches_r2c_bench.log 2>&1; echo launch $?
ls -la gpurun_out
