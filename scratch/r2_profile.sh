# round-2 evidence: full ncu capture of the 4 k_update_tc launches of one C3 clustering, launch
# list of the bench command (cold-cache, serialised: shares not absolute times)
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:k_update_tc -c 4 -o gpurun_out/ncu_tc_r2 -f python scratch/tcprof.py C3 > gpurun_out/ncu_tc_r2.log 2>&1; echo full $?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches_r2.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-direct > gpurun_out/launches_r2_bench.log 2>&1; echo launch $?
