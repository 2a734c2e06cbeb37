timeout 300 python -m pytest tests/test_gpu_sync_brute.py -x -q > gpurun_out/g12_tests.log 2>&1; echo tests $?
timeout 200 python scratch/syncbench.py C1 C2 C4-d10 C3 > gpurun_out/g12_sync.log 2>&1; echo sync $?
timeout 200 ncu --metrics gpu__time_duration.sum,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_fma.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:k_sync_brute -c 3 --csv --log-file gpurun_out/g12_ncu.csv python scratch/syncbench.py C2 > /dev/null 2>&1; echo ncu $?
