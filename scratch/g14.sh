timeout 400 python -m pytest tests/test_gpu_cw_factor.py -x -q > gpurun_out/g14_tests.log 2>&1; echo tests $?
timeout 200 python scratch/syncbench.py C2 > gpurun_out/g14_sync.log 2>&1; echo sync $?
