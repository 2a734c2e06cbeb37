timeout 1200 python -m pytest tests/test_gpu_def42.py tests/test_abi.py -x -q > gpurun_out/def42_tests.log 2>&1; echo tests $?
timeout 600 python scratch/def42bench.py C1 C2 C4-d10 C3 > gpurun_out/def42_bench.log 2>&1; echo bench $?
