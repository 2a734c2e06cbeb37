timeout 1200 python -m pytest tests/test_gpu_paths.py -k dense -x -q > gpurun_out/dense_tests.log 2>&1; echo tests $?
timeout 900 python scratch/densebench.py C1 C4-d2 C5 > gpurun_out/dense_bench.log 2>&1; echo bench $?
