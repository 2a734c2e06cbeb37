timeout 300 python -m pytest tests/test_gpu_def42.py -x -q > gpurun_out/g15_def42.log 2>&1; echo def42 $?
timeout 600 python -m pytest tests -m gpu -q > gpurun_out/g15_tests.log 2>&1; echo tests $?
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g15_smoke.log 2>&1; echo smoke $?
