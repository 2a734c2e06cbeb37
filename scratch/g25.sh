timeout 700 python -m pytest tests -m gpu -q > gpurun_out/g25_tests.log 2>&1; echo tests $?
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g25_smoke.log 2>&1; echo smoke $?
timeout 200 python scratch/def42bench.py C1 C2 > gpurun_out/g25_def42.log 2>&1; echo def42 $?
