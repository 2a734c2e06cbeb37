timeout 1800 python -m pytest tests -m gpu -q -k "not C3" > gpurun_out/r3_tests.log 2>&1; echo tests $?
timeout 600 python scratch/def42bench.py C1 C2 C4-d10 C3 > gpurun_out/def42_bench.log 2>&1; echo bench $?
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r3_smoke.log 2>&1; echo smoke $?
