# full GPU suite + smoke + bench on the in-tree library
timeout 1500 python -m pytest tests -m gpu -x -q -k "not C3" > gpurun_out/r2_tests.log 2>&1; echo tests $?
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2_smoke.log 2>&1; echo smoke $?
timeout 600 python bench.py > gpurun_out/r2_bench.log 2>&1; echo bench $?
