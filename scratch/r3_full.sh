# full GPU suite + smoke + bench on the in-tree library
timeout 1500 python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/r3_tests.log 2>&1; echo tests $?
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r3_smoke.log 2>&1; echo smoke $?
timeout 600 python bench.py > gpurun_out/r3_bench.log 2>&1; echo bench $?
