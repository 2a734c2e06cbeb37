timeout 700 python -m pytest tests -m gpu -q > gpurun_out/g21_tests.log 2>&1; echo tests $?
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g21_smoke.log 2>&1; echo smoke $?
