timeout 500 python -m pytest tests -m gpu -x -q > gpurun_out/g11_tests.log 2>&1; echo tests $?
timeout 120 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/g11_smoke.log 2>&1; echo smoke $?
timeout 300 python bench.py > gpurun_out/g11_bench.log 2>&1; echo bench $?
for cfg in C3 C4-d10 C2 C1; do timeout 90 python scratch/iterbench.py $cfg 2; done > gpurun_out/g11_iter.log 2>&1; echo iter $?
