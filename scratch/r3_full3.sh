timeout 1800 python -m pytest tests -m gpu -q -k "not C3" > gpurun_out/r3_tests.log 2>&1; echo tests $?
timeout 600 python bench.py > gpurun_out/r3_bench.log 2>&1; echo bench $?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_second" -c 20 --csv --log-file gpurun_out/second.csv python scratch/tcprof.py C3 > /dev/null 2>&1; echo ncu $?
