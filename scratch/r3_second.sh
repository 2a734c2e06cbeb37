timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_oracle_pins.py tests/test_gpu_full_parity.py tests/test_gpu_cw_factor.py -m gpu -q -k "not C3" > gpurun_out/r3_tests.log 2>&1; echo tests $?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_second" -c 20 --csv --log-file gpurun_out/second.csv python scratch/tcprof.py C3 > /dev/null 2>&1; echo ncu $?
