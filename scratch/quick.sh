# dev loop on the GPU box: small parity, per-iteration timings, GPU test suite
BIG=0 DIMS=${DIMS:-2,5,10} timeout 150 python scratch/tccheck.py > gpurun_out/q_tccheck.log 2>&1; echo tccheck $?
for cfg in ${CFGS:-C3 C4-d10 C2}; do timeout 90 python scratch/iterbench.py $cfg 2; done > gpurun_out/q_iter.log 2>&1; echo iter $?
if [ "${TESTS:-1}" = 1 ]; then timeout 400 python -m pytest tests -m gpu -x -q > gpurun_out/q_tests.log 2>&1; echo tests $?; fi
if [ "${PROF:-0}" = 1 ]; then EGGSYNC_TC_DEBUG=1 EGGSYNC_TC_PROF=1 timeout 90 python scratch/iterbench.py C3 1 > gpurun_out/q_prof.log 2>&1; fi
if [ "${LAUNCH:-0}" = 1 ]; then timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/q_launch.csv python scratch/tcprof.py C3 > /dev/null 2>&1; fi
