# dev loop on the GPU box: small parity, per-iteration timings, GPU test suite
BIG=0 DIMS=${DIMS:-2,5,10} timeout 600 python scratch/tccheck.py > gpurun_out/q_tccheck.log 2>&1; echo tccheck $?
for cfg in ${CFGS:-C3 C4-d10 C2}; do timeout 300 python scratch/iterbench.py $cfg 2; done > gpurun_out/q_iter.log 2>&1; echo iter $?
if [ "${TESTS:-1}" = 1 ]; then timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/q_tests.log 2>&1; echo tests $?; fi
