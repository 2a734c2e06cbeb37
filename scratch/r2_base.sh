# round-2 baseline on a fresh box: per-iteration times, tc producer/classifier breakdown, bench line
for cfg in C3 C4-d10 C2 C1; do timeout 120 python scratch/iterbench.py $cfg 2; done > gpurun_out/r2b_iter.log 2>&1; echo iter $?
EGGSYNC_TC_DEBUG=1 EGGSYNC_TC_PROF=1 timeout 120 python scratch/iterbench.py C3 1 > gpurun_out/r2b_prof.log 2>&1; echo prof $?
timeout 600 python bench.py > gpurun_out/r2b_bench.log 2>&1; echo bench $?
