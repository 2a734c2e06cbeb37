for tc in 1 0; do for cfg in C3 C2 C4-d10 C4-d5; do EGGSYNC_TC=$tc timeout 300 python scratch/iterbench.py $cfg 2; done; done > gpurun_out/iter.log 2>&1
EGGSYNC_TC_DEBUG=1 EGGSYNC_TC_PROF=1 timeout 300 python scratch/iterbench.py C3 1 > gpurun_out/iter_dbg.log 2>&1
