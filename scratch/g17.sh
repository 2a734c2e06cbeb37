for tc in 0 1; do EGGSYNC_TC=$tc timeout 120 python scratch/iterbench.py C3 2; done > gpurun_out/g17_iter.log 2>&1; echo iter $?
for tc in 0 1; do EGGSYNC_TC=$tc timeout 120 python scratch/iterbench.py C4-d10 2; done >> gpurun_out/g17_iter.log 2>&1; echo iter $?
