export EGGSYNC_LIB=/root/repo/scratch/variants/lib_d10.so
for la in 1 2 3 4; do EGGSYNC_TC_LA=$la timeout 100 python scratch/iterbench.py C3 2 | tail -1 | sed "s/^/LA=$la /"; done > gpurun_out/dev_la.log 2>&1
EGGSYNC_TC_LA=2 EGGSYNC_LIB=/root/repo/scratch/variants/lib_d10p.so timeout 120 python scratch/iterbench.py C3 1 > gpurun_out/dev_prof.log 2>&1
