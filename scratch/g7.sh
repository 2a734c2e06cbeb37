EGGSYNC_TC_DEBUG=1 timeout 90 python scratch/iterbench.py C4-d10 1 > gpurun_out/c4dbg.log 2>&1
EGGSYNC_TC=0 timeout 90 python scratch/iterbench.py C4-d10 1 >> gpurun_out/c4dbg.log 2>&1
EGGSYNC_LIB=/root/repo/scratch/variants/dr4/libeggsync.so timeout 90 python scratch/iterbench.py C3 2 > gpurun_out/dr4.log 2>&1
EGGSYNC_LIB=/root/repo/scratch/variants/dr4/libeggsync.so BIG=0 DIMS=2,5,10 timeout 120 python scratch/tccheck.py >> gpurun_out/dr4.log 2>&1
