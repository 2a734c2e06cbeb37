BIG=0 DIMS=2,10 timeout 120 python scratch/tccheck.py > gpurun_out/v_ns3.log 2>&1
EGGSYNC_LIB=/root/repo/scratch/variants/ns2/libeggsync.so BIG=0 DIMS=2,10 timeout 120 python scratch/tccheck.py > gpurun_out/v_ns2.log 2>&1
