timeout 300 python scratch/iterbench.py C5 1 > gpurun_out/c5.log 2>&1; echo tc $?
TESTS=1 CFGS="C3 C4-d10 C2" bash scratch/quick.sh
