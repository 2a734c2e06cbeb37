for v in pw4 pw1 pw2 pw8 pw4; do EGGSYNC_LIB=scratch/variants/lib_$v.so CFG=C3 timeout 120 python scratch/varbench.py; done > gpurun_out/g27.log 2>&1; echo var $?
for v in pw4 pw2 pw8; do EGGSYNC_LIB=scratch/variants/lib_$v.so CFG=C4-d10 timeout 120 python scratch/varbench.py; done >> gpurun_out/g27.log 2>&1; echo var $?
