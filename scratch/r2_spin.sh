for v in d10p d10s; do echo $v; EGGSYNC_LIB=/root/repo/scratch/variants/lib_$v.so timeout 120 python scratch/iterbench.py C3 1 2>&1 | grep -v "^\[tc\]"; done > gpurun_out/dev_spin.log 2>&1
