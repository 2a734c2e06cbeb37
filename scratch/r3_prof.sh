# per-role cycle accounting (EGG_TC_PROF build) + one full ncu capture of the iteration-1 k_update_tc launch of C3 (HEAD lib)
EGGSYNC_LIB=/root/repo/scratch/variants/lib_d10p.so timeout 200 python scratch/iterbench.py C3 1 > gpurun_out/r3_prof.log 2>&1; echo prof $?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_update_tc -c 1 -o gpurun_out/ncu_tc_r3a -f python scratch/tcprof.py C3 > gpurun_out/ncu_tc_r3a.log 2>&1; echo ncu $?
