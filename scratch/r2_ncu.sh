# one full ncu capture of the iteration-1 k_update_tc launch of a C3 clustering (dev lib)
export EGGSYNC_LIB=${EGGSYNC_LIB:-/root/repo/scratch/variants/lib_d10.so}
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_update_tc -c 1 -o gpurun_out/ncu_tc_dev -f python scratch/tcprof.py C3 > gpurun_out/ncu_tc_dev.log 2>&1
echo ncu $?
