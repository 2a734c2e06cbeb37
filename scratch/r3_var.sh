# dev variant (D=10 only): TC parity checks + C3 per-iteration timings + prof build
export EGGSYNC_LIB=/root/repo/scratch/variants/lib_d10.so
EGGSYNC_TC_DEBUG=1 BIG=1 timeout 300 python scratch/tc2check.py > gpurun_out/var_check.log 2>&1; echo check $?
timeout 200 python scratch/iterbench.py C3 3 > gpurun_out/var_iter.log 2>&1; echo iter $?
[ -n "$PROF" ] && EGGSYNC_LIB=/root/repo/scratch/variants/lib_d10p.so timeout 120 python scratch/iterbench.py C3 1 > gpurun_out/var_prof.log 2>&1; echo prof $?
