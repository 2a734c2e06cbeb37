# parity + timing of dev variants: VARS="d10 d10g2" (lib_<v>.so), prof variants lib_<v>p.so
for v in ${VARS:-d10 d10g2}; do
  echo "== $v"
  EGGSYNC_LIB=/root/repo/scratch/variants/lib_$v.so BIG=1 timeout 300 python scratch/tc2check.py 2>&1 | grep -v "^\[tc"
  EGGSYNC_LIB=/root/repo/scratch/variants/lib_$v.so timeout 200 python scratch/iterbench.py C3 2 2>&1 | tail -1
  if [ -f scratch/variants/lib_${v}p.so ]; then EGGSYNC_LIB=/root/repo/scratch/variants/lib_${v}p.so timeout 120 python scratch/iterbench.py C3 1 2>&1 | grep "tc-prof" | head -2; fi
done > gpurun_out/dev_var.log 2>&1
