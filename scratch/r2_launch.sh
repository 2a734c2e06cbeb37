timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2_launch.csv python scratch/tcprof.py C3 > /dev/null 2>&1; echo launch $?
