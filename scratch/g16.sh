timeout 300 python bench.py > gpurun_out/g16_bench.log 2>&1; echo bench $?
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/g16_launch.csv python bench.py --steps 1 --warmup 3 --no-cpu --no-e2e > gpurun_out/g16_ncu_bench.log 2>&1; echo ncu $?
timeout 200 python scratch/stagebench.py > gpurun_out/g16_stages.log 2>&1; echo stages $?
