set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
BIG=0 DIMS=2,5,10 timeout 600 python scratch/tccheck.py > gpurun_out/tccheck.log 2>&1; echo tccheck $?
timeout 300 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_tc.log 2>&1; echo bench $?
EGGSYNC_TC=0 timeout 300 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_simt.log 2>&1; echo bench0 $?
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo tests $?
tail -3 gpurun_out/*.log
