set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_full.py -x -q 2>&1 | tail -15 > gpurun_out/t_full.log
timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench3.log 2>&1
tail -c 1500 gpurun_out/bench3.log
cat gpurun_out/t_full.log
