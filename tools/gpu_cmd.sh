timeout 1200 python -m pytest tests -m gpu -x -q --durations=5 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python tools/tune.py --config 3 --sources 512 --settings "parts=1;parts=2;parts=4;parts=8" --trace 0 > gpurun_out/tune3.log 2>&1
tail -3 gpurun_out/pytest_gpu.log; grep -v TRACE gpurun_out/tune3.log
