timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python tools/tune.py --config 3 --sources 512 --settings "parts=8;parts=4" --trace 0 > gpurun_out/tune9.log 2>&1
tail -2 gpurun_out/pytest_gpu.log; grep -v TRACE gpurun_out/tune9.log | cut -c1-150
