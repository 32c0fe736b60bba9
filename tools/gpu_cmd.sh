timeout 1200 python -m pytest tests -m gpu -x -q --durations=5 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python tools/tune.py --config 3 --sources 256 --settings "fmt=0;dir=2,fmt=1;fmt=1" --trace 0,1 > gpurun_out/tune2.log 2>&1
tail -3 gpurun_out/pytest_gpu.log; grep -v TRACE gpurun_out/tune2.log
