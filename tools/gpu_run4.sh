timeout 1200 python -m pytest tests/test_gpu_full.py -x -q -k "cfg3 or cfg2" 2>&1 | tail -5 > gpurun_out/t_full.log
PROF_TAG=bcb_c3 bash tools/gpu_prof_bcb.sh
cat gpurun_out/t_full.log; tail -2 gpurun_out/prof_bcb_c3.log
