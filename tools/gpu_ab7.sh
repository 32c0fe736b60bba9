#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_full.py tests/test_gpu_parity.py -m gpu -x -q -k "bfs_batch_small or bfs_batch_kronecker or overflow or one_format_directed or cfg3_full or cfg2_full or batched or random_small or closed or hub" > gpurun_out/ab7_tests.log 2>&1
echo "default tests rc=$? $(tail -1 gpurun_out/ab7_tests.log)"
AB_VARIANTS="" AB_CONFIGS="3|2|5" AB_REPS=2 AB_STEPS=3 bash tools/gpu_ab.sh
timeout 900 python tools/tune.py --config 3 --sources 1024 --settings "bpull=8" --trace 640 > gpurun_out/d7_def.log 2>&1
python tools/trace_summary.py < gpurun_out/d7_def.log
