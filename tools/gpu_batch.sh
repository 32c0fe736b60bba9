#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "batched or small_graphs or random_small or hub or star or cfg1 or kronecker_reduced or errors or device" > gpurun_out/pytest_batch.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_batch.log
tail -30 gpurun_out/pytest_batch.log
timeout 600 python tools/tune.py --config 3 --sources 512 --reps 1 --settings "batch=0;batch=1;batch=1,bpull=2;batch=1,bpull=32" 2>&1 | grep -v TRACE | tail -8
