#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "batched or small_graphs or random_small or hub or star or cfg1 or kronecker_reduced or errors or device" > gpurun_out/pytest_batch.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_batch.log
tail -3 gpurun_out/pytest_batch.log; grep -m3 -A30 "^____" gpurun_out/pytest_batch.log | head -50
for w in 32 64; do
  timeout 600 python tools/tune.py --config 3 --sources 512 --reps 1 --settings "batch=1,width=$w" 2>&1 | grep -v TRACE | tail -2 | cut -c1-100
  timeout 600 python tools/tune.py --config 2 --sources 1024 --reps 1 --settings "batch=1,width=$w" 2>&1 | grep -v TRACE | tail -2 | cut -c1-100
done
