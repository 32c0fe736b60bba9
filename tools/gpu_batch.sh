#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "batched or small_graphs or random_small or hub or star or cfg1 or kronecker_reduced or errors or device or lattice_partitions or cfg2" > gpurun_out/pytest_batch.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_batch.log
tail -2 gpurun_out/pytest_batch.log; grep -m2 -A25 "^____" gpurun_out/pytest_batch.log | head -40
timeout 600 python tools/tune.py --config 3 --sources 1024 --reps 1 --settings "order=1" 2>&1 | grep -v TRACE | cut -c1-90
timeout 600 python tools/tune.py --config 2 --sources 1024 --reps 1 --settings "order=1" 2>&1 | grep -v TRACE | cut -c1-90
timeout 600 python tools/tune.py --config 6 --sources 4096 --reps 1 --settings "order=1" 2>&1 | grep -v TRACE | cut -c1-90
timeout 600 python tools/tune.py --config 5 --sources 256 --reps 1 --settings "order=1" 2>&1 | grep -v TRACE | cut -c1-90
