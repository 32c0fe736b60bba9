#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "batched or small_graphs or random_small or hub or star or cfg1 or kronecker_reduced or errors or device" > gpurun_out/pytest_batch.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_batch.log
tail -3 gpurun_out/pytest_batch.log
for v in "" "-DTBC_BUNROLL=6" "-DTBC_BUNROLL=8"; do
  echo "== variant $v"
  TBC_VARIANT="$v" timeout 600 python tools/tune.py --config 3 --sources 512 --reps 1 --settings "batch=1;batch=1,bpull=2;batch=1,bpull=32" 2>&1 | grep -v TRACE | tail -6 | cut -c1-100
done
