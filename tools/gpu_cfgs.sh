#!/bin/bash
mkdir -p gpurun_out
( for c in 1 2; do timeout 600 python tools/tune.py --config $c --sources 1024 --reps 2 --settings "batch=1;batch=0" 2>&1 | grep -v TRACE | cut -c1-160; done
  timeout 900 python tools/tune.py --config 4 --sources 64 --reps 1 --settings "batch=1;batch=0" 2>&1 | grep -v TRACE | cut -c1-160
) > gpurun_out/cfgs.log 2>&1
cat gpurun_out/cfgs.log
