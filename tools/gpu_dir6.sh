#!/bin/bash
# direction study on cfg 3: pull ratio sweep, width 32, one-format (pull forward + push backward) trace
mkdir -p gpurun_out
timeout 900 python tools/tune.py --config 3 --sources 1024 --settings "bpull=8;bpull=0;bpull=2;bpull=4;bpull=16;bpull=64;width=32" > gpurun_out/d6_dir.log 2>&1; grep -v TRACE gpurun_out/d6_dir.log
TUNE_ONE_FORMAT=1 timeout 900 python tools/tune.py --config 3 --sources 1024 --settings "bpull=8" --trace 640 > gpurun_out/d6_of.log 2>&1; grep -v TRACE gpurun_out/d6_of.log | tail -3
python tools/trace_summary.py < gpurun_out/d6_of.log
timeout 900 python tools/tune.py --config 3 --sources 1024 --settings "bpull=8" --trace 640 > gpurun_out/d6_def.log 2>&1
python tools/trace_summary.py < gpurun_out/d6_def.log
