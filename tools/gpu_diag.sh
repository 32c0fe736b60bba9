#!/bin/bash
mkdir -p gpurun_out
( timeout 300 python tools/diag_parts.py --parts 1,2,3,8 --reps 5
  timeout 300 python tools/diag_parts.py --parts 1,8 --reps 3 --scale 15 --k 64 ) > gpurun_out/diag.log 2>&1
cut -c1-200 gpurun_out/diag.log | grep -v "bad=\[0, 0, 0" | head -40
