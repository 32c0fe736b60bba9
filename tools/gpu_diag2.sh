#!/bin/bash
# region profile (TBC_PROF build) + per-level trace of one batch on cfg 3; pair counts per pass kind
mkdir -p gpurun_out
TBC_VARIANT="-DTBC_PROF" timeout 900 python tools/tune.py --config 3 --sources 1024 --settings "width=64" --trace 640 > gpurun_out/d2_prof_c3.log 2>&1
echo "prof rc=$?"; grep -v TRACE gpurun_out/d2_prof_c3.log | tail -5
python tools/trace_summary.py 40 < gpurun_out/d2_prof_c3.log | head -60
