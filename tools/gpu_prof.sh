#!/bin/bash
# ncu --set full of the second k_bc launch (16 sources of cfg3) with source-level stalls
mkdir -p gpurun_out
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:k_bc -s 1 -c 1 -f -o gpurun_out/prof_kbc python tools/prof_run.py --sources ${PROF_SOURCES:-64} ${PROF_ARGS} > gpurun_out/prof.log 2>&1
echo "ncu rc=$?" >> gpurun_out/prof.log
tail -3 gpurun_out/prof.log
