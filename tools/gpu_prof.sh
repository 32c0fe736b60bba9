#!/bin/bash
# ncu --set full of the second k_bc launch (cfg3, PROF_SOURCES sources) with source-level stalls
mkdir -p gpurun_out
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:k_bc[b]? -s 1 -c 1 -f -o gpurun_out/prof_kbc python tools/prof_run.py --sources ${PROF_SOURCES:-64} ${PROF_ARGS} > gpurun_out/prof.log 2>&1
echo "ncu rc=$?" >> gpurun_out/prof.log
tail -3 gpurun_out/prof.log
ncu -i gpurun_out/prof_kbc.ncu-rep --page raw --csv > gpurun_out/prof_raw.csv 2>&1
ncu -i gpurun_out/prof_kbc.ncu-rep --page details --csv > gpurun_out/prof_details.csv 2>&1
ncu -i gpurun_out/prof_kbc.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/prof_source.csv 2>&1
ls -la gpurun_out/
