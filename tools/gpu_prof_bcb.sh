#!/bin/bash
# source-level ncu --set full of the second k_bcb launch (PROF_CONFIG, PROF_SOURCES sources)
mkdir -p gpurun_out
TAG=${PROF_TAG:-bcb}
timeout 1500 ncu --set full --import-source on --clock-control none --kernel-name-base function -k regex:^k_bcb$ -s 1 -c 1 -f -o gpurun_out/prof_$TAG python tools/prof_run.py --config ${PROF_CONFIG:-3} --sources ${PROF_SOURCES:-256} ${PROF_ARGS} > gpurun_out/prof_$TAG.log 2>&1
echo "ncu rc=$?" >> gpurun_out/prof_$TAG.log
ncu -i gpurun_out/prof_$TAG.ncu-rep --page raw --csv > gpurun_out/prof_${TAG}_raw.csv 2>&1
ncu -i gpurun_out/prof_$TAG.ncu-rep --page details --csv > gpurun_out/prof_${TAG}_details.csv 2>&1
ncu -i gpurun_out/prof_$TAG.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/prof_${TAG}_source.csv 2>&1
