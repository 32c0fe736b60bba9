#!/bin/bash
# ncu --set full of the main k_bcs launch (PROF_CONFIG, PROF_SOURCES sources, narrow engine forced)
TAG=${PROF_TAG:-bcs}
timeout 1500 ncu --set full --import-source on --clock-control none --kernel-name-base function -k regex:^k_bcs$ -s 1 -c 1 -f -o gpurun_out/prof_$TAG python tools/prof_run.py --config ${PROF_CONFIG:-4} --sources ${PROF_SOURCES:-148} --settings batch=2 > gpurun_out/prof_$TAG.log 2>&1
echo "ncu rc=$?" >> gpurun_out/prof_$TAG.log
ncu -i gpurun_out/prof_$TAG.ncu-rep --page details --csv > gpurun_out/prof_${TAG}_details.csv 2>&1
ncu -i gpurun_out/prof_$TAG.ncu-rep --page raw --csv > gpurun_out/prof_${TAG}_raw.csv 2>&1
ncu -i gpurun_out/prof_$TAG.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/prof_${TAG}_source.csv 2>&1
