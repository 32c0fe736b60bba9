#!/bin/bash
# source-level ncu of k_bcb on cfg 3 (256 sources) + prefetch A/B
mkdir -p gpurun_out
PROF_TAG=c3 bash tools/gpu_prof_bcb.sh; tail -1 gpurun_out/prof_c3.log
python tools/ncu_inst.py gpurun_out/prof_c3_source.csv 45 > gpurun_out/prof_c3_inst.txt 2>&1; head -50 gpurun_out/prof_c3_inst.txt
python tools/ncu_stalls.py gpurun_out/prof_c3_source.csv > gpurun_out/prof_c3_stalls.txt 2>&1; head -40 gpurun_out/prof_c3_stalls.txt
rm -f gpurun_out/prof_c3.ncu-rep
AB_VARIANTS="|-DTBC_DYN_PREFETCH=1" AB_CONFIGS="3" AB_REPS=2 AB_STEPS=3 bash tools/gpu_ab.sh
