#!/bin/bash
# Final round measurement: default bench line (cfg 3), the ncu launch list of the same command, and one
# ncu --set full capture of k_bcb (cfg 3, 256 sources) with source-level stall sampling.
mkdir -p gpurun_out
timeout 400 python bench.py > gpurun_out/final_bench.log 2>&1; tail -1 gpurun_out/final_bench.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/final_launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/final_launch_run.log 2>&1; echo "launch list rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_bcb -s 1 -c 1 -f -o gpurun_out/final_prof \
  python tools/prof_run.py --config 3 --sources 256 > gpurun_out/final_prof.log 2>&1; echo "ncu full rc=$?"
ncu -i gpurun_out/final_prof.ncu-rep --page details --csv > gpurun_out/final_prof_details.csv 2>&1
ncu -i gpurun_out/final_prof.ncu-rep --page raw --csv > gpurun_out/final_prof_raw.csv 2>&1
ncu -i gpurun_out/final_prof.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/final_prof_source.csv 2>&1
rm -f gpurun_out/final_prof.ncu-rep
ls -la gpurun_out
