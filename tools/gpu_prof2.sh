#!/bin/bash
mkdir -p gpurun_out
for c in 2 6; do
  timeout 1200 ncu --set full --import-source on --clock-control none -k regex:k_bcb -s 1 -c 1 -f -o gpurun_out/prof_cfg$c python tools/prof_run.py --config $c --sources 256 > gpurun_out/prof_cfg$c.log 2>&1
  echo "cfg$c ncu rc=$?"
  ncu -i gpurun_out/prof_cfg$c.ncu-rep --page raw --csv > gpurun_out/prof_cfg${c}_raw.csv 2>&1
  ncu -i gpurun_out/prof_cfg$c.ncu-rep --page details --csv > gpurun_out/prof_cfg${c}_details.csv 2>&1
  ncu -i gpurun_out/prof_cfg$c.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/prof_cfg${c}_source.csv 2>&1
  rm -f gpurun_out/prof_cfg$c.ncu-rep
done
