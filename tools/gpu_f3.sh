#!/bin/bash
mkdir -p gpurun_out
timeout 900 python bench.py --config 8 --steps 2 --warmup 3 > gpurun_out/f3_cfg8.json 2>&1; echo "cfg8 rc=$?"; tail -1 gpurun_out/f3_cfg8.json | cut -c1-300
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 5000 --csv --log-file gpurun_out/f3_launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/f3_launch_run.log 2>&1; echo "launch list rc=$?"
grep -c k_bcb gpurun_out/f3_launches.csv
