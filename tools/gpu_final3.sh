#!/bin/bash
# final re-verification with the default static share 80 %: gpu tests, smoke, traffic, bench lines
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/f4_gputests.log 2>&1; echo "gpu tests rc=$? $(tail -1 gpurun_out/f4_gputests.log)"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f4_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/f4_smoke.log
timeout 900 python tools/measure_traffic.py --config 3 > gpurun_out/f4_traffic_c3.log 2>&1; echo "traffic rc=$?"
cp profiles/traffic_cfg3_*.json gpurun_out/ 2>/dev/null
timeout 600 python bench.py > gpurun_out/f4_cfg3.json 2> gpurun_out/f4_cfg3.err; echo "bench cfg3 rc=$?"
timeout 300 python bench.py --config 2 --steps 10 --warmup 3 > gpurun_out/f4_cfg2.json 2>&1
timeout 900 python bench.py --config 5 --steps 3 --warmup 3 > gpurun_out/f4_cfg5.json 2>&1
timeout 900 python bench.py --config 5 --steps 3 --warmup 3 --inplace 1 --no-cpu-baseline > gpurun_out/f4_cfg5_inplace.json 2>&1
timeout 900 python bench.py --config 5 --steps 3 --warmup 3 --inplace 1 --width 32 --no-cpu-baseline > gpurun_out/f4_cfg5_inplace_w32.json 2>&1
timeout 600 python bench.py --config 6 --steps 3 --warmup 3 --order 0 --no-cpu-baseline > gpurun_out/f4_cfg6.json 2>&1
timeout 600 python bench.py --config 7 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/f4_cfg7.json 2>&1
timeout 600 python bench.py --config 3 --steps 5 --warmup 3 --one-format --no-cpu-baseline > gpurun_out/f4_cfg3_oneformat.json 2>&1
python tools/results_table.py gpurun_out/f4_cfg*.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 5000 --csv --log-file gpurun_out/f4_launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/f4_launch_run.log 2>&1; echo "launch list rc=$?"
