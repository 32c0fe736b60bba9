#!/bin/bash
# Round-2 final measurement (session 2): traffic of the bench launch, bench lines of every config,
# the launch list of the default bench command, one ncu --set full capture of k_bcb (cfg 3, 256 sources)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python tools/measure_traffic.py --config 3 > gpurun_out/f2_traffic_c3.log 2>&1; echo "traffic rc=$?"; tail -2 gpurun_out/f2_traffic_c3.log
cp profiles/traffic_cfg3_*.json gpurun_out/ 2>/dev/null
timeout 600 python bench.py > gpurun_out/f2_cfg3.json 2> gpurun_out/f2_cfg3.err; echo "bench cfg3 rc=$?"
timeout 600 python bench.py --config 3 --steps 5 --warmup 3 --one-format --no-cpu-baseline > gpurun_out/f2_cfg3_oneformat.json 2>&1
timeout 900 python bench.py --config 3 --steps 3 --warmup 3 --engine coot --no-cpu-baseline > gpurun_out/f2_cfg3_coot.json 2>&1
timeout 300 python bench.py --config 1 --steps 50 --warmup 5 > gpurun_out/f2_cfg1.json 2>&1
timeout 300 python bench.py --config 2 --steps 10 --warmup 3 > gpurun_out/f2_cfg2.json 2>&1
timeout 900 python bench.py --config 4 --steps 3 --warmup 3 > gpurun_out/f2_cfg4.json 2>&1
timeout 900 python bench.py --config 5 --steps 3 --warmup 3 > gpurun_out/f2_cfg5.json 2>&1
timeout 900 python bench.py --config 5 --steps 3 --warmup 3 --inplace 1 --no-cpu-baseline > gpurun_out/f2_cfg5_inplace.json 2>&1
timeout 900 python bench.py --config 5 --steps 3 --warmup 3 --inplace 1 --width 32 --no-cpu-baseline > gpurun_out/f2_cfg5_inplace_w32.json 2>&1
timeout 600 python bench.py --config 6 --steps 3 --warmup 3 --order 0 --no-cpu-baseline > gpurun_out/f2_cfg6.json 2>&1
timeout 600 python bench.py --config 7 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/f2_cfg7.json 2>&1
timeout 900 python bench.py --config 8 --steps 2 --warmup 3 > gpurun_out/f2_cfg8.json 2>&1
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/f2_cfg3_reference.json 2>&1
python tools/results_table.py gpurun_out/f2_cfg*.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/f2_launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/f2_launch_run.log 2>&1; echo "launch list rc=$?"
PROF_TAG=f2c3 bash tools/gpu_prof_bcb.sh; tail -1 gpurun_out/prof_f2c3.log
python tools/ncu_inst.py gpurun_out/prof_f2c3_source.csv 40 > gpurun_out/prof_f2c3_inst.txt 2>&1
python tools/ncu_stalls.py gpurun_out/prof_f2c3_source.csv > gpurun_out/prof_f2c3_stalls.txt 2>&1
rm -f gpurun_out/prof_f2c3.ncu-rep gpurun_out/prof_f2c3_source.csv
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f2_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/f2_smoke.log
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/f2_gputests.log 2>&1; echo "gpu tests rc=$? $(tail -1 gpurun_out/f2_gputests.log)"
