#!/bin/bash
# bench lines for every config (round 2); results under gpurun_out/r2b_*.json
timeout 900 python tools/measure_traffic.py --config 3 > gpurun_out/r2b_traffic_c3.log 2>&1
cp profiles/traffic_cfg3_csc_k4096_e1_w64.json gpurun_out/ 2>/dev/null
timeout 600 python bench.py --config 3 --steps 10 --warmup 3 > gpurun_out/r2b_cfg3.json 2>gpurun_out/r2b_cfg3.err
timeout 600 python bench.py --config 3 --steps 5 --warmup 3 --one-format --no-cpu-baseline > gpurun_out/r2b_cfg3_oneformat.json 2>&1
timeout 300 python bench.py --config 1 --steps 20 --warmup 5 > gpurun_out/r2b_cfg1.json 2>&1
timeout 300 python bench.py --config 2 --steps 10 --warmup 3 > gpurun_out/r2b_cfg2.json 2>&1
timeout 900 python bench.py --config 4 --steps 3 --warmup 3 > gpurun_out/r2b_cfg4.json 2>&1
timeout 900 python bench.py --config 5 --steps 2 --warmup 3 > gpurun_out/r2b_cfg5.json 2>&1
timeout 600 python bench.py --config 6 --steps 3 --warmup 3 --order 0 --no-cpu-baseline > gpurun_out/r2b_cfg6.json 2>&1
timeout 600 python bench.py --config 7 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/r2b_cfg7.json 2>&1
timeout 900 python bench.py --config 8 --steps 2 --warmup 3 > gpurun_out/r2b_cfg8.json 2>&1
timeout 600 python bench.py --impl reference --config 3 --steps 2 --warmup 3 > gpurun_out/r2b_cfg3_reference.json 2>&1
for f in gpurun_out/r2b_cfg*.json; do python tools/bline.py $f; done
