#!/bin/bash
mkdir -p gpurun_out
timeout 900 python bench.py --config 6 --steps 3 --warmup 3 > gpurun_out/bench_cfg6.json 2> gpurun_out/bench_cfg6.err; echo "rc=$?" >> gpurun_out/bench_cfg6.err
timeout 900 python bench.py --config 6 --steps 3 --warmup 3 --width 64 --no-cpu-baseline > gpurun_out/bench_cfg6_w64.json 2>> gpurun_out/bench_cfg6.err
timeout 1500 python bench.py --config 7 --steps 3 --warmup 3 > gpurun_out/bench_cfg7.json 2> gpurun_out/bench_cfg7.err; echo "rc=$?" >> gpurun_out/bench_cfg7.err
for f in gpurun_out/bench_cfg6.json gpurun_out/bench_cfg6_w64.json gpurun_out/bench_cfg7.json; do python -c "
import json,sys
d=json.loads(open('$f').read())
print('$f', round(d['value'],2), 'vs paper', round(d['vs_baseline'] or 0,2), 'ms/step', round(d['ms_per_step'],1), 'e2e', round(d['e2e']['value'],2), 'frac', round(d['roofline']['frac'],3), 'cpu', d['cpu_baseline'] and round(d['cpu_baseline']['value'],3))
" 2>&1 | tail -1; done
tail -3 gpurun_out/bench_cfg6.err gpurun_out/bench_cfg7.err
