#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python bench.py --config 5 --steps 3 --warmup 3 > gpurun_out/bench_cfg5.json 2> gpurun_out/bench_cfg5.err; echo "cfg5 rc=$?"
timeout 900 python bench.py --config 2 --steps 5 --warmup 3 > gpurun_out/bench_cfg2.json 2> gpurun_out/bench_cfg2.err; echo "cfg2 rc=$?"
timeout 900 python bench.py --config 6 --steps 3 --warmup 3 > gpurun_out/bench_cfg6.json 2> gpurun_out/bench_cfg6.err; echo "cfg6 rc=$?"
timeout 1500 python bench.py --config 7 --steps 3 --warmup 3 > gpurun_out/bench_cfg7.json 2> gpurun_out/bench_cfg7.err; echo "cfg7 rc=$?"
for f in gpurun_out/bench_cfg5.json gpurun_out/bench_cfg2.json gpurun_out/bench_cfg6.json gpurun_out/bench_cfg7.json; do python -c "
import json
d=json.loads(open('$f').read())
print('$f', round(d['value'],3), d['config'].get('engine_mode'), 'ms/step', round(d['ms_per_step'],1), 'e2e', round(d['e2e']['value'],3), 'frac', d.get('roofline',{}).get('frac'), 'cpu', d['cpu_baseline'] and round(d['cpu_baseline']['value'],3), 'vs', d['vs_baseline'])
"; done
