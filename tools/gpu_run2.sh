set -x
timeout 900 python -m pytest tests/test_gpu_full.py -x -q 2>&1 | tail -15 > gpurun_out/t_full.log
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "not cfg4 and not cfg5" 2>&1 | tail -15 > gpurun_out/t_par.log
for c in 4 1 2 3; do timeout 300 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_c$c.log 2>&1; done
cat gpurun_out/t_full.log gpurun_out/t_par.log
for c in 4 1 2 3; do python -c "
import json,sys
for l in open('gpurun_out/bench_c$c.log'):
    if l.startswith('{'):
        d=json.loads(l); print($c, round(d['value'],2), d['ms_per_step'], d['config']['engine_mode'], d['config'].get('engine_choice'), round(d['roofline']['frac'],3))
" ; tail -2 gpurun_out/bench_c$c.log | cut -c1-300; done
