#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_full.py tests/test_gpu_parity.py -m gpu -x -q -k "inplace or bfs_batch_small or overflow or one_format or cfg2_full or cfg3_full or batched or random_small or closed or hub" > gpurun_out/ab14_tests.log 2>&1
echo "tests rc=$? $(tail -1 gpurun_out/ab14_tests.log)"; grep -m5 -E "^E |FAILED" gpurun_out/ab14_tests.log
AB_VARIANTS="|LIB:paper_conf_icppw_artiless21_b200/libturbobc_base.so" AB_CONFIGS="3|2|5" AB_REPS=1 AB_STEPS=3 bash tools/gpu_ab.sh
for c in 3 5; do
timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline --inplace 1 > gpurun_out/ab14_c${c}_ip.json 2>&1; python -c "
import json; d=[json.loads(l) for l in open('gpurun_out/ab14_c${c}_ip.json') if l.startswith('{')][-1]; print('cfg$c inplace', round(d['value'],1), 'ovf', d['traversal']['list_overflows'], 'ws GB', d['setup']['workspace_bytes']/1e9)"
done
timeout 900 python -m pytest tests/test_gpu_full.py -m gpu -x -q -k "cfg5_rank0" > gpurun_out/ab14_c5fix.log 2>&1; echo "cfg5 fixture rc=$? $(tail -1 gpurun_out/ab14_c5fix.log)"
