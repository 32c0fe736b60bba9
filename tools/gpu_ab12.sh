#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_full.py tests/test_gpu_parity.py -m gpu -x -q -k "bfs_batch_small or bfs_batch_kronecker or overflow or one_format or cfg3_full or cfg2_full or batched or random_small or closed or hub" > gpurun_out/ab12_tests.log 2>&1
echo "quick tests rc=$? $(tail -1 gpurun_out/ab12_tests.log)"; grep -m5 -E "^E |FAILED" gpurun_out/ab12_tests.log
AB_VARIANTS="|LIB:paper_conf_icppw_artiless21_b200/libturbobc_base.so" AB_CONFIGS="3|2|5" AB_REPS=1 AB_STEPS=3 bash tools/gpu_ab.sh
timeout 300 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/ab12_c3.json 2>&1; python -c "
import json; d=[json.loads(l) for l in open('gpurun_out/ab12_c3.json') if l.startswith('{')][-1]; print(d['value'], d['traversal'], d['setup'])"
