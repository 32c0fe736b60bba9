#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_full.py tests/test_gpu_parity.py -m gpu -x -q -k "bfs_batch_small or bfs_batch_kronecker or overflow or one_format or cfg3_full or cfg2_full or batched or random_small or closed or hub" > gpurun_out/ab9_tests.log 2>&1
echo "quick tests rc=$? $(tail -1 gpurun_out/ab9_tests.log)"; grep -m5 -E "^E |Error|FAILED" gpurun_out/ab9_tests.log
AB_VARIANTS="|LIB:paper_conf_icppw_artiless21_b200/libturbobc_base.so" AB_CONFIGS="3|2|5" AB_REPS=2 AB_STEPS=3 bash tools/gpu_ab.sh
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/ab9_full.log 2>&1; echo "full gpu tests rc=$? $(tail -1 gpurun_out/ab9_full.log)"; grep -m5 -E "^E |FAILED" gpurun_out/ab9_full.log
