#!/bin/bash
# walk variant: parity first, then A/B on cfg 3 / 2
mkdir -p gpurun_out
for v in "-DTBC_WALK=1" "-DTBC_WALK=1 -DTBC_BBLOCK=768"; do
  TBC_VARIANT="$v" timeout 900 python -m pytest tests/test_gpu_full.py tests/test_gpu_parity.py -m gpu -x -q -k "bfs_batch_small or bfs_batch_kronecker or overflow or one_format_directed or cfg3_full or batched or random_small or closed or hub" > gpurun_out/ab3_tests.log 2>&1
  echo "variant '$v' tests rc=$? $(tail -1 gpurun_out/ab3_tests.log)"; grep -m3 -E "Error|assert" gpurun_out/ab3_tests.log
done
AB_VARIANTS="|-DTBC_WALK=1|-DTBC_WALK=1 -DTBC_BBLOCK=768|-DTBC_BBLOCK=768|-DTBC_WALK=1 -DTBC_WALK_U=6" AB_CONFIGS="3|2" AB_REPS=2 AB_STEPS=3 bash tools/gpu_ab.sh
