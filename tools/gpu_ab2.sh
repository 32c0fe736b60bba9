#!/bin/bash
# quick parity on the variants, then an alternating A/B on cfg 3 and cfg 2
mkdir -p gpurun_out
for v in "" "-DTBC_BKI=4"; do
  TBC_VARIANT="$v" timeout 600 python -m pytest tests/test_gpu_full.py -m gpu -x -q -k "bfs_batch_small or bfs_batch_kronecker or overflow or one_format_directed or cfg3_full" > gpurun_out/ab2_tests.log 2>&1
  echo "variant '$v' tests rc=$? $(tail -1 gpurun_out/ab2_tests.log)"
done
TBC_VARIANT="-DTBC_BKI=4" timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/ab2_tests2.log 2>&1; echo "bki4 parity rc=$? $(tail -1 gpurun_out/ab2_tests2.log)"
AB_VARIANTS="|-DTBC_DYN_PREFETCH=0|-DTBC_BKI=4|-DTBC_BKI=4 -DTBC_BUNROLL64=6" AB_CONFIGS="3|2" AB_REPS=2 AB_STEPS=3 bash tools/gpu_ab.sh
