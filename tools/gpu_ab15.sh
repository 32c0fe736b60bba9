#!/bin/bash
mkdir -p gpurun_out
TBC_VARIANT="-DTBC_OTILE_PF=1" timeout 600 python -m pytest tests/test_gpu_full.py tests/test_gpu_parity.py -m gpu -x -q -k "bfs_batch_small or overflow or cfg3_full or batched or random_small or closed or hub" > gpurun_out/ab15_tests.log 2>&1
echo "otile_pf tests rc=$? $(tail -1 gpurun_out/ab15_tests.log)"
AB_VARIANTS="|-DTBC_OTILE_PF=1|-DTBC_BUNROLL64=10|-DTBC_BUNROLL64=12|-DTBC_STATIC_PCT=40|-DTBC_STATIC_PCT=80" AB_CONFIGS="3|5" AB_REPS=2 AB_STEPS=3 bash tools/gpu_ab.sh
for b in 1 2; do timeout 300 python bench.py --config 1 --steps 50 --warmup 5 --batch $b --no-cpu-baseline > gpurun_out/ab15_c1_b$b.json 2>&1; python tools/bline.py gpurun_out/ab15_c1_b$b.json | cut -c1-200; done
