#!/bin/bash
mkdir -p gpurun_out
TBC_VARIANT="-DTBC_DEFER_CLAIM=1" timeout 900 python -m pytest tests/test_gpu_full.py tests/test_gpu_parity.py -m gpu -x -q -k "bfs_batch_small or bfs_batch_kronecker or overflow or cfg3_full or cfg2_full or batched or random_small or closed or hub" > gpurun_out/ab8_tests.log 2>&1
echo "defer tests rc=$? $(tail -1 gpurun_out/ab8_tests.log)"
AB_VARIANTS="|-DTBC_DEFER_CLAIM=1|-DTBC_EXP_NOGATHER=1" AB_CONFIGS="3|2" AB_REPS=2 AB_STEPS=3 bash tools/gpu_ab.sh
for v in "" "-DTBC_EXP_NOGATHER=1"; do
TBC_VARIANT="$v" timeout 900 python tools/tune.py --config 3 --sources 1024 --settings "bpull=8" --trace 640 > gpurun_out/d8.log 2>&1
echo "variant '$v'"; grep -v TRACE gpurun_out/d8.log | tail -1 | cut -c1-120; python tools/trace_summary.py < gpurun_out/d8.log
done
