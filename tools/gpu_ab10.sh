#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "random_small" > gpurun_out/ab10_t1.log 2>&1
rc=$?; echo "random_small rc=$rc $(tail -1 gpurun_out/ab10_t1.log)"
if [ $rc -ne 0 ]; then
  TBC_VARIANT="-DTBC_WATCHDOG_S=600" timeout 900 compute-sanitizer --tool memcheck --print-limit 10 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "random_small_graphs_many and False" > gpurun_out/ab10_mc.log 2>&1
  grep -m30 -E "Invalid|at 0x|by thread|Address|ERROR SUMMARY|tbc_batch" gpurun_out/ab10_mc.log
  exit 1
fi
timeout 600 python -m pytest tests/test_gpu_full.py tests/test_gpu_parity.py -m gpu -x -q -k "bfs_batch_small or bfs_batch_kronecker or overflow or one_format or cfg3_full or cfg2_full or batched or closed or hub" > gpurun_out/ab10_tests.log 2>&1
echo "quick tests rc=$? $(tail -1 gpurun_out/ab10_tests.log)"; grep -m5 -E "^E |FAILED" gpurun_out/ab10_tests.log
AB_VARIANTS="|LIB:paper_conf_icppw_artiless21_b200/libturbobc_base.so" AB_CONFIGS="3|2|5" AB_REPS=2 AB_STEPS=3 bash tools/gpu_ab.sh
