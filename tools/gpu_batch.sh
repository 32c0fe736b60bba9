#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "batched or small_graphs or random_small or hub or star or cfg1 or kronecker_reduced or errors or device" > gpurun_out/pytest_batch.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_batch.log
tail -2 gpurun_out/pytest_batch.log
for v in "" "-DTBC_BCHUNK=0" "-DTBC_BSTATIC=0.5 -DTBC_BCHUNK=4" "-DTBC_BSTATIC=0.85 -DTBC_BCHUNK=1"; do
  echo "== $v"
  TBC_VARIANT="$v" timeout 600 python tools/tune.py --config 3 --sources 1024 --reps 1 --settings "bparts=0" 2>&1 | grep -v TRACE | cut -c1-90
  TBC_VARIANT="$v" timeout 600 python tools/tune.py --config 2 --sources 1024 --reps 1 --settings "bparts=0" 2>&1 | grep -v TRACE | cut -c1-90
done
echo "== HEAD"
TBC_LIB_PATH=$PWD/paper_conf_icppw_artiless21_b200/libturbobc_head.so timeout 600 python tools/tune.py --config 3 --sources 1024 --reps 1 --settings "bparts=0" 2>&1 | grep -v TRACE | cut -c1-90
TBC_LIB_PATH=$PWD/paper_conf_icppw_artiless21_b200/libturbobc_head.so timeout 600 python tools/tune.py --config 2 --sources 1024 --reps 1 --settings "bparts=0" 2>&1 | grep -v TRACE | cut -c1-90
