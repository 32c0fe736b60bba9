#!/bin/bash
# One GPU pass: parity tests, bench line, ncu launch list of the bench command, ncu --set full of the hot kernel.
set -x
mkdir -p gpurun_out
nvidia-smi > gpurun_out/nvsmi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q --durations=15 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/bench_ncu.log 2>&1
[ -z "$NO_PROF" ] && PROF_SOURCES=128 bash tools/gpu_prof.sh
tail -3 gpurun_out/pytest_gpu.log; cat gpurun_out/bench.json
