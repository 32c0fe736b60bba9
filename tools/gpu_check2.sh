#!/bin/bash
# session re-check: gpu tests, smoke, default bench line
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c2_build.log 2>&1; echo "build rc=$?"
timeout 1800 python -m pytest tests -m gpu -x -q --durations=25 > gpurun_out/c2_gputests.log 2>&1; echo "gpu tests rc=$?"; tail -30 gpurun_out/c2_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c2_smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/c2_smoke.log
timeout 400 python bench.py > gpurun_out/c2_bench.json 2> gpurun_out/c2_bench.err; echo "bench rc=$?"; tail -1 gpurun_out/c2_bench.json
