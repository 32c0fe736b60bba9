timeout 1500 python -m pytest tests/test_gpu_full.py tests/test_gpu_parity.py -x -q 2>&1 | tail -5 > gpurun_out/t_all.log
for c in 3 5 2; do timeout 400 python bench.py --config $c --steps 3 --warmup 2 --no-cpu-baseline > gpurun_out/bench_c$c.log 2>&1; done
cat gpurun_out/t_all.log
for c in 3 5 2; do python tools/bline.py gpurun_out/bench_c$c.log; grep -o '"list_peak[^,]*\|"device_bytes[^,]*\|"workspace_bytes[^}]*' gpurun_out/bench_c$c.log; tail -2 gpurun_out/bench_c$c.log | grep -i error; done
