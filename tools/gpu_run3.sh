timeout 900 python -m pytest tests/test_gpu_full.py -x -q -k "narrow or auto or bfs_batch or cfg4" 2>&1 | tail -5 > gpurun_out/t_full.log
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "not cfg5" 2>&1 | tail -5 > gpurun_out/t_par.log
for c in 4 1; do timeout 300 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_c$c.log 2>&1; done
timeout 600 ncu --set full --import-source on --kernel-name-base function -k k_bcs --launch-skip 1 --launch-count 1 -o gpurun_out/k_bcs_cfg4 python bench.py --config 4 --sources 200 --steps 1 --warmup 0 --no-cpu-baseline > gpurun_out/ncu_c4.log 2>&1
cat gpurun_out/t_full.log gpurun_out/t_par.log
for c in 4 1; do python tools/bline.py gpurun_out/bench_c$c.log; done
tail -3 gpurun_out/ncu_c4.log
