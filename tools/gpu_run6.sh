timeout 900 python tools/measure_traffic.py --config 3 > gpurun_out/traffic_c3.log 2>&1
timeout 900 python tools/measure_traffic.py --config 4 > gpurun_out/traffic_c4.log 2>&1
cp profiles/traffic_cfg*.json gpurun_out/ 2>/dev/null
timeout 400 python bench.py --config 3 --steps 5 --warmup 3 > gpurun_out/bench_c3.log 2>&1
timeout 600 python bench.py --config 3 --engine coot --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/bench_c3_coot.log 2>&1
timeout 600 python bench.py --config 4 --steps 3 --warmup 3 > gpurun_out/bench_c4.log 2>&1
tail -c 600 gpurun_out/traffic_c3.log; tail -c 300 gpurun_out/traffic_c4.log
for f in bench_c3 bench_c3_coot bench_c4; do python tools/bline.py gpurun_out/$f.log; done
