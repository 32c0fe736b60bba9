python -c "from paper_conf_icppw_artiless21_b200 import build as b; b.build(variant='-DTBC_LANE_ITEMS=4'); b.build(variant='-DTBC_LANE_ITEMS=16')" 
timeout 900 python tools/tune.py --config 3 --sources 512 --reps 1 --settings "list=12;list=16;list=20;list=24;list=20,stream=3;list=20,bpush=3;list=20,bpush=10;list=20,atomic=30;list=20,scan=6" > gpurun_out/tune6.log 2>&1
TBC_VARIANT=-DTBC_LANE_ITEMS=4 timeout 600 python tools/tune.py --config 3 --sources 512 --reps 1 --settings "list=12;list=20" > gpurun_out/tune6b.log 2>&1
TBC_VARIANT=-DTBC_LANE_ITEMS=16 timeout 600 python tools/tune.py --config 3 --sources 512 --reps 1 --settings "list=12;list=20" > gpurun_out/tune6c.log 2>&1
cat gpurun_out/tune6.log gpurun_out/tune6b.log gpurun_out/tune6c.log | grep -v TRACE | cut -c1-120
