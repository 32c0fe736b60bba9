#!/bin/bash
# A/B of the batch width (auto vs forced 32 / 64) after the W = 64 unroll change.
run() {
  timeout 400 python bench.py --config $1 $2 --steps 3 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 |
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['config'].get('engine_mode'))"
}
for cfg in 5 4; do
  for rep in 1 2; do
    for w in "" "--width 64"; do echo "cfg$cfg rep$rep '$w' -> $(run $cfg "$w")"; done
  done
done
