#!/bin/bash
# A/B of the gathers-in-flight unroll (TBC_BUNROLL) on cfg 3 / cfg 5 / cfg 2, alternating variants.
for cfg in 3 5 2; do
  for rep in 1 2; do
    for v in "" "-DTBC_BUNROLL=4" "-DTBC_BUNROLL=8"; do
      r=$(TBC_VARIANT="$v" timeout 300 python bench.py --config $cfg --steps 3 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 |
          python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), d['roofline']['frac'].__round__(3), d['clocks']['sm_mhz'])")
      echo "cfg$cfg rep$rep variant='$v' -> $r"
    done
  done
done
