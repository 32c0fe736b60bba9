#!/bin/bash
# A/B of the gathers-in-flight unroll of the W = 64 instantiation (TBC_BUNROLL64), alternating variants.
run() {  # cfg extra-args variant
  TBC_VARIANT="$3" timeout 300 python bench.py --config $1 $2 --steps 3 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 |
    python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), d['roofline']['frac'].__round__(3), d['clocks']['sm_mhz'])"
}
for spec in "3|" "2|" "6|--order 0" "7|"; do
  cfg=${spec%%|*}; extra=${spec#*|}
  for rep in 1 2; do
    for v in "" "-DTBC_BUNROLL64=10" "-DTBC_BUNROLL64=12"; do
      echo "cfg$cfg $extra rep$rep variant='$v' -> $(run $cfg "$extra" "$v")"
    done
  done
done
echo "cfg5 default -> $(run 5 '' '')"
