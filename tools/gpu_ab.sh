#!/bin/bash
# A/B of library variants (TBC_VARIANT -D flags, prebuilt in-tree), alternating, on configs.
#   AB_VARIANTS="|-DX=1|-DX=2"  AB_CONFIGS="3|2|5 --sources 256"  AB_REPS=2  bash tools/gpu_ab.sh
IFS='|' read -ra VARS <<< "${AB_VARIANTS:-}"
IFS='|' read -ra CFGS <<< "${AB_CONFIGS:-3}"
run() {  # "cfg extra" variant ("LIB:path" runs a prebuilt library instead)
  if [[ "$2" == LIB:* ]]; then export TBC_LIB_PATH="${2#LIB:}"; else unset TBC_LIB_PATH; fi
  TBC_VARIANT="${2#LIB:*}" timeout 400 python bench.py --config $1 --steps ${AB_STEPS:-3} --warmup 2 --no-cpu-baseline > /tmp/ab_out.txt 2>&1
  grep '^{' /tmp/ab_out.txt | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['config']['engine_mode'][:30])" 2>/dev/null || tail -3 /tmp/ab_out.txt
}
for c in "${CFGS[@]}"; do
  for rep in $(seq ${AB_REPS:-2}); do
    for v in "${VARS[@]}"; do
      echo "cfg[$c] rep$rep variant='$v' -> $(run "$c" "$v")"
    done
  done
done
