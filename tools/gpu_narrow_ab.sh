for v in "" "-DTBC_SBLOCK=256" "-DTBC_SBLOCK=1024"; do
  TBC_VARIANT="$v" timeout 900 python tools/tune.py --config 4 --sources 592 --reps 1 --settings "batch=2;batch=2,slots=100;batch=2,slots=148;batch=2,slots=296" 2>&1 | grep setting | python -c "
import sys, json
for l in sys.stdin:
    d = json.loads(l); print('variant=$v', d['setting'], round(d['gteps'], 2), round(d['ms_per_source'], 3))"
done
