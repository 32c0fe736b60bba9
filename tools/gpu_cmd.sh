for v in "-DTBC_BLOCK=768 -DTBC_LANE_ITEMS=4" "-DTBC_BLOCK=640 -DTBC_LANE_ITEMS=4" "-DTBC_BLOCK=1024 -DTBC_LANE_ITEMS=4" "-DTBC_BLOCK=512 -DTBC_LANE_ITEMS=4" "-DTBC_BLOCK=768 -DTBC_LANE_ITEMS=8"; do
  echo "== $v"
  TBC_VARIANT="$v" timeout 600 python tools/tune.py --config 3 --sources 512 --reps 1 --settings "parts=8;parts=4" 2>&1 | grep -v TRACE | cut -c1-110
done
