#!/bin/bash
timeout 600 python tools/tune.py --config 3 --sources 512 --reps 1 --settings "hot=0;hot=-1;hot=200000;hot=500000;hot=1000000;hot=4194304" 2>&1 | grep -v TRACE | cut -c1-90
TBC_VARIANT="-DTBC_BHOT=0" timeout 600 python tools/tune.py --config 3 --sources 512 --reps 1 --settings "hot=0" 2>&1 | grep -v TRACE | cut -c1-90
timeout 600 python tools/tune.py --config 2 --sources 1024 --reps 1 --settings "hot=0;hot=-1;width=64,hot=0;width=64,hot=-1" 2>&1 | grep -v TRACE | cut -c1-90
