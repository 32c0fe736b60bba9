#!/bin/bash
timeout 600 python tools/tune.py --config 3 --sources 2048 --reps 1 --settings "width=32;width=64;width=32,bparts=2" 2>&1 | grep -v TRACE | cut -c1-90
timeout 900 python tools/tune.py --config 5 --sources 512 --reps 1 --settings "width=32;width=64" 2>&1 | grep -v TRACE | cut -c1-90
timeout 600 python tools/tune.py --config 2 --sources 1024 --reps 1 --settings "width=64;width=32;width=64,bparts=4" 2>&1 | grep -v TRACE | cut -c1-90
