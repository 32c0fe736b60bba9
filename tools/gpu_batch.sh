#!/bin/bash
timeout 900 python tools/tune.py --config 3 --sources 2048 --reps 1 --settings "bparts=1;bparts=2;bpull=2;bpull=32;bpull=128" 2>&1 | grep -v TRACE | cut -c1-90
timeout 900 python tools/tune.py --config 5 --sources 512 --reps 1 --settings "bparts=1;bparts=2;bpull=32" 2>&1 | grep -v TRACE | cut -c1-90
timeout 600 python tools/tune.py --config 2 --sources 1024 --reps 1 --settings "bpull=2;bpull=8;bpull=32;bparts=2" 2>&1 | grep -v TRACE | cut -c1-90
