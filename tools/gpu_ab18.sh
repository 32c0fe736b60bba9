#!/bin/bash
AB_VARIANTS="|-DTBC_BUNROLL64=6" AB_CONFIGS="3|2" AB_REPS=2 AB_STEPS=3 bash tools/gpu_ab.sh
