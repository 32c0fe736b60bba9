#!/bin/bash
# L2 policy / smem-address variants A/B on cfg 3 and 2
AB_VARIANTS="|-DTBC_HOT_MB=32|-DTBC_HOT_MB=64|-DTBC_CLEAR_EF=1|-DTBC_WS_ASM=1" AB_CONFIGS="3|2" AB_REPS=2 AB_STEPS=3 bash tools/gpu_ab.sh
