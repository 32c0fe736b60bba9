#!/bin/bash
AB_VARIANTS="|LIB:paper_conf_icppw_artiless21_b200/libturbobc_base.so" AB_CONFIGS="3|2|5" AB_REPS=2 AB_STEPS=3 bash tools/gpu_ab.sh
