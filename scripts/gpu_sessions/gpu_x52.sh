#!/bin/bash
# r2 x52: C4 v15 (pole records L1-prefetched 2 / 3 poles ahead, loads L1-allocating) vs v13 (fma accumulation)
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 900 python scripts/rs_variant_time.py libs_x/rs_v13.so libs_x/rs_v15_2.so libs_x/rs_v15_3.so > $OUT/rs_x52.txt 2>&1
cut -c1-300 $OUT/rs_x52.txt
