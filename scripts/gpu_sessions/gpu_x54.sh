#!/bin/bash
# r2 x54: C4 v16 (pole l requested 2 poles ahead), v17 (M0..M3 in per-thread shared-memory slots: no spills), v18 (both) vs v13
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 900 python scripts/rs_variant_time.py libs_x/rs_v13.so libs_x/rs_v16.so libs_x/rs_v17.so libs_x/rs_v18.so > $OUT/rs_x54.txt 2>&1
cut -c1-300 $OUT/rs_x54.txt
