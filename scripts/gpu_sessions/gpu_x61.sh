#!/bin/bash
# r2 x61: C4 v21 = v20 + the record's first half (EA, RT) requested two poles ahead, the second half one ahead (rotation; 222 B of spills) vs v20
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 900 python scripts/rs_variant_time.py paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so libs_x/rs_v21.so > $OUT/rs_x61.txt 2>&1
cut -c1-300 $OUT/rs_x61.txt
