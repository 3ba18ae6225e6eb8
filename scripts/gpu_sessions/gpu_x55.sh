#!/bin/bash
# r2 x55: C4 v19 = v13 + windows sorted by l with run boundaries in the window record (R-A12; no per-pole l load): timing + RS parity
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 900 python scripts/rs_variant_time.py paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so > $OUT/rs_x55.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_rs_su3.py tests/test_gpu_multi.py -q -x > $OUT/pt_x55.txt 2>&1
tail -15 $OUT/pt_x55.txt; cut -c1-400 $OUT/rs_x55.txt
