#!/bin/bash
# r2 x62: C4 v22 = v20 + the record's first half (EA, RT) two poles ahead, the second half (RA, RF) at the pole's own start (no extra registers): timing vs v20 + RS parity
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 900 python scripts/rs_variant_time.py paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so libs_x/rs_v22.so > $OUT/rs_x62.txt 2>&1
cp libs_x/rs_v22.so paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so; touch paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so
timeout 900 python -m pytest tests/test_gpu_rs_su3.py -q -x -k rs_ > $OUT/pt_x62.txt 2>&1
tail -2 $OUT/pt_x62.txt; cut -c1-300 $OUT/rs_x62.txt
