#!/bin/bash
# r2 x51: C4 v14 (own sincos: constant-bank polynomials, shifter reduction) vs v13
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 900 python scripts/rs_variant_time.py libs_x/rs_v13.so libs_x/rs_v14.so > $OUT/rs_x51.txt 2>&1
cp libs_x/rs_v14.so paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so
touch paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so
timeout 900 python -m pytest tests/test_gpu_rs_su3.py -q -x > $OUT/pt_x51.txt 2>&1
tail -3 $OUT/pt_x51.txt; cut -c1-400 $OUT/rs_x51.txt
