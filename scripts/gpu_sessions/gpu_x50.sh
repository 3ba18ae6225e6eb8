#!/bin/bash
# r2 x50: C4 v13 (pole contributions accumulated by fma chains) vs v12 (committed): timing + RS parity
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 900 python scripts/rs_variant_time.py libs_x/rs_v12.so libs_x/rs_v13.so > $OUT/rs_x50.txt 2>&1
cp libs_x/rs_v13.so paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so
touch paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so
timeout 900 python -m pytest tests/test_gpu_rs_su3.py -q -x > $OUT/pt_x50.txt 2>&1
tail -3 $OUT/pt_x50.txt; cut -c1-400 $OUT/rs_x50.txt
