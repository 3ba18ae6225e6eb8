#!/bin/bash
# r2 x38: C4 with the packed 2-bit l table (one word per 16 poles)
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 900 python scripts/rs_variant_time.py paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so > $OUT/rs_v10_x38.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_rs_su3.py tests/test_gpu_resources.py tests/test_gpu_multi.py -q -x > $OUT/pt_x38.txt 2>&1
cat $OUT/rs_v10_x38.txt; tail -3 $OUT/pt_x38.txt
