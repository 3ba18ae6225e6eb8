#!/bin/bash
# r2 x46: C4 with the one-step reciprocal: RS parity + resources tests, C4 timing
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests/test_gpu_rs_su3.py tests/test_gpu_resources.py tests/test_gpu_multi.py -q > $OUT/pt_x46.txt 2>&1
timeout 900 python scripts/rs_variant_time.py paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so > $OUT/rs_v12_x46.txt 2>&1
tail -3 $OUT/pt_x46.txt; cut -c1-300 $OUT/rs_v12_x46.txt
