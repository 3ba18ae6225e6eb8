#!/bin/bash
# r2 x56: C4 v20 = v19 + one prepared 64 B record per material entry (k0rs, conc, window offset | count; R-A13): timing + RS parity
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 900 python scripts/rs_variant_time.py paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so > $OUT/rs_x56.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_rs_su3.py tests/test_gpu_multi.py -q -x > $OUT/pt_x56.txt 2>&1
tail -15 $OUT/pt_x56.txt; cut -c1-400 $OUT/rs_x56.txt
