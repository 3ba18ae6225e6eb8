#!/bin/bash
# r2 x32: C1 at 64 iterations per trip (teams <= 256): parity, resources, time
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 600 python -m pytest tests/test_gpu_spmd.py tests/test_gpu_resources.py tests/test_gpu_probes.py -q -x > $OUT/pt_x32.txt 2>&1
timeout 300 python scripts/c1_variant_time.py paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so > $OUT/c1_wide_x32.txt 2>&1
OMPRT_DEBUG=0 timeout 600 python scripts/debug_cost.py > $OUT/debug_cost_x32.txt 2>&1
tail -3 $OUT/pt_x32.txt; cat $OUT/c1_wide_x32.txt; head -c 1500 $OUT/debug_cost_x32.txt
