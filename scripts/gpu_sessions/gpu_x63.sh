#!/bin/bash
# r2 x63: omprt_rs_prepare also checks every reachable window was prepared: RS tests + multi
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests/test_gpu_rs_su3.py tests/test_gpu_multi.py -q -x > $OUT/pt_x63.txt 2>&1
tail -3 $OUT/pt_x63.txt
