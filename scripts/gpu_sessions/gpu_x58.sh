#!/bin/bash
# r2 x58: warp-cooperative merge levels of the e2e table derivation: derive + e2e tests, launch list, e2e time
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests/test_gpu_xsbench.py -q -x -k "derive or end_to_end or host" > $OUT/pt_x58.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file $OUT/e2e_launches_x58.csv python scripts/e2e_profile.py 4 > $OUT/e2e_ncu_x58.txt 2>&1
timeout 600 python scripts/e2e_time.py > $OUT/e2e_time_x58.txt 2>&1
tail -3 $OUT/pt_x58.txt; tail -5 $OUT/e2e_time_x58.txt
