#!/bin/bash
# r2 x57: launch list of the e2e XS steps (omprt_xs_run_host_steps, derived tables) -- where the e2e step's extra ~0.25 ms goes
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 600 python scripts/e2e_profile.py 4 > $OUT/e2e_plain_x57.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file $OUT/e2e_launches_x57.csv python scripts/e2e_profile.py 4 > $OUT/e2e_ncu_x57.txt 2>&1
tail -2 $OUT/e2e_plain_x57.txt
