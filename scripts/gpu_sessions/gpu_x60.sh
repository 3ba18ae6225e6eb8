#!/bin/bash
# r2 x60: e2e XS step A/B -- merge levels with 4 (round 1), 8, 16 outputs per thread (host clock, 20 steps, interleaved)
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
for r in 1 2 3; do
  for L in derive_old derive_m8 derive_m16; do
    echo "$L $(timeout 300 python scripts/e2e_time.py 20 libs_x/$L.so)" >> $OUT/e2e_ab_x60.txt
  done
done
cat $OUT/e2e_ab_x60.txt
