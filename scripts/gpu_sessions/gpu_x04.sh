#!/bin/bash
# r2 x04: C1 register budgets, C5 twin, the headline launch under ncu (stream window)
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 600 python scripts/c1_variant_time.py libs_x/c1_48.so libs_x/c1_56.so > $OUT/c1_variants_x04.txt 2>&1
timeout 600 python scripts/quick_time.py su3 > $OUT/quick_su3_x04.txt 2>&1
timeout 300 python scripts/ncu_xs_timed.py win 3 > $OUT/xs_timed_x04.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:omprt_xs_flat_rt -c 1 \
  -o $OUT/prof_xs_timed_x04 python scripts/ncu_xs_timed.py win 1 > $OUT/ncu_full_xs_x04.txt 2>&1
ncu -i $OUT/prof_xs_timed_x04.ncu-rep --page raw --csv --print-units base > $OUT/raw_xs_timed_x04.csv 2>&1
ncu -i $OUT/prof_xs_timed_x04.ncu-rep --page source --csv --print-units base > $OUT/src_xs_timed_x04.csv 2>&1
rm -f $OUT/*.ncu-rep
cat $OUT/c1_variants_x04.txt $OUT/quick_su3_x04.txt $OUT/xs_timed_x04.txt | cut -c1-600
