#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
for V in 56 48; do
timeout 600 ncu --set full --clock-control none -k regex:"axpy_(rt|twin)" -s 2 -c 2 \
  -o $OUT/prof_c1_$V python scripts/c1_once.py libs_x/c1_$V.so > /dev/null 2>&1
ncu -i $OUT/prof_c1_$V.ncu-rep --page raw --csv --print-units base > $OUT/raw_c1_${V}_x05.csv 2>&1
done
rm -f $OUT/*.ncu-rep
