#!/bin/bash
# r2 x44: ncu of C4's dynamic flattened kernels without the queue (runtime +4.6 % vs twin)
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
for K in omprt_rs_dflat_rt cuda_rs_dflat_twin; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"^${K}" -c 1 \
    -o $OUT/prof_${K}_x44 python scripts/run_kernels.py rsd10m 1 > $OUT/ncu_${K}_x44.txt 2>&1
  ncu -i $OUT/prof_${K}_x44.ncu-rep --page raw --csv --print-units base > $OUT/raw_${K}_x44.csv 2>&1
  ncu -i $OUT/prof_${K}_x44.ncu-rep --page source --csv --print-units base > $OUT/src_${K}_x44.csv 2>&1
  rm -f $OUT/*.ncu-rep
done
