#!/bin/bash
# ncu --set full of the RSBench kernels (nested, flattened lock-step, dynamic) on 1M lookups.
TAG=${1:-x09}
shift
KS=${@:-omprt_rs_rt omprt_rs_flat_rt omprt_rs_dflat_rt}
OUT=gpurun_out
mkdir -p $OUT
for K in $KS; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"^${K}" -c 1 \
    -o $OUT/prof_${K}_$TAG python scripts/run_kernels.py rs1m 1 > $OUT/ncu_${K}_$TAG.txt 2>&1
  ncu -i $OUT/prof_${K}_$TAG.ncu-rep --page raw --csv --print-units base > $OUT/raw_${K}_$TAG.csv 2>&1
  ncu -i $OUT/prof_${K}_$TAG.ncu-rep --page source --csv --print-units base > $OUT/src_${K}_$TAG.csv 2>&1
done
