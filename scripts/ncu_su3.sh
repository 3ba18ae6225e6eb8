#!/bin/bash
# ncu --set full of the SU(3) kernels (plain 256-bit, warp-staged) on 32^4 sites.
TAG=${1:-x19}
OUT=gpurun_out
mkdir -p $OUT
for K in omprt_su3_rt omprt_su3_wstaged_rt cuda_su3_twin; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"^${K}" -c 1 \
    -o $OUT/prof_${K}_$TAG python scripts/run_kernels.py su3 1 > $OUT/ncu_${K}_$TAG.txt 2>&1
  ncu -i $OUT/prof_${K}_$TAG.ncu-rep --page raw --csv --print-units base > $OUT/raw_${K}_$TAG.csv 2>&1
  rm -f $OUT/prof_${K}_$TAG.ncu-rep
done
