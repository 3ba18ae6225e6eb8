#!/bin/bash
# r2 x53: ncu --set full of C4 (queued flattened RSBench kernel, 10M lookups) at v13
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
K=omprt_rs_qflat_rt
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"^${K}" -c 1 \
  -o $OUT/prof_${K}_x53 python scripts/run_kernels.py rs10m 1 > $OUT/ncu_${K}_x53.txt 2>&1
ncu -i $OUT/prof_${K}_x53.ncu-rep --page raw --csv --print-units base > $OUT/raw_rsq10m_x53.csv 2>&1
ncu -i $OUT/prof_${K}_x53.ncu-rep --page source --csv --print-units base > $OUT/src_rsq10m_x53.csv 2>&1
rm -f $OUT/*.ncu-rep
tail -3 $OUT/ncu_${K}_x53.txt
