#!/bin/bash
# r2 x36: ncu --set full of the C4 kernel at the bench's 10M lookups
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"^omprt_rs_qflat_rt" -c 1 \
  -o $OUT/prof_rsq10m_x36 python scripts/run_kernels.py rs10m 1 > $OUT/ncu_rsq10m_x36.txt 2>&1
ncu -i $OUT/prof_rsq10m_x36.ncu-rep --page raw --csv --print-units base > $OUT/raw_rsq10m_x36.csv 2>&1
ncu -i $OUT/prof_rsq10m_x36.ncu-rep --page source --csv --print-units base > $OUT/src_rsq10m_x36.csv 2>&1
rm -f $OUT/*.ncu-rep
tail -3 $OUT/ncu_rsq10m_x36.txt; ls -la $OUT
