#!/bin/bash
# exploration run; ncu reports are exported to CSV on the box and deleted (64 MiB return cap)
TAG=${1:-x01}
OUT=gpurun_out
mkdir -p $OUT
export PYTHONUNBUFFERED=1
timeout 900 python scripts/experiments/xs_explore.py > $OUT/xs_explore_$TAG.txt 2>&1
for k in rs generic su3 axpy; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"omprt_|cuda_" -s 0 -c 3 \
    -o /tmp/prof_${k}_$TAG python scripts/run_kernels.py $k 1 > $OUT/ncu_${k}_$TAG.txt 2>&1
  ncu -i /tmp/prof_${k}_$TAG.ncu-rep --page raw --csv --print-units base > $OUT/raw_${k}_$TAG.csv 2>&1
  ncu -i /tmp/prof_${k}_$TAG.ncu-rep --page source --csv --print-units base > $OUT/src_${k}_$TAG.csv 2>&1
  du -sh $OUT/src_${k}_$TAG.csv
done
ls -la $OUT
du -sh $OUT
