#!/bin/bash
# r2 x01: measured roofs; does the XS flat launch's L2 window survive ncu (kernel vs
# application replay)?
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 300 python scripts/peaks_probe.py > $OUT/peaks_x01.txt 2>&1
timeout 300 python scripts/ncu_xs_timed.py win 3 > $OUT/xs_timed_x01.txt 2>&1
timeout 300 python scripts/ncu_xs_timed.py nowin 3 >> $OUT/xs_timed_x01.txt 2>&1
for M in win nowin; do
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none -k regex:omprt_xs_flat_rt --csv \
    --log-file $OUT/ncu_quick_${M}_x01.csv python scripts/ncu_xs_timed.py $M 2 > $OUT/ncu_quick_${M}_x01.txt 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:omprt_xs_flat_rt -c 1 \
  -o $OUT/prof_xs_kernelreplay_x01 python scripts/ncu_xs_timed.py win 1 > $OUT/ncu_full_kr_x01.txt 2>&1
ncu -i $OUT/prof_xs_kernelreplay_x01.ncu-rep --page raw --csv --print-units base > $OUT/raw_xs_kr_x01.csv 2>&1
timeout 1800 ncu --set full --clock-control none --replay-mode application -k regex:omprt_xs_flat_rt -c 1 \
  -o $OUT/prof_xs_appreplay_x01 python scripts/ncu_xs_timed.py win 1 > $OUT/ncu_full_ar_x01.txt 2>&1
ncu -i $OUT/prof_xs_appreplay_x01.ncu-rep --page raw --csv --print-units base > $OUT/raw_xs_ar_x01.csv 2>&1

rm -f $OUT/*.ncu-rep
cat $OUT/peaks_x01.txt $OUT/xs_timed_x01.txt; tail -3 $OUT/ncu_quick_*_x01.csv
