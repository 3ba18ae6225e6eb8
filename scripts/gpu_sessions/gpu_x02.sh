#!/bin/bash
# r2 x02: the window under ncu (stream attribute, cache-control none); RSBench body variants
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
for M in win stream nowin; do timeout 300 python scripts/ncu_xs_timed.py $M 3; done > $OUT/xs_timed_x02.txt 2>&1
for M in stream; do
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none -k regex:omprt_xs_flat_rt --csv \
    --log-file $OUT/ncu_quick_${M}_x02.csv python scripts/ncu_xs_timed.py $M 2 > $OUT/ncu_quick_${M}_x02.txt 2>&1
done
timeout 600 ncu --cache-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none -k regex:omprt_xs_flat_rt --csv \
    --log-file $OUT/ncu_quick_ccnone_x02.csv python scripts/ncu_xs_timed.py win 2 > $OUT/ncu_quick_ccnone_x02.txt 2>&1
timeout 900 python scripts/rs_variant_time.py libs_x/v0.so libs_x/v1.so libs_x/v2.so libs_x/v3.so > $OUT/rs_variants_x02.txt 2>&1
rm -f $OUT/*.ncu-rep
cat $OUT/xs_timed_x02.txt $OUT/rs_variants_x02.txt; grep -h "gpu__time\|dram__bytes_read" $OUT/ncu_quick_*_x02.csv
