#!/bin/bash
# r2 x11: XS next-step bracket prefetch through shared memory (xs_explore11.cu); RS body v4
# (in-range reciprocal, folded asymptotic numerator) against the committed body
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
XSX_SRC=xs_explore11.cu XSX_ACCEL=1 XSX_LOG2BINS=18 timeout 900 python scripts/experiments/xs_explore.py > $OUT/xs_explore_x11_prefetch.txt 2>&1
timeout 900 python scripts/rs_variant_time.py libs_x/rs_v4.so paper_conf_ipps_doerfertphtdcg22_b200/libomprt.so > $OUT/rs_variants_x11.txt 2>&1
tail -6 $OUT/xs_explore_x11_prefetch.txt; cat $OUT/rs_variants_x11.txt | cut -c1-400
