#!/bin/bash
TAG=${1:-x03}
OUT=gpurun_out
mkdir -p $OUT
export PYTHONUNBUFFERED=1
XSX_SRC=xs_explore2.cu XSX_ACCEL=1 timeout 900 python scripts/experiments/xs_explore.py > $OUT/xs_explore_$TAG.txt 2>&1
timeout 600 python scripts/run_kernels.py generic 1 > /dev/null 2>&1
timeout 600 ncu --section LaunchStats --section Occupancy --section SpeedOfLight -k regex:"generic" -c 3 python scripts/run_kernels.py generic 1 > $OUT/ncu_generic_$TAG.txt 2>&1
timeout 900 python bench.py --steps 5 --warmup 3 --no-e2e > $OUT/bench_$TAG.txt 2>&1
