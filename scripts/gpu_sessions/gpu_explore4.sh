#!/bin/bash
TAG=${1:-x04}
OUT=gpurun_out
mkdir -p $OUT
export PYTHONUNBUFFERED=1
XSX_SRC=xs_explore3.cu XSX_ACCEL=1 timeout 900 python scripts/experiments/xs_explore.py > $OUT/xs_explore_$TAG.txt 2>&1
