#!/bin/bash
TAG=${1:-x02}
OUT=gpurun_out
mkdir -p $OUT
export PYTHONUNBUFFERED=1
timeout 900 python scripts/experiments/xs_explore.py > $OUT/xs_explore_$TAG.txt 2>&1
timeout 900 python bench.py --steps 5 --warmup 3 --no-e2e > $OUT/bench_$TAG.txt 2>&1
ls -la $OUT
