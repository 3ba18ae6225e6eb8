#!/bin/bash
TAG=${1:-x06}
OUT=gpurun_out
mkdir -p $OUT
export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests/test_gpu_rs_su3.py tests/test_gpu_resources.py -q -x > $OUT/pytest_su3_$TAG.txt 2>&1
timeout 600 python scripts/quick_time.py su3 rs > $OUT/quick_$TAG.txt 2>&1
timeout 600 compute-sanitizer --tool memcheck python scripts/sanitize_run.py > $OUT/sanitize_memcheck_$TAG.txt 2>&1
timeout 600 compute-sanitizer --tool racecheck python scripts/sanitize_run.py > $OUT/sanitize_racecheck_$TAG.txt 2>&1
