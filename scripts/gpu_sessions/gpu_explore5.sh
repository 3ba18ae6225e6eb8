#!/bin/bash
TAG=${1:-x05}
OUT=gpurun_out
mkdir -p $OUT
export PYTHONUNBUFFERED=1
timeout 600 python scripts/experiments/rs_explore.py > $OUT/rs_explore_$TAG.txt 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize_run.py > $OUT/sanitize_${tool}_$TAG.txt 2>&1
  echo "exit $?" >> $OUT/sanitize_${tool}_$TAG.txt
done
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 --no-secondary --no-e2e > $OUT/bench_2rank_sharedgpu_$TAG.txt 2>&1
echo "exit $?" >> $OUT/bench_2rank_sharedgpu_$TAG.txt
