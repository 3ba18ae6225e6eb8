#!/bin/bash
# final code check: the whole GPU suite and smoke (no re-measurement)
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 1500 python -m pytest tests -m gpu -q -rf --timeout 600 > $OUT/pytest_gpu_final.txt 2>&1
echo "pytest exit $?" >> $OUT/pytest_gpu_final.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke_final.txt 2>&1
echo "smoke exit $?" >> $OUT/smoke_final.txt
tail -3 $OUT/pytest_gpu_final.txt; tail -2 $OUT/smoke_final.txt
