OUT=gpurun_out; export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests/test_gpu_rs_su3.py tests/test_gpu_resources.py -q -x > $OUT/pytest_rs_x34.txt 2>&1; echo "exit $?" >> $OUT/pytest_rs_x34.txt
timeout 600 python scripts/quick_time.py rsq rs > $OUT/quick_rsq_x34.txt 2>&1
for T in memcheck racecheck synccheck; do timeout 600 compute-sanitizer --tool $T python scripts/sanitize_run.py > $OUT/sanitize_${T}_x34.txt 2>&1; done
