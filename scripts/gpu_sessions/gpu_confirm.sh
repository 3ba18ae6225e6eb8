OUT=gpurun_out; TAG=${1:-r19}; mkdir -p $OUT; export PYTHONUNBUFFERED=1
nvidia-smi -L > $OUT/nvidia_smi_$TAG.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -rf --timeout 600 > $OUT/pytest_gpu_$TAG.txt 2>&1; echo "pytest exit $?" >> $OUT/pytest_gpu_$TAG.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke_$TAG.txt 2>&1; echo "smoke exit $?" >> $OUT/smoke_$TAG.txt
timeout 900 python bench.py --steps 10 --warmup 3 > $OUT/bench_$TAG.txt 2>&1; echo "bench exit $?" >> $OUT/bench_$TAG.txt
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > $OUT/bench_ref_$TAG.txt 2>&1
