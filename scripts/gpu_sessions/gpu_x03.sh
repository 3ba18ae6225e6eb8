#!/bin/bash
# r2 x03: GPU tests, bench (new fields), the window as a stream attribute under ncu, and the
# N>1 path with 2 ranks sharing the GPU
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 1500 python -m pytest tests -m gpu -q -rf --timeout 600 > $OUT/pytest_gpu_x03.txt 2>&1
echo "pytest exit $?" >> $OUT/pytest_gpu_x03.txt
timeout 900 python bench.py --steps 10 --warmup 3 > $OUT/bench_x03.txt 2>&1
echo "bench exit $?" >> $OUT/bench_x03.txt
timeout 300 python scripts/ncu_xs_timed.py stream 3 > $OUT/xs_timed_x03.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none -k regex:omprt_xs_flat_rt --csv \
    --log-file $OUT/ncu_quick_stream_x03.csv python scripts/ncu_xs_timed.py stream 2 > $OUT/ncu_quick_stream_x03.txt 2>&1
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 3 --warmup 3 > $OUT/bench_2rank_x03.txt 2>&1
rm -f $OUT/*.ncu-rep
tail -5 $OUT/pytest_gpu_x03.txt; cat $OUT/xs_timed_x03.txt; grep -h "gpu__time\|dram__bytes_read" $OUT/ncu_quick_stream_x03.csv | cut -c1-50,200-; tail -c 3000 $OUT/bench_x03.txt
