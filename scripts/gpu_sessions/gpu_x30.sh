#!/bin/bash
# r2 x30: the HBM stream probe + roof probes (bench.measure_peaks), C1 L2-prefetch variants
OUT=gpurun_out; mkdir -p $OUT; export PYTHONUNBUFFERED=1
timeout 300 python -m pytest tests/test_gpu_probes.py -q -x > $OUT/pt_probes_x30.txt 2>&1
timeout 300 python -c "
import json, torch, bench
from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
torch.cuda.set_device(0); omprt.omprt_init(0)
print(json.dumps(bench.measure_peaks(omprt, torch, torch.device('cuda',0), torch.cuda.current_stream()), indent=1))
" > $OUT/peaks_x30.txt 2>&1
timeout 300 scripts/experiments/c1_prefetch > $OUT/c1_prefetch_x30.txt 2>&1
tail -3 $OUT/pt_probes_x30.txt; grep -E "hbm|fp64" $OUT/peaks_x30.txt; cat $OUT/c1_prefetch_x30.txt
