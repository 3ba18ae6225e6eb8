"""Measured roofs on this B200 (live, CUDA events; the numbers bench.py reports against):
L2 -> SM read bandwidth (streaming, random 32 B sectors, random 96 B records) of an
L2-resident buffer with 256-bit L1-non-allocating loads, and FP64 FMA throughput.
  python scripts/peaks_probe.py  -> one JSON line"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    import bench
    from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
    torch.cuda.set_device(0)
    omprt.omprt_init(0)
    dev = torch.device("cuda", 0)
    out = bench.measure_peaks(omprt, torch, dev, torch.cuda.current_stream(), detail=True)
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
