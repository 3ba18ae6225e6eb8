"""One C1 launch each of the runtime-driven kernel and its twin (for ncu): python
scripts/c1_once.py [lib.so]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    import gen
    from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
    if len(sys.argv) > 1:
        omprt.load(sys.argv[1])
    torch.cuda.set_device(0)
    omprt.omprt_init(0)
    dev = torch.device("cuda", 0)
    n = 1 << 20
    x, b, c = gen.axpy_inputs(n)
    bt, ct = torch.from_numpy(b).to(dev), torch.from_numpy(c).to(dev)
    at = torch.empty_like(bt)
    s = torch.zeros(1, dtype=torch.float64, device=dev)
    for _ in range(2):
        omprt.omprt_spmd_axpy_sum(n, x, bt, ct, at, s, 8, 128)
        omprt.omprt_cuda_axpy_sum(n, x, bt, ct, at, s, 8, 128)
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()
