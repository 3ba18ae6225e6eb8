"""C1 (SPMD axpy + sum, 2^20, 8 x 128) runtime-driven vs twin for one or more builds of the
library (exploration of register budgets):  python scripts/c1_variant_time.py a.so [b.so ..]
Per build: cold trimmed means of 15 interleaved reps (bench._time_pair) and the warm
CUDA-graph figure (bench._time_graph), plus a[] and the sum checked bit-exact vs the
oracle."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def one(path):
    import numpy as np
    import torch

    import bench
    import gen
    import oracle
    from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
    omprt.load(path)
    torch.cuda.set_device(0)
    omprt.omprt_init(0)
    dev = torch.device("cuda", 0)
    s = torch.cuda.current_stream()
    scrub = torch.empty(64 << 20, dtype=torch.float32, device=dev)
    n = 1 << 20
    x, b, c = gen.axpy_inputs(n)
    bt, ct = torch.from_numpy(b).to(dev), torch.from_numpy(c).to(dev)
    at = torch.empty_like(bt)
    sm = torch.zeros(1, dtype=torch.float64, device=dev)
    rt1 = lambda: omprt.omprt_spmd_axpy_sum(n, x, bt, ct, at, sm, 8, 128)
    tw1 = lambda: omprt.omprt_cuda_axpy_sum(n, x, bt, ct, at, sm, 8, 128)
    t_rt, t_tw = bench._time_pair(rt1, tw1, s, scrub)
    g_rt, g_tw = bench._time_graph(rt1, tw1, s)
    # teams of 512 threads: the 8-iteration trips (the wide ones need <= 256)
    n_rt, n_tw = bench._time_pair(lambda: omprt.omprt_spmd_axpy_sum(n, x, bt, ct, at, sm, 8, 512),
                                  lambda: omprt.omprt_cuda_axpy_sum(n, x, bt, ct, at, sm, 8, 512),
                                  s, scrub)
    sm.zero_()
    rt1()
    torch.cuda.synchronize()
    ok = bool((at.cpu().numpy() == oracle.axpy(x, b, c)).all())
    tab = omprt.kernel_table()
    print(json.dumps({"lib": path, "rt_ms": t_rt, "twin_ms": t_tw, "graph_rt_ms": g_rt,
                      "graph_twin_ms": g_tw, "a_bit_exact": ok,
                      "x512_rt_ms": n_rt, "x512_twin_ms": n_tw,
                      "regs": [tab["omprt_axpy_rt"]["regs"], tab["cuda_axpy_twin"]["regs"]]}),
          flush=True)


if __name__ == "__main__":
    if sys.argv[1] != "--one":
        for p in sys.argv[1:]:
            subprocess.run([sys.executable, __file__, "--one", p])
    else:
        one(sys.argv[2])
