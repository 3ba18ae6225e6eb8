"""Time OMPRT_TMA_STREAM axpy+sum for library builds with different stage counts and
output paths (scripts/experiments/libomprt_s<K>_st<0|1>.so).
  python scripts/experiments/c1_tma_explore.py lib1.so [lib2.so ...]"""
import json
import os
import statistics
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(os.path.dirname(HERE))


def one(so):
    sys.path.insert(0, ROOT)
    import torch

    import gen
    from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
    omprt.load(so)
    torch.cuda.set_device(0)
    omprt.omprt_init(0)
    n = 1 << 20
    x, b, c = gen.axpy_inputs(n)
    bt, ct = torch.from_numpy(b).to("cuda"), torch.from_numpy(c).to("cuda")
    at = torch.empty_like(bt)
    sm = torch.zeros(1, dtype=torch.float64, device="cuda")
    scrub = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
    s = torch.cuda.current_stream()
    res = {}
    for name, fn, T, N in (("rt_8x128", omprt.omprt_spmd_axpy_sum, 8, 128),
                           ("twin_8x128", omprt.omprt_cuda_axpy_sum, 8, 128),
                           ("rt_8x256", omprt.omprt_spmd_axpy_sum, 8, 256),
                           ("twin_8x256", omprt.omprt_cuda_axpy_sum, 8, 256)):
        out = []
        for _ in range(15):
            scrub.fill_(1.0)
            a0, b0 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(s)
            fn(n, x, bt, ct, at, sm, T, N, omprt.OMPRT_TMA_STREAM)
            b0.record(s)
            torch.cuda.synchronize()
            out.append(a0.elapsed_time(b0))
        ms = statistics.median(out[3:])
        res[name] = {"ms": round(ms, 5), "GBps_alg": round(24 * n / ms / 1e6, 1)}
    print(json.dumps({"lib": os.path.basename(so), **res}), flush=True)


if __name__ == "__main__":
    if len(sys.argv) == 2:
        one(sys.argv[1])
    else:
        for so in sys.argv[1:]:
            subprocess.run([sys.executable, __file__, os.path.abspath(so)])
