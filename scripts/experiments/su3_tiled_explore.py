"""Time OMPRT_TMA_TILED SU(3) for library builds with different warps per team x tile
buffers per warp (scripts/experiments/libomprt_w<W>_b<K>.so, -DOMPRT_SU3_TILED_*).
  python scripts/experiments/su3_tiled_explore.py lib1.so [lib2.so ...]"""
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
    ns = 32 ** 4
    A, B = gen.su3_inputs(ns)
    At, Bt = torch.from_numpy(A).to("cuda"), torch.from_numpy(B).to("cuda")
    Ct = torch.empty_like(At)
    ck = torch.zeros(1, dtype=torch.float64, device="cuda")
    scrub = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
    s = torch.cuda.current_stream()
    res = {}
    for name, fn in (("rt", omprt.omprt_su3_mult), ("twin", omprt.omprt_cuda_su3_mult)):
        out = []
        for _ in range(12):
            scrub.fill_(1.0)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            fn(At, Bt, Ct, ns, ck, 0, 128, omprt.OMPRT_TMA_TILED)
            b.record(s)
            torch.cuda.synchronize()
            out.append(a.elapsed_time(b))
        ms = statistics.median(out[2:])
        res[name] = {"ms": ms, "GBps_alg": 1152 * ns / ms / 1e6}
    ref = oracle_check = None
    print(json.dumps({"lib": os.path.basename(so), **res}), flush=True)


if __name__ == "__main__":
    if len(sys.argv) == 2:
        one(sys.argv[1])
    else:
        for so in sys.argv[1:]:
            subprocess.run([sys.executable, __file__, os.path.abspath(so)])
