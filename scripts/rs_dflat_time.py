"""C4's dynamic flattened kernel without the Abrarov queue, runtime-driven vs twin, 10M
lookups, 5 interleaved cold reps each (min):  python scripts/rs_dflat_time.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    import gen
    from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
    torch.cuda.set_device(0)
    omprt.omprt_init(0)
    d = omprt.RSDeviceTables(gen.RSTables(), "cuda")
    n = 10_000_000
    v = torch.empty(n, dtype=torch.uint64, device="cuda")
    s = torch.cuda.current_stream()
    scrub = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
    D = omprt.OMPRT_FLAT | omprt.OMPRT_SCHED_DYNAMIC
    fns = {"rt": lambda: omprt.omprt_rs_lookup(d, 1070, 0, n, v, None, 0, 128, D),
           "twin": lambda: omprt.omprt_cuda_rs_lookup(d, 1070, 0, n, v, None, 0, 128, D)}
    res = {k: [] for k in fns}
    for _ in range(5):
        for k, f in fns.items():
            torch.cuda.synchronize()
            scrub.fill_(1.0)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            f()
            b.record(s)
            torch.cuda.synchronize()
            res[k].append(a.elapsed_time(b))
    print({k: (min(x), sorted(x)) for k, x in res.items()})


if __name__ == "__main__":
    main()
