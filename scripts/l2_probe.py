"""Does the L2 set-aside for persisting accesses (omprt_init reserves the device maximum)
slow the streaming kernels down?  Times SU(3) 32^4, C1 and the XS flat lookup with the
set-aside at its maximum and removed, plus the flattened RSBench variants.
  python scripts/l2_probe.py"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    import gen
    from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
    torch.cuda.set_device(0)
    omprt.omprt_init(0)
    dev, s = "cuda", torch.cuda.current_stream()
    scrub = torch.empty(64 << 20, dtype=torch.float32, device=dev)

    def t(fn, reps=7, reset=True):
        fn()
        torch.cuda.synchronize()
        out = []
        for _ in range(reps):
            torch.cuda.synchronize()
            if reset:
                omprt.omprt_l2_reset_persisting()
            scrub.fill_(1.0)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            fn()
            b.record(s)
            torch.cuda.synchronize()
            out.append(a.elapsed_time(b))
        return statistics.median(out)

    ns = 32 ** 4
    Ah, Bh = gen.su3_inputs(ns)
    At, Bt = torch.from_numpy(Ah).to(dev), torch.from_numpy(Bh).to(dev)
    Ct = torch.empty_like(At)
    ck = torch.zeros(1, dtype=torch.float64, device=dev)
    A = omprt.OMPRT_ASSUME_OVERSUB
    tabs = gen.XSTables(**gen.XS_SMALL)
    d = omprt.XSDeviceTables(tabs, dev, accel=True)
    n = 17_000_000
    ver = torch.empty(n, dtype=torch.uint64, device=dev)
    res = {}
    for setaside in ("max", 0, "max"):
        got = omprt.omprt_l2_set_aside(1 << 40 if setaside == "max" else 0)
        r = {"granted": got}
        r["su3"] = t(lambda: omprt.omprt_su3_mult(At, Bt, Ct, ns, ck, 0, 128, A))
        r["su3_twin"] = t(lambda: omprt.omprt_cuda_su3_mult(At, Bt, Ct, ns, ck, 0, 128, 0))
        r["su3_noreset"] = t(lambda: omprt.omprt_su3_mult(At, Bt, Ct, ns, ck, 0, 128, A),
                             reset=False)
        r["xs_flat"] = t(lambda: omprt.omprt_xs_lookup(d, 1070, 0, n, ver, None, 0, 256,
                                                       omprt.OMPRT_XS_FLAT), 5)
        r["su3_after_xs"] = t(lambda: omprt.omprt_su3_mult(At, Bt, Ct, ns, ck, 0, 128, A))
        res[f"setaside_{setaside}_{len(res)}"] = r
        print(json.dumps(r), flush=True)
    omprt.omprt_l2_set_aside(1 << 40)
    rs = gen.RSTables()
    rd = omprt.RSDeviceTables(rs, dev)
    m = 1_000_000
    v = torch.empty(m, dtype=torch.uint64, device=dev)
    F = omprt.OMPRT_FLAT
    r = {"rs_rt_1M": t(lambda: omprt.omprt_rs_lookup(rd, 1070, 0, m, v, None, 0, 128, A), 3)}
    ref = v.clone()
    r["rs_twin_1M"] = t(lambda: omprt.omprt_cuda_rs_lookup(rd, 1070, 0, m, v, None, 0, 128, 0), 3)
    r["rs_rt_flat_1M"] = t(lambda: omprt.omprt_rs_lookup(rd, 1070, 0, m, v, None, 0, 128, F), 3)
    r["rs_rt_flat_same"] = bool((v == ref).all())
    r["rs_twin_flat_1M"] = t(lambda: omprt.omprt_cuda_rs_lookup(rd, 1070, 0, m, v, None, 0, 128, F), 3)
    r["rs_twin_flat_same"] = bool((v == ref).all())
    print(json.dumps(r), flush=True)


if __name__ == "__main__":
    main()
