"""Static (Fig. 5) vs dynamic schedule on the flattened XS and RS lookups, runtime vs twin,
and the XS flat kernel under L2 set-asides of several sizes (CUDA events, L2 flushed).
  python scripts/sched_probe.py [xs] [rs] [rs10m] [aside]"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main(which):
    import torch

    import gen
    from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
    torch.cuda.set_device(0)
    omprt.omprt_init(0)
    dev, s = "cuda", torch.cuda.current_stream()
    scrub = torch.empty(64 << 20, dtype=torch.float32, device=dev)

    def t(fn, reps=5):
        fn()
        torch.cuda.synchronize()
        out = []
        for _ in range(reps):
            torch.cuda.synchronize()
            omprt.omprt_l2_reset_persisting()
            scrub.fill_(1.0)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            fn()
            b.record(s)
            torch.cuda.synchronize()
            out.append(a.elapsed_time(b))
        return round(statistics.median(out), 4)

    F, D = omprt.OMPRT_XS_FLAT, omprt.OMPRT_SCHED_DYNAMIC
    if "xs" in which or "aside" in which:
        tabs = gen.XSTables(**gen.XS_SMALL)
        d = omprt.XSDeviceTables(tabs, dev, accel=True)
        n = 17_000_000
        ver = torch.empty(n, dtype=torch.uint64, device=dev)
        ref = torch.empty(n, dtype=torch.uint64, device=dev)
        omprt.omprt_xs_lookup(d, 1070, 0, n, ref, None, 0, 256, F)
    if "xs" in which:
        omprt.omprt_l2_set_aside(1 << 40)
        r = {}
        omprt.omprt_l2_set_aside(1 << 40)
        for name, fn, fl in [("rt_flat", omprt.omprt_xs_lookup, F),
                             ("twin_flat", omprt.omprt_cuda_xs_lookup, F),
                             ("rt_dflat", omprt.omprt_xs_lookup, F | D),
                             ("twin_dflat", omprt.omprt_cuda_xs_lookup, F | D)]:
            ver.zero_()
            r[name] = t(lambda: fn(d, 1070, 0, n, ver, None, 0, 256, fl))
            r[name + "_same"] = bool((ver == ref).all())
        print(json.dumps({"xs_17M_ms": r}), flush=True)
    if "aside" in which:
        r = {}
        for mb in (0, 24, 40, 64, 1 << 20):
            got = omprt.omprt_l2_set_aside(mb << 20)
            r[f"{got >> 20}MB_flat"] = t(lambda: omprt.omprt_xs_lookup(d, 1070, 0, n, ver, None, 0, 256, F))
            r[f"{got >> 20}MB_dflat"] = t(lambda: omprt.omprt_xs_lookup(d, 1070, 0, n, ver, None, 0, 256, F | D))
        omprt.omprt_l2_set_aside(0)
        print(json.dumps({"xs_aside_ms": r}), flush=True)
    for tag, m in (("rs", 1_000_000), ("rs10m", 10_000_000)):
        if tag not in which:
            continue
        rs = gen.RSTables()
        rd = omprt.RSDeviceTables(rs, dev)
        v = torch.empty(m, dtype=torch.uint64, device=dev)
        ref = torch.empty(m, dtype=torch.uint64, device=dev)
        reps = 3 if m <= 1_000_000 else 1
        r = {"rt_nested": t(lambda: omprt.omprt_rs_lookup(rd, 1070, 0, m, ref, None, 0, 128,
                                                          omprt.OMPRT_ASSUME_OVERSUB), reps)}
        for name, fn, fl in [("rt_flat", omprt.omprt_rs_lookup, F),
                             ("twin_flat", omprt.omprt_cuda_rs_lookup, F),
                             ("rt_dflat", omprt.omprt_rs_lookup, F | D),
                             ("twin_dflat", omprt.omprt_cuda_rs_lookup, F | D)]:
            v.zero_()
            r[name] = t(lambda: fn(rd, 1070, 0, m, v, None, 0, 128, fl), reps)
            r[name + "_same"] = bool((v == ref).all())
        print(json.dumps({f"{tag}_ms": r}), flush=True)


if __name__ == "__main__":
    main(sys.argv[1:] or ["xs", "rs", "aside"])
