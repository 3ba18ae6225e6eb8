"""XS step with the verification reduction fused into the flattened lookup kernel vs the
separate K11 sum kernel, L2 set-aside at its maximum, interleaved cold reps.
  python scripts/fused_probe.py"""
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
    omprt.omprt_l2_set_aside(1 << 40)
    t = gen.XSTables(**gen.XS_SMALL)
    d = omprt.XSDeviceTables(t, "cuda", accel=True)
    n = 17_000_000
    ver = torch.zeros(n, dtype=torch.uint64, device="cuda")
    ck = torch.zeros(1, dtype=torch.uint64, device="cuda")
    scrub = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
    s = torch.cuda.current_stream()
    F, FU = omprt.OMPRT_XS_FLAT, omprt.OMPRT_FUSED_REDUCTION

    def sep():
        ck.zero_()
        omprt.omprt_xs_lookup(d, gen.XS_LOOKUP_SEED, 0, n, ver, None, 0, 256, F)
        omprt.omprt_u64_sum(ver, n, ck)

    def fused():
        ck.zero_()
        omprt.omprt_xs_lookup(d, gen.XS_LOOKUP_SEED, 0, n, None, ck, 0, 256, F | FU)

    fns = {"separate_K11": sep, "fused": fused}
    ms = {k: [] for k in fns}
    cks = {}
    for r in range(12):
        for k in (list(fns) if r % 2 == 0 else list(fns)[::-1]):
            torch.cuda.synchronize()
            omprt.omprt_l2_reset_persisting()
            scrub.fill_(1.0)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            fns[k]()
            b.record(s)
            torch.cuda.synchronize()
            ms[k].append(a.elapsed_time(b))
            cks[k] = int(ck.cpu().numpy()[0])
    res = {k: statistics.median(v[2:]) for k, v in ms.items()}
    res["same_checksum"] = cks["fused"] == cks["separate_K11"]
    print(json.dumps(res))


if __name__ == "__main__":
    main()
