"""XS flattened lookups with the L2 set-aside at its maximum: tables packed as
[unionized | bins | brackets] (one access-policy window over all three) vs separate
allocations (window over the brackets only).  Interleaved, cold (reset + flush) per rep.
  python scripts/l2_pack_probe.py"""
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
    got = omprt.omprt_l2_set_aside(1 << 40)
    t = gen.XSTables(**gen.XS_SMALL)
    n = 17_000_000
    tabs = {"packed": omprt.XSDeviceTables(t, "cuda", accel=True, packed=True),
            "separate": omprt.XSDeviceTables(t, "cuda", accel=True, packed=False)}
    for lb in (17, 18, 19):  # finer search bins (still inside the window up to 2^19)
        tabs[f"packed_bins{lb}"] = omprt.XSDeviceTables(t, "cuda", accel=True, packed=True,
                                                        log2_bins=lb)
    ver = {k: torch.zeros(n, dtype=torch.uint64, device="cuda") for k in tabs}
    scrub = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
    s = torch.cuda.current_stream()
    ms = {k: [] for k in tabs}
    F = omprt.OMPRT_XS_FLAT
    for r in range(12):
        ks = list(tabs)
        for k in (ks if r % 2 == 0 else ks[::-1]):
            torch.cuda.synchronize()
            omprt.omprt_l2_reset_persisting()
            scrub.fill_(1.0)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            omprt.omprt_xs_lookup(tabs[k], gen.XS_LOOKUP_SEED, 0, n, ver[k], None, 0, 256, F)
            b.record(s)
            torch.cuda.synchronize()
            ms[k].append(a.elapsed_time(b))
    res = {k: statistics.median(v[2:]) for k, v in ms.items()}
    res["same"] = all(bool(torch.equal(ver["packed"], v)) for v in ver.values())
    res["set_aside"] = got
    print(json.dumps(res))


if __name__ == "__main__":
    main()
