"""Time the C4 path (queued flattened RSBench kernel, runtime-driven and twin) of one or more
builds of the library -- exploration of rs_body variants, each build a separate .so:
  python scripts/rs_variant_time.py /path/a.so [/path/b.so ...]
Per build: kernel ms at 10M lookups (cold L2, 3 interleaved reps, min), the verification
checksum, and whether runtime and twin give bit-identical macroscopic values (1M lookups)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def one(path):
    import numpy as np
    import torch

    import gen
    from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
    omprt.load(path)
    torch.cuda.set_device(0)
    omprt.omprt_init(0)
    dev = torch.device("cuda", 0)
    d = omprt.RSDeviceTables(gen.RSTables(), dev)
    n = 10_000_000
    v = torch.empty(n, dtype=torch.uint64, device=dev)
    FQ = omprt.OMPRT_FLAT | omprt.OMPRT_SCHED_DYNAMIC | omprt.OMPRT_RS_QUEUE
    FQ |= int(os.environ.get("RSV_EXTRA_FLAGS", "0"), 0)
    scrub = torch.empty(64 << 20, dtype=torch.float32, device=dev)
    s = torch.cuda.current_stream()
    fns = {"rt": lambda: omprt.omprt_rs_lookup(d, 1070, 0, n, v, None, 0, 128, FQ),
           "twin": lambda: omprt.omprt_cuda_rs_lookup(d, 1070, 0, n, v, None, 0, 128, FQ)}
    res = {k: [] for k in fns}
    cks = {}
    for rep in range(4):
        for k, f in fns.items():
            torch.cuda.synchronize()
            scrub.fill_(1.0)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            f()
            b.record(s)
            torch.cuda.synchronize()
            if rep:
                res[k].append(a.elapsed_time(b))
            cks[k] = int(v.sum().item())
    m = 1_000_000
    mac = {}
    for k, fn in (("rt", omprt.omprt_rs_lookup), ("twin", omprt.omprt_cuda_rs_lookup)):
        mm = torch.empty(4 * m, dtype=torch.float64, device=dev)
        vv = torch.empty(m, dtype=torch.uint64, device=dev)
        fn(d, 1070, 0, m, vv, mm, 0, 128, FQ)
        torch.cuda.synchronize()
        mac[k] = mm.cpu().numpy()
    tab = omprt.kernel_table()
    D = omprt.OMPRT_FLAT | omprt.OMPRT_SCHED_DYNAMIC
    m0 = torch.empty(4 * m, dtype=torch.float64, device=dev)
    v0 = torch.empty(m, dtype=torch.uint64, device=dev)
    omprt.omprt_rs_lookup(d, 1070, 0, m, v0, m0, 0, 128, D)  # no queue: the reference order
    torch.cuda.synchronize()
    ref = m0.cpu().numpy().reshape(-1, 4)
    got = mac["rt"].reshape(-1, 4)
    normwise = float((np.abs(got - ref).max(axis=1) / np.abs(ref).max(axis=1)).max())
    out = {"lib": path, "flags": FQ, "max_normwise_vs_unqueued": normwise, "rt_ms": min(res["rt"]), "twin_ms": min(res["twin"]),
           "rt_all": res["rt"], "twin_all": res["twin"], "checksums": cks,
           "rt_twin_macro_bit_identical": bool((mac["rt"].view(np.uint64) ==
                                                mac["twin"].view(np.uint64)).all()),
           "regs": [tab["omprt_rs_qflat_rt"]["regs"], tab["cuda_rs_qflat_twin"]["regs"]],
           "local": [tab["omprt_rs_qflat_rt"]["local_bytes"],
                     tab["cuda_rs_qflat_twin"]["local_bytes"]]}
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    if sys.argv[1] != "--one":
        for p in sys.argv[1:]:
            subprocess.run([sys.executable, __file__, "--one", p])
    else:
        one(sys.argv[2])
