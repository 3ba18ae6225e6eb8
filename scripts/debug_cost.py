"""NEXT f4 -- cost of the debug machinery (§III-G) and of thread ICV states
(P:106-108): release build vs the debug build (assertions + tracing compiled in) with the
runtime bits from OMPRT_DEBUG (read at omprt_init; run this once with OMPRT_DEBUG=0 and once
with OMPRT_DEBUG=1), plus the ICV-probe kernel (a nested parallel in every thread) with and
without thread ICV states.  Prints one JSON line.  Kernel times: CUDA events, median of 7,
L2 flushed before each repetition.

  OMPRT_DEBUG=0 python scripts/debug_cost.py ; OMPRT_DEBUG=1 python scripts/debug_cost.py
"""
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
    dev = "cuda"
    s = torch.cuda.current_stream()
    scrub = torch.empty(64 << 20, dtype=torch.float32, device=dev)

    def t(fn, reps=7):
        fn()
        torch.cuda.synchronize()
        out = []
        for _ in range(reps):
            scrub.fill_(1.0)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            fn()
            b.record(s)
            torch.cuda.synchronize()
            out.append(a.elapsed_time(b))
        return statistics.median(out)

    D, A = omprt.OMPRT_DEBUG_BUILD, omprt.OMPRT_ASSUME_OVERSUB
    res = {"OMPRT_DEBUG": os.environ.get("OMPRT_DEBUG", "0")}
    n = 1 << 20
    x, b, c = gen.axpy_inputs(n)
    bt, ct = torch.from_numpy(b).to(dev), torch.from_numpy(c).to(dev)
    at = torch.empty_like(bt)
    sm = torch.zeros(1, dtype=torch.float64, device=dev)
    res["c1_axpy"] = {
        "release_ms": t(lambda: omprt.omprt_spmd_axpy_sum(n, x, bt, ct, at, sm, 8, 128)),
        "debug_ms": t(lambda: omprt.omprt_spmd_axpy_sum(n, x, bt, ct, at, sm, 8, 128, D))}
    T = 4096
    inp = torch.from_numpy(gen.generic_inputs(T, 256)).to(dev)
    out = torch.empty(T * 256, dtype=torch.float64, device=dev)
    res["c2_generic"] = {
        "release_ms": t(lambda: omprt.omprt_generic_team(T, 256, 256, inp, out)),
        "debug_ms": t(lambda: omprt.omprt_generic_team(T, 256, 256, inp, out, None, None, D))}
    tabs = gen.XSTables(**gen.XS_SMALL)
    d = omprt.XSDeviceTables(tabs, dev)
    L = 4_000_000
    ver = torch.empty(L, dtype=torch.uint64, device=dev)
    res["c3_xs_4M"] = {
        "release_ms": t(lambda: omprt.omprt_xs_lookup(d, 1070, 0, L, ver, None, 0, 256, A)),
        "debug_ms": t(lambda: omprt.omprt_xs_lookup(d, 1070, 0, L, ver, None, 0, 256, A | D))}
    N = 256
    rec = torch.empty(T * (1 + 3 * N) * 7, dtype=torch.int32, device=dev)
    res["icv_nested_4096x256"] = {
        "register_context_ms": t(lambda: omprt.omprt_icv_probe(T, N, 4, rec, 0)),
        "thread_states_ms": t(lambda: omprt.omprt_icv_probe(T, N, 4, rec,
                                                            omprt.OMPRT_THREAD_STATES)),
        "general_sm_ms": t(lambda: omprt.omprt_icv_probe(T, N, 4, rec, omprt.OMPRT_GENERAL_SM))}
    if res["OMPRT_DEBUG"] != "0":
        res["icv_nested_4096x256"]["thread_states_debug_ms"] = t(
            lambda: omprt.omprt_icv_probe(T, N, 4, rec, omprt.OMPRT_THREAD_STATES | D))
    for k, v in res.items():
        if isinstance(v, dict) and "release_ms" in v:
            v["debug_over_release"] = v["debug_ms"] / v["release_ms"] - 1
    code, _ = omprt.omprt_device_status(0)
    res["device_status"] = code
    print(json.dumps(res))


if __name__ == "__main__":
    main()
