"""Quick CUDA-event timings of the secondary configs' variants (median of 7, L2 flushed).
  python scripts/quick_time.py [su3] [rs] [c1] [c2]"""
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

    def t(fn, reps=7):
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
        return statistics.median(out)

    A = omprt.OMPRT_ASSUME_OVERSUB
    res = {}
    if "su3" in which:
        ns = 32 ** 4
        Ah, Bh = gen.su3_inputs(ns)
        At, Bt = torch.from_numpy(Ah).to(dev), torch.from_numpy(Bh).to(dev)
        Ct = torch.empty_like(At)
        ck = torch.zeros(1, dtype=torch.float64, device=dev)
        variants = [("rt", omprt.omprt_su3_mult, A), ("twin", omprt.omprt_cuda_su3_mult, 0),
                    ("rt_wstaged", omprt.omprt_su3_mult, omprt.OMPRT_WARP_STAGED),
                    ("rt_tiled", omprt.omprt_su3_mult, omprt.OMPRT_TMA_TILED),
                    ("twin_tiled", omprt.omprt_cuda_su3_mult, omprt.OMPRT_TMA_TILED),
                    ("twin_wstaged", omprt.omprt_cuda_su3_mult, omprt.OMPRT_WARP_STAGED)]
        for name, fn, fl in variants:
            res[f"su3_{name}"] = {"ms": []}
        for _ in range(3):  # interleaved passes: run-to-run drift shows up as spread
            for name, fn, fl in variants:
                res[f"su3_{name}"]["ms"].append(t(lambda: fn(At, Bt, Ct, ns, ck, 0, 128, fl), 11))
        for name, _, _ in variants:
            ms = min(res[f"su3_{name}"]["ms"])
            res[f"su3_{name}"]["GBps_alg"] = 1152 * ns / ms / 1e6
    if "c1" in which:
        n = 1 << 20
        x, b, c = gen.axpy_inputs(n)
        bt, ct = torch.from_numpy(b).to(dev), torch.from_numpy(c).to(dev)
        at = torch.empty_like(bt)
        sm = torch.zeros(1, dtype=torch.float64, device=dev)
        TS_ = omprt.OMPRT_TMA_STREAM
        for name, fn, fl, T, N in [("rt", omprt.omprt_spmd_axpy_sum, 0, 8, 128),
                                   ("twin", omprt.omprt_cuda_axpy_sum, 0, 8, 128),
                                   ("rt_tma", omprt.omprt_spmd_axpy_sum, TS_, 8, 128),
                                   ("twin_tma", omprt.omprt_cuda_axpy_sum, TS_, 8, 128),
                                   ("rt_tma_8x256", omprt.omprt_spmd_axpy_sum, TS_, 8, 256),
                                   ("rt_tma_148x128", omprt.omprt_spmd_axpy_sum, TS_, 148, 128)]:
            ms = t(lambda: fn(n, x, bt, ct, at, sm, T, N, fl), 11)
            res[f"c1_{name}"] = {"ms": ms, "GBps_alg": 24 * n / ms / 1e6}
    if "c2" in which:
        T = 4096
        inp = torch.from_numpy(gen.generic_inputs(T, 256)).to(dev)
        out = torch.empty(T * 256, dtype=torch.float64, device=dev)
        A_ = omprt.OMPRT_ASSUME_OVERSUB
        for name, fl in [("rt", A_), ("rt_general_sm", omprt.OMPRT_GENERAL_SM),
                         ("rt_spmdized", A_ | omprt.OMPRT_SPMDIZE),
                         ("rt_deglobalized", A_ | omprt.OMPRT_DEGLOBALIZE)]:
            res[f"c2_{name}"] = {"ms": t(lambda: omprt.omprt_generic_team(T, 256, 256, inp, out, None, None, fl), 11)}
        res["c2_twin"] = {"ms": t(lambda: omprt.omprt_cuda_generic_team(T, 256, 256, inp, out), 11)}
        for k in [k for k in res if k.startswith("c2_")]:
            res[k]["GBps_alg"] = 16 * T * 256 / res[k]["ms"] / 1e6
    if "rs" in which:
        rs = gen.RSTables()
        rd = omprt.RSDeviceTables(rs, dev)
        n = 1_000_000
        v = torch.empty(n, dtype=torch.uint64, device=dev)
        res["rs_rt_1M"] = {"ms": t(lambda: omprt.omprt_rs_lookup(rd, 1070, 0, n, v, None, 0, 128, A), 3)}
        res["rs_twin_1M"] = {"ms": t(lambda: omprt.omprt_cuda_rs_lookup(rd, 1070, 0, n, v, None, 0, 128, 0), 3)}
        ref = v.clone()
        F = omprt.OMPRT_FLAT
        res["rs_rt_flat_1M"] = {"ms": t(lambda: omprt.omprt_rs_lookup(rd, 1070, 0, n, v, None, 0, 128, F), 3)}
        res["rs_rt_flat_1M"]["same"] = bool((v == ref).all())
        res["rs_twin_flat_1M"] = {"ms": t(lambda: omprt.omprt_cuda_rs_lookup(rd, 1070, 0, n, v, None, 0, 128, F), 3)}
        res["rs_twin_flat_1M"]["same"] = bool((v == ref).all())
    if "rsq" in which:  # C4 at 10M: dynamic lock-step flat vs the queued-Abrarov form
        rs = gen.RSTables()
        rd = omprt.RSDeviceTables(rs, dev)
        n = 10_000_000
        FD = omprt.OMPRT_FLAT | omprt.OMPRT_SCHED_DYNAMIC
        Q = FD | omprt.OMPRT_RS_QUEUE
        outs = {}
        variants = [("rt_dflat", omprt.omprt_rs_lookup, FD), ("twin_dflat", omprt.omprt_cuda_rs_lookup, FD),
                    ("rt_qflat", omprt.omprt_rs_lookup, Q), ("twin_qflat", omprt.omprt_cuda_rs_lookup, Q)]
        for name, fn, fl in variants:
            v = torch.empty(n, dtype=torch.uint64, device=dev)
            m = torch.empty(4 * n, dtype=torch.float64, device=dev)
            outs[name] = (v, m)
            res[f"rs10M_{name}"] = {"ms": []}
        for _ in range(2):
            for name, fn, fl in variants:
                v, m = outs[name]
                res[f"rs10M_{name}"]["ms"].append(
                    t(lambda: fn(rd, 1070, 0, n, v, m, 0, 128, fl), 3))
        v0, m0 = outs["rt_dflat"]
        m0 = m0.view(n, 4)
        for name in outs:
            v, m = outs[name]
            m = m.view(n, 4)
            err = ((m - m0).abs().max(dim=1).values / m0.abs().max(dim=1).values).max().item()
            res[f"rs10M_{name}"].update({"min_ms": min(res[f"rs10M_{name}"]["ms"]),
                                         "flips_vs_rt_dflat": int((v != v0).sum().item()),
                                         "max_norm_err_vs_rt_dflat": err})
    if "xs" in which:
        tabs = gen.XSTables(**gen.XS_SMALL)
        d = omprt.XSDeviceTables(tabs, dev, accel=True)
        n = 17_000_000
        ver = torch.empty(n, dtype=torch.uint64, device=dev)
        ck = torch.zeros(1, dtype=torch.uint64, device=dev)
        F, FU = omprt.OMPRT_XS_FLAT, omprt.OMPRT_FUSED_REDUCTION
        NW = omprt.OMPRT_XS_NO_L2_PERSIST
        for name, fn, fl in [("rt_flat", omprt.omprt_xs_lookup, F),
                             ("rt_flat_fused", omprt.omprt_xs_lookup, F | FU),
                             ("twin_flat_fused", omprt.omprt_cuda_xs_lookup, F | FU),
                             ("rt_flat_fused_nowin", omprt.omprt_xs_lookup, F | FU | NW)]:
            res[f"xs_{name}"] = {"ms": t(lambda: fn(d, 1070, 0, n, ver, ck, 0, 256, fl), 5)}
        ng = torch.from_numpy(tabs.nuclide_grid.reshape(-1)).to(dev)
        U = torch.empty(tabs.n_union, dtype=torch.float64, device=dev)
        i16 = torch.empty(tabs.n_union * tabs.n_isotopes, dtype=torch.int16, device=dev)
        tmp = torch.empty(omprt.omprt_xs_derive_tmp_bytes(68, 11303), dtype=torch.uint8,
                          device=dev)
        res["xs_derive"] = {"ms": t(lambda: omprt.omprt_xs_derive(ng, 68, 11303, U, i16, tmp), 5)}
    print(json.dumps(res))


if __name__ == "__main__":
    main(sys.argv[1:] or ["su3", "rs"])
