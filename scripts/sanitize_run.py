"""Small launches of every runtime kernel family (and twins) for compute-sanitizer
(memcheck / racecheck / synccheck / initcheck; SURVEY §4 T-sanitize).

  compute-sanitizer --tool racecheck python scripts/sanitize_run.py
"""
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
    dev = "cuda"
    A = omprt.OMPRT_ASSUME_OVERSUB
    # C1 (+ chunked)
    n = 1 << 14
    x, b, c = gen.axpy_inputs(n)
    bt, ct = torch.from_numpy(b).to(dev), torch.from_numpy(c).to(dev)
    at = torch.empty_like(bt)
    s = torch.zeros(1, dtype=torch.float64, device=dev)
    omprt.omprt_spmd_axpy_sum(n, x, bt, ct, at, s, 8, 128)
    omprt.omprt_cuda_axpy_sum(n, x, bt, ct, at, s, 8, 128)
    omprt.omprt_spmd_axpy_sum_chunked(n, 4, x, bt, ct, at, s, 8, 128)
    omprt.omprt_spmd_axpy_sum(n, x, bt, ct, at, s, 128, 128, A)
    D = omprt.OMPRT_SCHED_DYNAMIC  # schedule(dynamic, C): team-shared chunk counter
    own = torch.empty(n, dtype=torch.int32, device=dev)
    cnt = torch.zeros(n, dtype=torch.int32, device=dev)
    omprt.omprt_spmd_axpy_sum_chunked(n, 3, x, bt, ct, at, s, 8, 128,
                                      D | omprt.OMPRT_RECORD_OWNER, own, cnt)
    omprt.omprt_cuda_axpy_sum_chunked(n, 3, x, bt, ct, at, s, 8, 128, D)
    # C2: all state machines, stack placements, SPMDized, deglobalized, postlogue
    T = 16
    inp = torch.from_numpy(gen.generic_inputs(T, 256)).to(dev)
    out = torch.empty(T * 256, dtype=torch.float64, device=dev)
    post = torch.empty(T, dtype=torch.float64, device=dev)
    for f in (0, A, omprt.OMPRT_GENERAL_SM, omprt.OMPRT_SMALL_STACK, omprt.OMPRT_NO_STACK,
              omprt.OMPRT_SPMDIZE | A, omprt.OMPRT_DEGLOBALIZE | A):
        omprt.omprt_generic_team(T, 256, 256, inp, out, None, post, f | omprt.OMPRT_POSTLOGUE)
    omprt.omprt_cuda_generic_team(T, 256, 256, inp, out, None, post, omprt.OMPRT_POSTLOGUE)
    rec = torch.empty(T * (1 + 3 * 64) * 7, dtype=torch.int32, device=dev)
    for f in (0, omprt.OMPRT_THREAD_STATES, omprt.OMPRT_GENERAL_SM):
        omprt.omprt_icv_probe(T, 64, 4, rec, f)
    # C3 (reduced grid)
    t = gen.XSTables(n_isotopes=68, n_gridpoints=200)
    d = omprt.XSDeviceTables(t, dev, accel=True)
    m = 4096
    ver = torch.empty(m, dtype=torch.uint64, device=dev)
    ck = torch.zeros(1, dtype=torch.uint64, device=dev)
    omprt.omprt_xs_lookup(d, 1070, 0, m, ver, None, 0, 256, A)
    omprt.omprt_xs_lookup(d.plain(), 1070, 0, m, ver, None, 0, 256, A)
    omprt.omprt_xs_lookup(d, 1070, 0, m, None, ck, 0, 256, A | omprt.OMPRT_FUSED_REDUCTION)
    omprt.omprt_cuda_xs_lookup(d, 1070, 0, m, ver, None, 0, 256, 0)
    omprt.omprt_u64_sum(ver, m, ck)
    # flattened (static, dynamic), fused, with the L2 window; the macro test build
    F = omprt.OMPRT_XS_FLAT
    omprt.omprt_l2_set_aside(1 << 40)
    mac = torch.empty(5 * m, dtype=torch.float64, device=dev)
    omprt.omprt_xs_lookup(d, 1070, 0, m, ver, None, 0, 256, 0, macro=mac)
    omprt.omprt_xs_lookup(d, 1070, 0, m, ver, None, 3, 256, F, macro=mac)
    for fl in (F, F | D):
        for tab in (d,):
            omprt.omprt_xs_lookup(tab, 1070, 0, m, ver, None, 3, 256, fl)
            omprt.omprt_xs_lookup(tab, 1070, 0, m, None, ck, 3, 256,
                                  fl | omprt.OMPRT_FUSED_REDUCTION)
            omprt.omprt_cuda_xs_lookup(tab, 1070, 0, m, ver, None, 3, 256, fl)
    torch.cuda.synchronize()
    omprt.omprt_l2_set_aside(0)
    # C4 (reduced tables)
    rs = gen.RSTables(n_nuclides=355, avg_poles=20, avg_windows=4)
    rd = omprt.RSDeviceTables(rs, dev)
    v = torch.empty(512, dtype=torch.uint64, device=dev)
    omprt.omprt_rs_lookup(rd, 1070, 0, 512, v, None, 0, 128, A)
    omprt.omprt_cuda_rs_lookup(rd, 1070, 0, 512, v, None, 0, 128, 0)
    mac = torch.empty(512 * 4, dtype=torch.float64, device=dev)
    for fl in (F, F | D, F | D | omprt.OMPRT_RS_QUEUE):  # lock-step: static, dynamic, queued
        omprt.omprt_rs_lookup(rd, 1070, 0, 512, v, mac, 2, 128, fl)
        omprt.omprt_cuda_rs_lookup(rd, 1070, 0, 512, v, None, 2, 128, fl)
    # C5
    ns = 1024
    Ah, Bh = gen.su3_inputs(ns)
    At, Bt = torch.from_numpy(Ah).to(dev), torch.from_numpy(Bh).to(dev)
    Ct = torch.empty_like(At)
    cs = torch.zeros(1, dtype=torch.float64, device=dev)
    omprt.omprt_su3_mult(At, Bt, Ct, ns, cs, 0, 128, A)
    omprt.omprt_cuda_su3_mult(At, Bt, Ct, ns, cs, 0, 128, 0)
    # staged / streamed variants: SU(3) warp cp.async, 2-D tensor tiles; C1 TMA-streamed Fig. 5
    # columns
    for fl in [omprt.OMPRT_WARP_STAGED, omprt.OMPRT_TMA_TILED]:
        omprt.omprt_su3_mult(At, Bt, Ct, ns, cs, 2, 128, fl)
        omprt.omprt_cuda_su3_mult(At, Bt, Ct, ns, cs, 2, 128, fl)
    n1 = 8 * 128 * 40 + 77  # whole boxes, a partial box and a ragged last trip
    x1, b1, c1 = gen.axpy_inputs(n1)
    b1t, c1t = torch.from_numpy(b1).to(dev), torch.from_numpy(c1).to(dev)
    a1t = torch.empty_like(b1t)
    omprt.omprt_spmd_axpy_sum(n1, x1, b1t, c1t, a1t, s, 8, 128, omprt.OMPRT_TMA_STREAM)
    omprt.omprt_cuda_axpy_sum(n1, x1, b1t, c1t, a1t, s, 8, 128, omprt.OMPRT_TMA_STREAM)
    # lock-step loops with the warp-collective hook
    st = torch.zeros(5000, dtype=torch.int32, device=dev)
    hk = torch.zeros(3 * 64, dtype=torch.int32, device=dev)
    er = torch.zeros(1, dtype=torch.int32, device=dev)
    for dyn in (False, True):
        omprt.omprt_lockstep_probe(5000, 3, 64, dyn, st, hk, er)
    # the e2e derivation (merge levels, index rows, brackets, bins) and pipelined host steps
    import numpy as np
    tx = gen.XSTables(n_isotopes=68, n_gridpoints=40)  # the material lists name 68 nuclides
    g = np.ascontiguousarray(tx.nuclide_grid.reshape(68, 40, 6).copy())
    g[:, :, 0] = np.sort(np.floor(g[:, :, 0] * 64.0) / 64.0, axis=1)  # ties
    for grid in (tx.nuclide_grid, g):
        gt = torch.from_numpy(np.ascontiguousarray(grid.reshape(-1))).to(dev)
        U = torch.empty(68 * 40, dtype=torch.float64, device=dev)
        i16 = torch.empty(68 * 40 * 68, dtype=torch.int16, device=dev)
        tmp = torch.empty(omprt.omprt_xs_derive_tmp_bytes(68, 40), dtype=torch.uint8, device=dev)
        omprt.omprt_xs_derive(gt, 68, 40, U, i16, tmp)
    raw = {k: torch.from_numpy(getattr(tx, k)).pin_memory()
           for k in ("nuclide_grid", "num_nucs", "mats", "concs")}
    hs = omprt.xs_host_struct(tx, raw, derive=True)
    omprt.omprt_xs_run_host_steps(hs, gen.XS_LOOKUP_SEED, 0, 20_000, 2, flags=F)
    torch.cuda.synchronize()
    print("sanitize_run: ok, device status", omprt.omprt_device_status(0)[0],
          "lockstep errors", int(er.item()))


if __name__ == "__main__":
    main()
