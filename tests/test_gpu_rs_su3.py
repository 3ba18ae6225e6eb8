"""GPU parity: RSBench-shaped lookups (tolerance contract) and SU(3)
(bit-exact, §8(c) C6)."""
import os

import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


@pytest.fixture(scope="module")
def rs_dev(rt, rs_tables):
    return rt.RSDeviceTables(rs_tables, DEV)


def _rs(rt, d, first, count, which, flags=0, teams=0):
    ver = torch.zeros(max(count, 1), dtype=torch.uint64, device=DEV)
    mac = torch.zeros(max(count, 1) * 4, dtype=torch.float64, device=DEV)
    fn = rt.omprt_rs_lookup if which == "rt" else rt.omprt_cuda_rs_lookup
    fn(d, gen.RS_LOOKUP_SEED, first, count, ver, mac, teams, 128, flags)
    torch.cuda.synchronize()
    return ver.cpu().numpy()[:count], mac.cpu().numpy()[: 4 * count].reshape(count, 4)


@pytest.mark.parametrize("variant", ["rt", "rt_assume", "twin", "rt_flat", "twin_flat",
                                     "rt_dflat", "twin_dflat", "rt_qflat", "twin_qflat"])
def test_rs_parity(rt, rs_dev, rs_tables, variant):
    first, count = 4321, 20_000 + 17
    D = rt.OMPRT_FLAT | rt.OMPRT_SCHED_DYNAMIC
    Q = D | rt.OMPRT_RS_QUEUE
    flags = {"rt_assume": rt.OMPRT_ASSUME_OVERSUB, "rt_flat": rt.OMPRT_FLAT,
             "twin_flat": rt.OMPRT_FLAT, "rt_dflat": D, "twin_dflat": D,
             "rt_qflat": Q, "twin_qflat": Q}.get(variant, 0)
    ver, mac = _rs(rt, rs_dev, first, count, "twin" if variant.startswith("twin") else "rt",
                   flags)
    rv, rm = oracle.rs_lookup(rs_tables, first, count, want_macro=True,
                              threads=os.cpu_count() or 1)
    # macro xs normwise (sigma_E = sigma_T - sigma_A can cancel): 1e-10
    err = np.abs(mac - rm).max(axis=1) / np.abs(rm).max(axis=1)
    assert err.max() <= 1e-10, err.max()
    # verification: identical, except flips that are near-ties in the oracle
    flip = np.nonzero(ver != rv)[0]
    for q in flip:
        top2 = np.sort(rm[q])[-2:]
        assert top2[1] - top2[0] <= 1e-12 * abs(top2[1]), (q, rm[q], mac[q])
    assert flip.size <= 2


def _bitwise(v1, m1, v0, m0):
    assert (m1.view(np.uint64) == m0.view(np.uint64)).all()
    assert (v1 == v0).all()


def test_rs_rt_and_twin_agree(rt, rs_dev):
    """Same body in both kernels, every operation explicit (fma / __dmul_rn / __dadd_rn,
    SURVEY Q12): nvcc has no contraction left to choose, so the runtime-driven kernel and
    its twin compute the same bits."""
    n = 100_000
    v1, m1 = _rs(rt, rs_dev, 0, n, "rt", rt.OMPRT_ASSUME_OVERSUB)
    v2, m2 = _rs(rt, rs_dev, 0, n, "twin")
    _bitwise(v1, m1, v2, m2)


def _agree(v1, m1, v0, m0):
    """The queued form (R-A8) sums the Abrarov poles' contributions in another order (and
    which poles are queued depends on the dynamic schedule), so macro xs agree to rounding
    (1e-12 normwise) and verification exactly up to near-ties."""
    err = np.abs(m1 - m0).max(axis=1) / np.abs(m0).max(axis=1)
    assert err.max() <= 1e-12, err.max()
    for q in np.nonzero(v1 != v0)[0]:
        top2 = np.sort(m0[q])[-2:]
        assert top2[1] - top2[0] <= 1e-12 * abs(top2[1])


@pytest.mark.parametrize("teams", [0, 1, 7, 148])
def test_rs_flat_equals_nested(rt, rs_dev, teams):
    """The flattened loop (one nuclide per step, lookups i, i+T*N, ... per thread, lock-step
    warps) and its dynamic-schedule form run the same per-lookup arithmetic in the same
    order as the nested loop, for persistent grids of any size (teams=1: 128 threads walk
    all lookups, the LCG jump between a thread's lookups exercised thousands of times):
    bit-identical results; the queued form agrees to rounding (R-A8)."""
    first, n = 777, 30_011
    v0, m0 = _rs(rt, rs_dev, first, n, "rt")
    D = rt.OMPRT_FLAT | rt.OMPRT_SCHED_DYNAMIC
    Q = D | rt.OMPRT_RS_QUEUE  # R-A8: another summation order, agreement to rounding
    for which, fl in (("rt", rt.OMPRT_FLAT), ("twin", rt.OMPRT_FLAT), ("rt", D), ("twin", D)):
        v, m = _rs(rt, rs_dev, first, n, which, fl, teams)
        _bitwise(v, m, v0, m0)
    for which in ("rt", "twin"):
        v, m = _rs(rt, rs_dev, first, n, which, Q, teams)
        _agree(v, m, v0, m0)


def test_rs_queue_full_10M_checksum(rt, rs_dev, rs_tables):
    """The C4 bench path (queued Abrarov poles, bench's launch configuration) at the full 10M
    lookups: the verification checksum equals the plain dynamic lock-step kernel's, no
    lookup flips except at near-ties, and sampled windows across the whole range (the
    first, middle and last lookups of the batch) match the oracle lookup by lookup."""
    n = 10_000_000
    D = rt.OMPRT_FLAT | rt.OMPRT_SCHED_DYNAMIC
    v0, m0 = _rs(rt, rs_dev, 0, n, "rt", D)
    v1, m1 = _rs(rt, rs_dev, 0, n, "rt", D | rt.OMPRT_RS_QUEUE)
    _agree(v1, m1, v0, m0)
    assert int(v1.sum(dtype=np.uint64)) == int(v0.sum(dtype=np.uint64))
    for first in (0, 1_234_567, 5_000_000, 8_765_432, n - 300):
        rv, rm = oracle.rs_lookup(rs_tables, first, 300, want_macro=True,
                                  threads=os.cpu_count() or 1)
        mac, ver = m1[first:first + 300], v1[first:first + 300]
        err = np.abs(mac - rm).max(axis=1) / np.abs(rm).max(axis=1)
        assert err.max() <= 1e-10, (first, err.max())
        for q in np.nonzero(ver != rv)[0]:
            top2 = np.sort(rm[q])[-2:]
            assert top2[1] - top2[0] <= 1e-12 * abs(top2[1]), (first + q, rm[q])


def test_rs_queue_requires_dynamic_flat(rt, rs_dev):
    v = torch.zeros(16, dtype=torch.uint64, device=DEV)
    for fl in (rt.OMPRT_RS_QUEUE, rt.OMPRT_RS_QUEUE | rt.OMPRT_FLAT):
        with pytest.raises(Exception):
            rt.omprt_rs_lookup(rs_dev, 1, 0, 16, v, None, 0, 128, fl)


def test_rs_flat_rejects_assumption(rt, rs_dev):
    v = torch.zeros(16, dtype=torch.uint64, device=DEV)
    with pytest.raises(Exception):
        rt.omprt_rs_lookup(rs_dev, 1, 0, 16, v, None, 0, 128,
                           rt.OMPRT_FLAT | rt.OMPRT_ASSUME_OVERSUB)


def _su3(rt, fn, A, B, n, flags=0):
    At, Bt = torch.from_numpy(A).to(DEV), torch.from_numpy(B).to(DEV)
    Ct = torch.full((n * 72,), float("nan"), dtype=torch.float64, device=DEV)
    ck = torch.full((1,), 0.5, dtype=torch.float64, device=DEV)
    fn(At, Bt, Ct, n, ck, 0, 128, flags)
    torch.cuda.synchronize()
    return Ct.cpu().numpy(), float(ck.item()) - 0.5


@pytest.mark.parametrize("n", [8 ** 4, 8 ** 4 + 5, 32 ** 4])
@pytest.mark.parametrize("variant", ["rt", "rt_loop", "twin", "rt_wstaged", "twin_wstaged",
                                     "rt_tiled", "twin_tiled"])
def test_su3_bit_exact(rt, n, variant):
    A, B = gen.su3_inputs(n)
    fn = rt.omprt_cuda_su3_mult if variant.startswith("twin") else rt.omprt_su3_mult
    flags = {"rt": rt.OMPRT_ASSUME_OVERSUB, "rt_loop": 0, "twin": 0,
             "rt_wstaged": rt.OMPRT_WARP_STAGED, "twin_wstaged": rt.OMPRT_WARP_STAGED,
             "rt_tiled": rt.OMPRT_TMA_TILED, "twin_tiled": rt.OMPRT_TMA_TILED}[variant]
    C, ck = _su3(rt, fn, A, B, n, flags)
    Cref = oracle.su3_mult(A, B, n, threads=os.cpu_count() or 1)
    assert (C == Cref).all()
    re = Cref[0::2]
    assert abs(ck - oracle.sum_f64(re)) <= 1e-12 * oracle.sum_abs_f64(re)


@pytest.mark.parametrize("flag", ["OMPRT_WARP_STAGED", "OMPRT_TMA_TILED"])
@pytest.mark.parametrize("teams", [1, 3, 148])
def test_su3_staged_geometries(rt, flag, teams):
    """Few persistent teams (many tiles per warp, both buffers cycling) and a ragged last
    tile (n not a multiple of 32) stay bit-exact."""
    n = 4 * 192 * 3 + 37
    A, B = gen.su3_inputs(n)
    At, Bt = torch.from_numpy(A).to(DEV), torch.from_numpy(B).to(DEV)
    Ct = torch.full((n * 72 + 72,), float("nan"), dtype=torch.float64, device=DEV)
    rt.omprt_su3_mult(At, Bt, Ct, n, None, teams, 128, getattr(rt, flag))
    torch.cuda.synchronize()
    C = Ct.cpu().numpy()
    assert (C[:n * 72] == oracle.su3_mult(A, B, n)).all()
    assert np.isnan(C[n * 72:]).all()  # nothing written past the last record


def test_su3_staged_flags_exclusive(rt):
    A = torch.zeros(72 * 64, dtype=torch.float64, device=DEV)
    B = torch.zeros(72, dtype=torch.float64, device=DEV)
    for both in (rt.OMPRT_TMA_TILED | rt.OMPRT_WARP_STAGED,
                 rt.OMPRT_TMA_TILED | rt.OMPRT_ASSUME_OVERSUB):
        with pytest.raises(Exception):
            rt.omprt_su3_mult(A, B, A, 64, None, 0, 128, both)


def test_su3_tma_tiled_tail_and_sass(rt):
    """The ragged last tile: the box rows past n_sites are zero-filled on the load and not
    written on the store (the C buffer's NaN guard past the last site survives), for
    every tail length; and the kernel really moves data with tensor TMA (UTMALDG/UTMASTG)."""
    for n in (1, 31, 33, 6 * 32 * 148 + 5):
        A, B = gen.su3_inputs(n)
        At, Bt = torch.from_numpy(A).to(DEV), torch.from_numpy(B).to(DEV)
        Ct = torch.full((n * 72 + 4 * 72,), float("nan"), dtype=torch.float64, device=DEV)
        ck = torch.zeros(1, dtype=torch.float64, device=DEV)
        rt.omprt_su3_mult(At, Bt, Ct, n, ck, 0, 128, rt.OMPRT_TMA_TILED)
        torch.cuda.synchronize()
        C = Ct.cpu().numpy()
        Cref = oracle.su3_mult(A, B, n)
        assert (C[:n * 72] == Cref).all() and np.isnan(C[n * 72:]).all()
    import subprocess
    so = os.path.join(os.path.dirname(rt.__file__), "libomprt.so")
    sass = subprocess.run(["cuobjdump", "-sass", so], capture_output=True, text=True).stdout
    assert "UTMALDG" in sass and "UTMASTG" in sass


def test_su3_pins_on_gpu(rt):
    n = 4096
    A, B = gen.su3_inputs(n, "identity")
    C, _ = _su3(rt, rt.omprt_su3_mult, A, B, n, rt.OMPRT_ASSUME_OVERSUB)
    assert (C == A).all()
    A, B = gen.su3_inputs(n, "third")
    C, ck = _su3(rt, rt.omprt_su3_mult, A, B, n, rt.OMPRT_ASSUME_OVERSUB)
    assert (C.reshape(n, 4, 3, 3, 2)[..., 0] == 1.0).all() and ck == 36.0 * n


def _prepared_expected(t):
    """The prepared layout written out with numpy (R-A9, R-A12): EA halved, each window's
    records stably sorted by l, the window's 4th word = its l-run boundaries."""
    P = t.poles.reshape(-1, 8)
    exp = P.copy()
    exp[:, 0] = P[:, 0] * 0.5
    exp[:, 1] = (0.0 - P[:, 1]) * 0.5
    W = t.windows.reshape(-1, 4).copy()
    runs = np.zeros(W.shape[0], dtype=np.uint64)
    out = exp.copy()
    for w, (s, e) in enumerate(t.win_range.reshape(-1, 2)):
        ls = t.pole_l[s:e]
        order = np.argsort(ls, kind="stable")
        out[s:e] = exp[s:e][order]
        c = [int((ls < k).sum()) for k in (1, 2, 3)]
        runs[w] = c[0] | (c[1] << 21) | (c[2] << 42)
    W.view(np.uint64)[:, 3] = runs
    # material entries (R-A13): k0rs of the nuclide, conc, win_off | n_windows << 32
    n_mats, mx = t.num_nucs.shape[0], t.max_num_nucs
    MN = np.zeros((n_mats * mx, 8))
    mats, concs = t.mats.reshape(n_mats, mx), t.concs.reshape(n_mats, mx)
    for m in range(n_mats):
        for j in range(int(t.num_nucs[m])):
            nuc = int(mats[m, j])
            r = MN[m * mx + j]
            r[0:4] = t.k0rs.reshape(-1, 4)[nuc]
            r[4] = concs[m, j]
            r.view(np.uint64)[5] = np.uint64(int(t.win_off[nuc]) | (int(t.n_windows[nuc]) << 32))
    return out, W, MN


def test_rs_prepare_pole_records(rt, rs_tables_small):
    """omprt_rs_prepare: EA.re / 2 and (0 - EA.im) / 2, the rest of each record unchanged --
    exactly the values numpy's IEEE arithmetic gives --, each window's records stably
    sorted by l and its l-run boundaries in the window record (R-A12); an unprepared or
    twice-prepared table is rejected."""
    d = rt.RSDeviceTables(rs_tables_small, DEV)
    got = d.poles_prepared.cpu().numpy().reshape(-1, 8)
    gotw = d.windows_prepared.cpu().numpy().reshape(-1, 4)
    gotm = d.matnuc.cpu().numpy().reshape(-1, 8)
    exp, expw, expm = _prepared_expected(rs_tables_small)
    assert (got.view(np.uint64) == exp.view(np.uint64)).all()
    assert (gotw.view(np.uint64) == expw.view(np.uint64)).all()
    assert (gotm.view(np.uint64) == expm.view(np.uint64)).all()
    assert d.c.prepared == 1
    with pytest.raises(rt.OmprtError):
        rt.omprt_rs_prepare(d, exp.shape[0], gotw.shape[0], d.n_mats, d.poles_prepared,
                            d.windows_prepared, d.matnuc)
    raw = rt.RSTablesC.from_buffer_copy(d.c)
    raw.prepared = 0
    d.c = raw
    v = torch.zeros(16, dtype=torch.uint64, device=DEV)
    with pytest.raises(rt.OmprtError):
        rt.omprt_rs_lookup(d, 1, 0, 16, v)


@pytest.mark.parametrize("defect", ["overlap", "l_range", "past_end", "nuclide", "n_windows"])
def test_rs_prepare_rejects_unsortable_windows(rt, rs_tables_small, defect):
    """Windows that overlap (their poles cannot be sorted independently), an l outside
    [0, 4), a range past the last pole, a material entry naming no nuclide or a nuclide
    whose windows run past the table's: omprt_rs_prepare fails with OMPRT_E_INVAL."""
    import copy
    t = copy.copy(rs_tables_small)
    t.win_range = rs_tables_small.win_range.copy()
    t.pole_l = rs_tables_small.pole_l.copy()
    t.mats = rs_tables_small.mats.copy()
    if defect == "overlap":
        t.win_range[5, 0] = t.win_range[4, 1] - 1
    elif defect == "l_range":
        t.pole_l[t.win_range[7, 0]] = 4
    elif defect == "past_end":
        t.win_range[-1, 1] = t.poles.shape[0] + 1
    elif defect == "nuclide":
        t.mats.reshape(-1)[3] = t.n_nuclides
    else:  # a nuclide's windows past the table's
        t.n_windows = rs_tables_small.n_windows.copy()
        t.n_windows[int(t.mats.reshape(-1)[0])] += 10_000
    with pytest.raises(rt.OmprtError):
        rt.RSDeviceTables(t, DEV)


@pytest.mark.parametrize("scale", [3.0, 30.0])
def test_rs_sigt_factor_angles_beyond_the_series_range(rt, rs_tables_small, scale):
    """The sigT factors outside the workload's angle range (k0rs scaled by 3: angles 2 k0rs
    sqrt(E) up to 6, past the first quadrant boundaries of the rational-rotation form,
    R-A10; by 30: up to 60, every quadrant of the sincos reduction many times over)
    still match the oracle within the C7 contract."""
    import copy
    t = copy.copy(rs_tables_small)
    t.k0rs = rs_tables_small.k0rs * scale
    d = rt.RSDeviceTables(t, DEV)
    first, count = 11, 5_000
    ver, mac = _rs(rt, d, first, count, "rt", rt.OMPRT_FLAT | rt.OMPRT_SCHED_DYNAMIC)
    rv, rm = oracle.rs_lookup(t, first, count, want_macro=True, threads=os.cpu_count() or 1)
    err = np.abs(mac - rm).max(axis=1) / np.abs(rm).max(axis=1)
    assert err.max() <= 1e-10, err.max()
