"""ctypes wrapper of the CPU oracle (oracle/oracle.c).

TEST INFRASTRUCTURE.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline and
`--impl reference` legs may import this package.  The product path
(paper_conf_ipps_doerfertphtdcg22_b200) never imports it and fails loudly without its CUDA
library.  The oracle shares no code with the CUDA path; inputs come from `gen/`.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c11", "-fPIC", "-shared"]


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain C, no CUDA)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "oracle.h"))):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            _lib = C.CDLL(_LIB)
            _declare(_lib)
    return _lib


_i32p = C.POINTER(C.c_int32)
_i64p = C.POINTER(C.c_int64)
_u64p = C.POINTER(C.c_uint64)
_f64p = C.POINTER(C.c_double)


class XSTablesC(C.Structure):
    _fields_ = [("n_isotopes", C.c_int32), ("n_gridpoints", C.c_int32),
                ("max_num_nucs", C.c_int32), ("pad", C.c_int32), ("n_union", C.c_int64),
                ("nuclide_grid", _f64p), ("unionized", _f64p), ("index_grid", _i32p),
                ("num_nucs", _i32p), ("mats", _i32p), ("concs", _f64p)]


class RSTablesC(C.Structure):
    _fields_ = [("n_nuclides", C.c_int32), ("numL", C.c_int32), ("max_num_nucs", C.c_int32),
                ("pad", C.c_int32), ("poles", _f64p), ("pole_l", _i32p), ("windows", _f64p),
                ("win_range", _i32p), ("win_off", _i32p), ("n_windows", _i32p),
                ("k0rs", _f64p), ("num_nucs", _i32p), ("mats", _i32p), ("concs", _f64p)]


def _declare(L):
    sig = {
        "oracle_static_owner_closed": (C.c_int, [C.c_int64, C.c_int64, C.c_int64, C.c_int64, _i32p, _i32p]),
        "oracle_fig5_simulate": (None, [C.c_int64, C.c_int32, C.c_int32, C.c_int, _i32p, _i32p]),
        "oracle_team_for_simulate": (None, [C.c_int64, C.c_int32, C.c_int, _i32p, _i32p]),
        "oracle_distribute_simulate": (None, [C.c_int64, C.c_int32, _i32p, _i32p]),
        "oracle_static_chunk_owner_closed": (C.c_int, [C.c_int64, C.c_int64, C.c_int64, C.c_int64, C.c_int64, _i32p, _i32p]),
        "oracle_chunk_simulate": (None, [C.c_int64, C.c_int64, C.c_int32, C.c_int32, C.c_int, _i32p, _i32p]),
        "oracle_dynamic_team_closed": (C.c_int, [C.c_int64, C.c_int64, C.c_int64]),
        "oracle_dynamic_simulate": (None, [C.c_int64, C.c_int64, C.c_int32, C.c_int32, C.c_uint64, _i32p, _i32p]),
        "oracle_axpy": (None, [C.c_int64, C.c_double, _f64p, _f64p, _f64p]),
        "oracle_sum_f64": (C.c_double, [_f64p, C.c_int64, C.c_double]),
        "oracle_sum_f64_ld": (C.c_longdouble, [_f64p, C.c_int64, C.c_double]),
        "oracle_sum_abs_f64": (C.c_double, [_f64p, C.c_int64]),
        "oracle_reduce_u64": (C.c_uint64, [_u64p, C.c_int64, C.c_int, C.c_uint64]),
        "oracle_reduce_f64": (C.c_double, [_f64p, C.c_int64, C.c_int, C.c_double]),
        "oracle_generic_team": (None, [C.c_int32, C.c_int32, C.c_int32, _f64p, _f64p, _i32p, _f64p]),
        "oracle_icv_table": (None, [C.c_int32, C.c_int32, C.c_int32, _i32p]),
        "oracle_lcg_fast_forward": (C.c_uint64, [C.c_uint64, C.c_uint64]),
        "oracle_lcg_step": (C.c_uint64, [C.c_uint64, C.c_uint64]),
        "oracle_lcg_double": (C.c_double, [_u64p]),
        "oracle_pick_mat": (C.c_int, [_u64p]),
        "oracle_grid_search": (C.c_int64, [_f64p, C.c_int64, C.c_double]),
        "oracle_xs_lookup": (C.c_int, [C.POINTER(XSTablesC), C.c_uint64, C.c_int64, C.c_int64, _u64p, _f64p]),
        "oracle_xs_lookup_nuclide_search": (C.c_int, [C.POINTER(XSTablesC), C.c_uint64, C.c_int64, C.c_int64, _u64p, _f64p]),
        "oracle_xs_bytes": (C.c_int64, [C.POINTER(XSTablesC), C.c_uint64, C.c_int64, C.c_int64]),
        "oracle_fast_exp": (C.c_double, [C.c_double]),
        "oracle_fast_nuclear_W": (None, [C.c_double, C.c_double, _f64p, _f64p]),
        "oracle_rs_lookup": (C.c_int, [C.POINTER(RSTablesC), C.c_uint64, C.c_int64, C.c_int64, _u64p, _f64p]),
        "oracle_rs_count": (None, [C.POINTER(RSTablesC), C.c_uint64, C.c_int64, C.c_int64, _i64p]),
        "oracle_su3_mult": (None, [_f64p, _f64p, _f64p, C.c_int64]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args


def _p(a, t):
    return a.ctypes.data_as(t) if a is not None else None


def _c(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


# ------------------------------------------------------------------------------ schedule
def static_owner_closed(iv, n, teams, threads):
    tm, th = C.c_int32(), C.c_int32()
    r = lib().oracle_static_owner_closed(iv, n, teams, threads, C.byref(tm), C.byref(th))
    return None if r else (tm.value, th.value)


def fig5_simulate(n, teams, threads, assume_oversub=False):
    owner = np.empty(n, np.int32)
    count = np.empty(n, np.int32)
    lib().oracle_fig5_simulate(n, teams, threads, int(assume_oversub), _p(owner, _i32p), _p(count, _i32p))
    return owner, count


def team_for_simulate(n, nthreads, assume_oversub=False):
    owner = np.empty(n, np.int32)
    count = np.empty(n, np.int32)
    lib().oracle_team_for_simulate(n, nthreads, int(assume_oversub), _p(owner, _i32p), _p(count, _i32p))
    return owner, count


def distribute_simulate(n, teams):
    owner = np.empty(n, np.int32)
    count = np.empty(n, np.int32)
    lib().oracle_distribute_simulate(n, teams, _p(owner, _i32p), _p(count, _i32p))
    return owner, count


def static_chunk_owner_closed(iv, n, chunk, teams, threads):
    tm, th = C.c_int32(), C.c_int32()
    r = lib().oracle_static_chunk_owner_closed(iv, n, chunk, teams, threads, C.byref(tm), C.byref(th))
    return None if r else (tm.value, th.value)


def chunk_simulate(n, chunk, teams, threads, assume_oversub=False):
    owner = np.empty(n, np.int32)
    count = np.empty(n, np.int32)
    lib().oracle_chunk_simulate(n, chunk, teams, threads, int(assume_oversub), _p(owner, _i32p),
                                _p(count, _i32p))
    return owner, count


def dynamic_team_closed(iv, n, teams):
    r = lib().oracle_dynamic_team_closed(iv, n, teams)
    return None if r < 0 else r


def dynamic_simulate(n, chunk, teams, threads, order_seed=0):
    owner = np.empty(n, np.int32)
    count = np.empty(n, np.int32)
    lib().oracle_dynamic_simulate(n, chunk, teams, threads, order_seed, _p(owner, _i32p),
                                  _p(count, _i32p))
    return owner, count


# ------------------------------------------------------------------------------ C1
def axpy(x, b, c):
    b, c = _c(b, np.float64), _c(c, np.float64)
    a = np.empty_like(b)
    lib().oracle_axpy(b.size, x, _p(b, _f64p), _p(c, _f64p), _p(a, _f64p))
    return a


def sum_f64(v, init=0.0):
    v = _c(v, np.float64)
    return lib().oracle_sum_f64(_p(v, _f64p), v.size, init)


def sum_f64_ld(v, init=0.0):
    v = _c(v, np.float64)
    return lib().oracle_sum_f64_ld(_p(v, _f64p), v.size, init)


def sum_abs_f64(v):
    v = _c(v, np.float64)
    return lib().oracle_sum_abs_f64(_p(v, _f64p), v.size)


OP_ADD, OP_MUL, OP_MIN, OP_MAX = 0, 1, 2, 3


def reduce_u64(v, op, orig):
    v = _c(v, np.uint64)
    return lib().oracle_reduce_u64(_p(v, _u64p), v.size, op, orig)


def reduce_f64(v, op, orig):
    v = _c(v, np.float64)
    return lib().oracle_reduce_f64(_p(v, _f64p), v.size, op, orig)


# ------------------------------------------------------------------------------ C2
def generic_team(teams, nthreads, inner_n, inp):
    inp = _c(inp, np.float64)
    out = np.empty(teams * inner_n, np.float64)
    owner = np.empty(teams * inner_n, np.int32)
    post = np.empty(teams, np.float64)
    lib().oracle_generic_team(teams, nthreads, inner_n, _p(inp, _f64p), _p(out, _f64p),
                              _p(owner, _i32p), _p(post, _f64p))
    return out, owner, post


ICV_FIELDS = 7


def icv_table(teams, nthreads, nested_request):
    rec = np.empty((teams, 1 + 3 * nthreads, ICV_FIELDS), np.int32)
    lib().oracle_icv_table(teams, nthreads, nested_request, _p(rec, _i32p))
    return rec


# ------------------------------------------------------------------------------ C3
def lcg_fast_forward(seed, n):
    return lib().oracle_lcg_fast_forward(seed, n)


def lcg_step(seed, n):
    return lib().oracle_lcg_step(seed, n)


def lcg_double(seed):
    s = C.c_uint64(seed)
    d = lib().oracle_lcg_double(C.byref(s))
    return d, s.value


def pick_mat(seed):
    s = C.c_uint64(seed)
    m = lib().oracle_pick_mat(C.byref(s))
    return m, s.value


def grid_search(A, quarry):
    A = _c(A, np.float64)
    return lib().oracle_grid_search(_p(A, _f64p), A.size, quarry)


def xs_struct(t):
    """Keeps references alive on the returned struct."""
    s = XSTablesC(t.n_isotopes, t.n_gridpoints, t.max_num_nucs, 0, t.n_union,
                  _p(t.nuclide_grid, _f64p), _p(t.unionized, _f64p), _p(t.index_grid, _i32p),
                  _p(t.num_nucs, _i32p), _p(t.mats, _i32p), _p(t.concs, _f64p))
    s._keep = t
    return s


def _parallel_ranges(count, threads):
    threads = max(1, min(threads, count))
    edges = [count * k // threads for k in range(threads + 1)]
    return [(edges[k], edges[k + 1] - edges[k]) for k in range(threads)]


def _run_threads(fn, count, threads):
    """Independent units partitioned into contiguous blocks over `threads` OS threads;
    ctypes releases the GIL, so the C oracle runs in parallel (semantics unchanged)."""
    if threads <= 1:
        fn(0, count)
        return
    ts = [threading.Thread(target=fn, args=r) for r in _parallel_ranges(count, threads)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()


def xs_lookup(t, first, count, seed=1070, want_macro=False, threads=1, nuclide_search=False):
    s = xs_struct(t)
    ver = np.empty(count, np.uint64)
    mac = np.empty((count, 5), np.float64) if want_macro else None
    f = lib().oracle_xs_lookup_nuclide_search if nuclide_search else lib().oracle_xs_lookup

    def run(off, cnt):
        if cnt:
            f(C.byref(s), seed, first + off, cnt, _p(ver[off:], _u64p),
              _p(mac[off:], _f64p) if mac is not None else None)
    _run_threads(run, count, threads)
    return (ver, mac) if want_macro else ver


def xs_bytes(t, first, count, seed=1070):
    s = xs_struct(t)
    return lib().oracle_xs_bytes(C.byref(s), seed, first, count)


# ------------------------------------------------------------------------------ C4
def fast_exp(x):
    return lib().oracle_fast_exp(x)


def fast_nuclear_W(z):
    wr, wi = C.c_double(), C.c_double()
    lib().oracle_fast_nuclear_W(z.real, z.imag, C.byref(wr), C.byref(wi))
    return complex(wr.value, wi.value)


def rs_struct(t):
    s = RSTablesC(t.n_nuclides, t.numL, t.max_num_nucs, 0, _p(t.poles, _f64p), _p(t.pole_l, _i32p),
                  _p(t.windows, _f64p), _p(t.win_range, _i32p), _p(t.win_off, _i32p),
                  _p(t.n_windows, _i32p), _p(t.k0rs, _f64p), _p(t.num_nucs, _i32p),
                  _p(t.mats, _i32p), _p(t.concs, _f64p))
    s._keep = t
    return s


def rs_lookup(t, first, count, seed=1070, want_macro=False, threads=1):
    s = rs_struct(t)
    ver = np.empty(count, np.uint64)
    mac = np.empty((count, 4), np.float64) if want_macro else None

    def run(off, cnt):
        if cnt:
            lib().oracle_rs_lookup(C.byref(s), seed, first + off, cnt, _p(ver[off:], _u64p),
                                   _p(mac[off:], _f64p) if mac is not None else None)
    _run_threads(run, count, threads)
    return (ver, mac) if want_macro else ver


def rs_count(t, first, count, seed=1070):
    s = rs_struct(t)
    ops = np.zeros(10, np.int64)
    lib().oracle_rs_count(C.byref(s), seed, first, count, _p(ops, _i64p))
    return ops


# ------------------------------------------------------------------------------ C5
def su3_mult(A, B, n_sites, threads=1):
    A, B = _c(A, np.float64), _c(B, np.float64)
    Cout = np.empty(n_sites * 72, np.float64)

    def run(off, cnt):
        if cnt:
            lib().oracle_su3_mult(_p(A[off * 72:], _f64p), _p(B, _f64p),
                                  _p(Cout[off * 72:], _f64p), cnt)
    _run_threads(run, n_sites, threads)
    return Cout
