"""Thin ctypes binding of libomprt.so (include/omprt.h): argument marshalling only.

Every function has the C name and the C argument order; device buffers are torch CUDA
tensors (PyTorch supplies memory, streams and process groups -- nothing else), host buffers
for `_host` calls are numpy arrays.  A nonzero status raises OmprtError.  There is no CPU
fallback: without the built library (or on a machine without a GPU) every call fails.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libomprt.so")

OMPRT_OK = 0
OMPRT_E_INVAL = -1
OMPRT_E_CUDA = -2
OMPRT_E_NOMEM = -3
OMPRT_E_STACK = -4
OMPRT_E_ASSERT = -5
OMPRT_E_NOTINIT = -6

OMPRT_ASSUME_OVERSUB = 1 << 0
OMPRT_RECORD_OWNER = 1 << 1
OMPRT_GENERAL_SM = 1 << 2
OMPRT_SMALL_STACK = 1 << 3
OMPRT_NO_STACK = 1 << 4
OMPRT_DEBUG_BUILD = 1 << 5
OMPRT_POSTLOGUE = 1 << 6
OMPRT_THREAD_STATES = 1 << 7
OMPRT_FUSED_REDUCTION = 1 << 8
OMPRT_UNCHECKED = 1 << 9
OMPRT_XS_ACCEL = 1 << 10
OMPRT_SPMDIZE = 1 << 11
OMPRT_DEGLOBALIZE = 1 << 12
OMPRT_WARP_STAGED = 1 << 14
OMPRT_XS_FLAT = 1 << 15
OMPRT_FLAT = OMPRT_XS_FLAT  # omprt_rs_lookup: flattened nuclide loop, persistent grid
OMPRT_SCHED_DYNAMIC = 1 << 17  # schedule(dynamic, C): team blocks, team-shared chunk counter
OMPRT_TMA_TILED = 1 << 18  # SU(3): one 2-D TMA tensor copy per warp tile, padded slots
OMPRT_TMA_STREAM = 1 << 19  # axpy: Fig. 5 loop with operands streamed by 2-D TMA boxes
OMPRT_RS_QUEUE = 1 << 20  # RSBench: Abrarov poles queued per warp, drained by all lanes (R-A8)
OMPRT_XS_NO_L2_PERSIST = 1 << 16

# Every symbol include/omprt.h declares (checked by tests/test_abi.py).
EXPORTS = [
    "omprt_init", "omprt_fini", "omprt_l2_reset_persisting", "omprt_l2_set_aside", "omprt_device_status", "omprt_last_error", "omprt_static_owner",
    "omprt_spmd_axpy_sum", "omprt_cuda_axpy_sum", "omprt_spmd_axpy_sum_chunked",
    "omprt_cuda_axpy_sum_chunked", "omprt_generic_team", "omprt_cuda_generic_team",
    "omprt_icv_probe", "omprt_lockstep_probe", "omprt_xs_lookup", "omprt_cuda_xs_lookup", "omprt_u64_sum",
    "omprt_xs_run_host", "omprt_xs_run_host_steps", "omprt_xs_accel_sizes", "omprt_xs_build_accel",
    "omprt_xs_derive_tmp_bytes", "omprt_xs_derive", "omprt_rs_lookup", "omprt_cuda_rs_lookup", "omprt_su3_mult",
    "omprt_cuda_su3_mult", "omprt_kernel_count", "omprt_kernel_name", "omprt_kernel_attrs",
    "omprt_probe_l2_read", "omprt_probe_fp64_fma", "omprt_probe_hbm_stream", "omprt_kernel_occupancy", "omprt_rs_prepare",
]


class OmprtError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"omprt error {code}: {msg}")
        self.code = code


class Options(C.Structure):
    _fields_ = [("pool_bytes_per_team", C.c_uint64), ("pool_teams", C.c_uint64),
                ("max_teams", C.c_uint64)]


class XSTablesC(C.Structure):
    _fields_ = [("nuclide_grid", C.c_void_p), ("unionized", C.c_void_p), ("index_grid", C.c_void_p),
                ("num_nucs", C.c_void_p), ("mats", C.c_void_p), ("concs", C.c_void_p),
                ("n_isotopes", C.c_int32), ("n_gridpoints", C.c_int32),
                ("max_num_nucs", C.c_int32), ("pad", C.c_int32), ("n_union", C.c_int64),
                ("bins", C.c_void_p), ("index_grid16", C.c_void_p), ("brackets", C.c_void_p),
                ("log2_bins", C.c_int32), ("pad2", C.c_int32)]


class RSTablesC(C.Structure):
    _fields_ = [("poles", C.c_void_p), ("pole_l", C.c_void_p), ("windows", C.c_void_p),
                ("win_range", C.c_void_p), ("win_off", C.c_void_p), ("n_windows", C.c_void_p),
                ("k0rs", C.c_void_p), ("num_nucs", C.c_void_p), ("mats", C.c_void_p),
                ("concs", C.c_void_p), ("matnuc", C.c_void_p), ("n_nuclides", C.c_int32),
                ("numL", C.c_int32),
                ("max_num_nucs", C.c_int32), ("prepared", C.c_int32)]


_lib = None
_vp, _i32, _i64, _u32, _u64, _f64 = C.c_void_p, C.c_int32, C.c_int64, C.c_uint32, C.c_uint64, C.c_double
_SIGS = {
    "omprt_init": [C.c_int, C.POINTER(Options)],
    "omprt_fini": [C.c_int],
    "omprt_l2_reset_persisting": [],
    "omprt_l2_set_aside": [C.c_uint64, C.POINTER(C.c_uint64)],
    "omprt_device_status": [C.c_int, C.POINTER(C.c_int), C.POINTER(C.c_int)],
    "omprt_last_error": [C.c_char_p, C.c_size_t],
    "omprt_static_owner": [_i64, _i64, _i32, _i32, C.POINTER(_i32), C.POINTER(_i32)],
    "omprt_spmd_axpy_sum": [_i64, _f64, _vp, _vp, _vp, _vp, _i32, _i32, _u32, _vp, _vp, _vp],
    "omprt_cuda_axpy_sum": [_i64, _f64, _vp, _vp, _vp, _vp, _i32, _i32, _u32, _vp, _vp, _vp],
    "omprt_spmd_axpy_sum_chunked": [_i64, _i64, _f64, _vp, _vp, _vp, _vp, _i32, _i32, _u32, _vp,
                                    _vp, _vp],
    "omprt_cuda_axpy_sum_chunked": [_i64, _i64, _f64, _vp, _vp, _vp, _vp, _i32, _i32, _u32, _vp,
                                    _vp, _vp],
    "omprt_generic_team": [_i32, _i32, _i32, _vp, _vp, _vp, _vp, _u32, _vp],
    "omprt_cuda_generic_team": [_i32, _i32, _i32, _vp, _vp, _vp, _vp, _u32, _vp],
    "omprt_icv_probe": [_i32, _i32, _i32, _vp, _u32, _vp],
    "omprt_lockstep_probe": [_i64, _i32, _i32, _i32, _vp, _vp, _vp, _vp],
    "omprt_xs_lookup": [XSTablesC, _u64, _i64, _i64, _vp, _vp, _vp, _i32, _i32, _u32, _vp],
    "omprt_cuda_xs_lookup": [XSTablesC, _u64, _i64, _i64, _vp, _vp, _vp, _i32, _i32, _u32, _vp],
    "omprt_u64_sum": [_vp, _i64, _vp, _vp],
    "omprt_xs_accel_sizes": [_i32, _i32, _i64, _i32, C.POINTER(_u64)],
    "omprt_xs_build_accel": [C.POINTER(XSTablesC), _vp, _vp, _vp, _i32, _vp],
    "omprt_xs_derive_tmp_bytes": [_i32, _i32, C.POINTER(_u64)],
    "omprt_xs_derive": [_vp, _i32, _i32, _vp, _vp, _vp, _u64, _vp],
    "omprt_xs_run_host": [XSTablesC, _u64, _i64, _i64, _i32, _u32, C.POINTER(_u64),
                          C.POINTER(_u64), C.POINTER(_u64), _vp],
    "omprt_xs_run_host_steps": [XSTablesC, _u64, _i64, _i64, _i32, _u32, _i32, C.POINTER(_u64),
                                C.POINTER(_u64), C.POINTER(_u64), _vp],
    "omprt_rs_prepare": [C.POINTER(RSTablesC), _i64, _i64, _i32, _vp, _vp, _vp, _vp],
    "omprt_rs_lookup": [RSTablesC, _u64, _i64, _i64, _vp, _vp, _i32, _i32, _u32, _vp],
    "omprt_cuda_rs_lookup": [RSTablesC, _u64, _i64, _i64, _vp, _vp, _i32, _i32, _u32, _vp],
    "omprt_su3_mult": [_vp, _vp, _vp, _i64, _vp, _i32, _i32, _u32, _vp],
    "omprt_cuda_su3_mult": [_vp, _vp, _vp, _i64, _vp, _i32, _i32, _u32, _vp],
    "omprt_probe_l2_read": [_vp, _u64, _i32, _i32, _i32, _i32, _vp, _vp],
    "omprt_probe_fp64_fma": [_i64, _i32, _vp, _vp],
    "omprt_probe_hbm_stream": [_vp, _vp, _u64, _i32, _i32, _vp, _vp],
    "omprt_kernel_count": [],
    "omprt_kernel_occupancy": [C.c_int, C.c_int, C.c_int, C.POINTER(C.c_int)],
    "omprt_kernel_name": [C.c_int],
    "omprt_kernel_attrs": [C.c_int, C.POINTER(C.c_int), C.POINTER(C.c_int), C.POINTER(C.c_int),
                           C.POINTER(C.c_int)],
}


def load(path: str = LIB_PATH):
    """Load libomprt.so (raises if it was not built -- there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(path):
            raise OSError(f"{path} is missing: run __graft_entry__.build() (no CPU fallback)")
        lib = C.CDLL(path)
        for name, args in _SIGS.items():
            f = getattr(lib, name)
            f.argtypes = args
            f.restype = C.c_char_p if name == "omprt_kernel_name" else C.c_int
        _lib = lib
    return _lib


def last_error() -> str:
    buf = C.create_string_buffer(512)
    load().omprt_last_error(buf, 512)
    return buf.value.decode(errors="replace")


def _check(code):
    if code != OMPRT_OK:
        raise OmprtError(code, last_error())
    return code


def _p(t, dtype=None, n=None):
    """Device pointer of a torch CUDA tensor (None -> NULL).  Checks what the C ABI cannot:
    contiguous, on the current CUDA device, of the element type the ABI expects (`dtype`,
    a torch dtype or a tuple of them) and holding at least `n` elements -- a wrong tensor is
    a ValueError here, not an out-of-bounds device access."""
    if t is None:
        return None
    if not t.is_cuda:
        raise ValueError("expected a CUDA tensor")
    if not t.is_contiguous():
        raise ValueError("expected a contiguous tensor")
    import torch
    if t.device.index != torch.cuda.current_device():
        raise ValueError(f"tensor on {t.device}, current device is cuda:{torch.cuda.current_device()}")
    if dtype is not None and t.dtype not in (dtype if isinstance(dtype, tuple) else (dtype,)):
        raise ValueError(f"expected dtype {dtype}, got {t.dtype}")
    if n is not None and t.numel() < n:
        raise ValueError(f"tensor holds {t.numel()} elements, the call needs {n}")
    return t.data_ptr()


def _T():
    import torch
    return torch


def _hp(a):
    """Host pointer of a numpy array or pinned torch CPU tensor."""
    if a is None:
        return None
    if hasattr(a, "ctypes"):
        return a.ctypes.data
    return a.data_ptr()


def _stream(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    return stream if isinstance(stream, int) else stream.cuda_stream


# ---------------------------------------------------------------- lifecycle / status
def omprt_init(device=0, pool_bytes_per_team=0, pool_teams=0, max_teams=0):
    o = Options(pool_bytes_per_team, pool_teams, max_teams)
    return _check(load().omprt_init(device, C.byref(o)))


def omprt_fini(device=0):
    return _check(load().omprt_fini(device))


def omprt_l2_reset_persisting():
    """Return persisting L2 lines (OMPRT_XS_FLAT's access-policy window) to normal; call
    with no launch in flight."""
    return _check(load().omprt_l2_reset_persisting())


def omprt_l2_set_aside(nbytes):
    """Resize the L2 set-aside for persisting accesses (0 removes it); returns the size
    granted."""
    got = C.c_uint64()
    _check(load().omprt_l2_set_aside(nbytes, C.byref(got)))
    return got.value


def omprt_device_status(device=0):
    code, info = C.c_int(), (C.c_int * 4)()
    _check(load().omprt_device_status(device, C.byref(code), info))
    return code.value, list(info)


def omprt_static_owner(iv, n, teams, threads):
    tm, th = _i32(), _i32()
    _check(load().omprt_static_owner(iv, n, teams, threads, C.byref(tm), C.byref(th)))
    return tm.value, th.value


# ---------------------------------------------------------------- C1
def _axpy_ptrs(n, b, c, a, sum_inout, owner, count):
    f64, i32, m = _T().float64, _T().int32, max(int(n), 0)
    return (_p(b, f64, m), _p(c, f64, m), _p(a, f64, m), _p(sum_inout, f64, 1),
            _p(owner, i32, m), _p(count, i32, m))


def omprt_spmd_axpy_sum(n, x, b, c, a, sum_inout, teams, threads, flags=0, owner=None,
                        count=None, stream=None):
    pb, pc, pa, ps, po, pn = _axpy_ptrs(n, b, c, a, sum_inout, owner, count)
    return _check(load().omprt_spmd_axpy_sum(n, x, pb, pc, pa, ps, teams, threads, flags, po, pn,
                                             _stream(stream)))


def omprt_cuda_axpy_sum(n, x, b, c, a, sum_inout, teams, threads, flags=0, owner=None,
                        count=None, stream=None):
    pb, pc, pa, ps, po, pn = _axpy_ptrs(n, b, c, a, sum_inout, owner, count)
    return _check(load().omprt_cuda_axpy_sum(n, x, pb, pc, pa, ps, teams, threads, flags, po, pn,
                                             _stream(stream)))


def omprt_spmd_axpy_sum_chunked(n, chunk, x, b, c, a, sum_inout, teams, threads, flags=0,
                                owner=None, count=None, stream=None):
    pb, pc, pa, ps, po, pn = _axpy_ptrs(n, b, c, a, sum_inout, owner, count)
    return _check(load().omprt_spmd_axpy_sum_chunked(n, chunk, x, pb, pc, pa, ps, teams, threads,
                                                     flags, po, pn, _stream(stream)))


def omprt_cuda_axpy_sum_chunked(n, chunk, x, b, c, a, sum_inout, teams, threads, flags=0,
                                owner=None, count=None, stream=None):
    pb, pc, pa, ps, po, pn = _axpy_ptrs(n, b, c, a, sum_inout, owner, count)
    return _check(load().omprt_cuda_axpy_sum_chunked(n, chunk, x, pb, pc, pa, ps, teams, threads,
                                                     flags, po, pn, _stream(stream)))


# ---------------------------------------------------------------- C2
def _generic_ptrs(teams, inner_n, inp, out, owner, postlogue):
    f64, m = _T().float64, max(int(teams) * int(inner_n), 0)
    return (_p(inp, f64, m), _p(out, f64, m), _p(owner, _T().int32, m),
            _p(postlogue, f64, max(int(teams), 0)))


def omprt_generic_team(teams, threads, inner_n, inp, out, owner=None, postlogue=None, flags=0,
                       stream=None):
    pi, po, pw, pp = _generic_ptrs(teams, inner_n, inp, out, owner, postlogue)
    return _check(load().omprt_generic_team(teams, threads, inner_n, pi, po, pw, pp, flags,
                                            _stream(stream)))


def omprt_cuda_generic_team(teams, threads, inner_n, inp, out, owner=None, postlogue=None,
                            flags=0, stream=None):
    pi, po, pw, pp = _generic_ptrs(teams, inner_n, inp, out, owner, postlogue)
    return _check(load().omprt_cuda_generic_team(teams, threads, inner_n, pi, po, pw, pp, flags,
                                                 _stream(stream)))


def omprt_icv_probe(teams, threads, nested_request, rec, flags=0, stream=None):
    return _check(load().omprt_icv_probe(teams, threads, nested_request, _p(rec), flags,
                                         _stream(stream)))


def omprt_lockstep_probe(n, teams, threads, dynamic, steps, hooks, errors, stream=None):
    return _check(load().omprt_lockstep_probe(n, teams, threads, int(dynamic), _p(steps),
                                              _p(hooks), _p(errors), _stream(stream)))


# ---------------------------------------------------------------- C3
class XSDeviceTables:
    """Device copies (torch tensors) of gen.XSTables and the by-value C struct.  With
    accel=True the B200 layouts are built on the device (omprt_xs_build_accel); packed=True
    (default) puts the unionized grid, the search bins and the bracket records in one
    allocation, in that order, so the flattened launch's L2 persisting window covers all
    three (xsbench.cuh flat_launch)."""

    def __init__(self, t, device="cuda", accel=False, log2_bins=18, packed=True):
        import torch
        self.host = t
        self.nuclide_grid = torch.from_numpy(t.nuclide_grid).to(device)
        self.unionized = torch.from_numpy(t.unionized).to(device)
        self.index_grid = torch.from_numpy(t.index_grid).to(device)
        self.num_nucs = torch.from_numpy(t.num_nucs).to(device)
        self.mats = torch.from_numpy(t.mats).to(device)
        self.concs = torch.from_numpy(t.concs).to(device)
        self.c = XSTablesC(_p(self.nuclide_grid), _p(self.unionized), _p(self.index_grid),
                           _p(self.num_nucs), _p(self.mats), _p(self.concs), t.n_isotopes,
                           t.n_gridpoints, t.max_num_nucs, 0, t.n_union, None, None, None, 0, 0)
        if accel:
            sizes = omprt_xs_accel_sizes(t.n_isotopes, t.n_gridpoints, t.n_union, log2_bins)
            self.index_grid16 = torch.empty(sizes[1] // 2, dtype=torch.uint16, device=device)
            if packed:  # [unionized | bins | brackets] in one allocation: one L2 window
                al = lambda b: (b + 255) // 256 * 256
                nu = al(8 * t.n_union)
                nb = al(sizes[0])
                self._pack = torch.empty(nu + nb + sizes[2], dtype=torch.uint8, device=device)
                self.unionized = self._pack[: 8 * t.n_union].view(torch.float64)
                self.unionized.copy_(torch.from_numpy(t.unionized))
                self.c.unionized = _p(self.unionized)
                self.bins = self._pack[nu: nu + sizes[0]].view(torch.int32)
                self.brackets = self._pack[nu + nb:].view(torch.float64)
            else:
                self.bins = torch.empty(sizes[0] // 4, dtype=torch.int32, device=device)
                self.brackets = torch.empty(sizes[2] // 8, dtype=torch.float64, device=device)
            omprt_xs_build_accel(self, self.bins, self.index_grid16, self.brackets, log2_bins)

    def plain(self):
        """A view of the same tables without the accelerated layouts."""
        v = XSDeviceTables.__new__(XSDeviceTables)
        v.__dict__.update(self.__dict__)
        v.c = XSTablesC.from_buffer_copy(self.c)
        v.c.bins = v.c.index_grid16 = v.c.brackets = None
        v.c.log2_bins = 0
        return v


def omprt_xs_accel_sizes(n_isotopes, n_gridpoints, n_union, log2_bins=18):
    sz = (_u64 * 3)()
    _check(load().omprt_xs_accel_sizes(n_isotopes, n_gridpoints, n_union, log2_bins, sz))
    return list(sz)


def omprt_xs_build_accel(tables, bins, index_grid16, brackets, log2_bins=18, stream=None):
    return _check(load().omprt_xs_build_accel(C.byref(tables.c), _p(bins), _p(index_grid16),
                                              _p(brackets), log2_bins, _stream(stream)))


def xs_host_struct(t, pinned=None, derive=False):
    """By-value struct of HOST table pointers (numpy arrays or pinned torch tensors).
    `pinned` maps field names to host buffers; with "index_grid16" (and no "index_grid")
    the compact 16-bit index grid crosses PCIe instead of the int32 one.  derive=True: only
    the raw data (nuclide grid + materials); the unionized and index grids are derived on
    the device."""
    src = pinned or {}
    g = lambda k: _hp(src[k]) if k in src else (_hp(getattr(t, k)) if k != "index_grid16" else None)
    if derive:
        return XSTablesC(g("nuclide_grid"), None, None, g("num_nucs"), g("mats"), g("concs"),
                         t.n_isotopes, t.n_gridpoints, t.max_num_nucs, 0, t.n_union, None,
                         None, None, 0, 0)
    idx = None if ("index_grid16" in src and "index_grid" not in src) else g("index_grid")
    return XSTablesC(g("nuclide_grid"), g("unionized"), idx, g("num_nucs"), g("mats"),
                     g("concs"), t.n_isotopes, t.n_gridpoints, t.max_num_nucs, 0, t.n_union,
                     None, g("index_grid16"), _hp(src.get("brackets")), 0, 0)


def omprt_xs_derive_tmp_bytes(n_isotopes, n_gridpoints):
    b = _u64()
    _check(load().omprt_xs_derive_tmp_bytes(n_isotopes, n_gridpoints, C.byref(b)))
    return b.value


def omprt_xs_derive(nuclide_grid, n_isotopes, n_gridpoints, unionized, index_grid16, tmp,
                    stream=None):
    """Device tensors: nuclide_grid f64 [n*6], unionized f64 [n], index_grid16 u16/i16
    [n*n_isotopes], tmp u8 [>= omprt_xs_derive_tmp_bytes]."""
    return _check(load().omprt_xs_derive(_p(nuclide_grid), n_isotopes, n_gridpoints,
                                         _p(unionized), _p(index_grid16), _p(tmp),
                                         tmp.numel() * tmp.element_size(), _stream(stream)))


def omprt_xs_run_host_steps(host_struct, seed, first, count, steps, threads=256, flags=0,
                            stream=None):
    cks = (_u64 * steps)()
    hb, db = _u64(), _u64()
    _check(load().omprt_xs_run_host_steps(host_struct, seed, first, count, threads, flags, steps,
                                          cks, C.byref(hb), C.byref(db), _stream(stream)))
    return list(cks), hb.value, db.value


def _lookup_ptrs(count, verification, checksum_inout, macro, width):
    u64, m = (_T().uint64, _T().int64), max(int(count), 0)
    return (_p(verification, u64, m), _p(checksum_inout, u64, 1),
            _p(macro, _T().float64, width * m))


def omprt_xs_lookup(tables, seed, first, count, verification, checksum_inout=None, teams=0,
                    threads=256, flags=0, stream=None, macro=None):
    """macro (test build): float64 [count*5] -- the 5 macroscopic cross sections per lookup."""
    pv, pc, pm = _lookup_ptrs(count, verification, checksum_inout, macro, 5)
    return _check(load().omprt_xs_lookup(tables.c, seed, first, count, pv, pc, pm, teams, threads,
                                         flags, _stream(stream)))


def omprt_cuda_xs_lookup(tables, seed, first, count, verification, checksum_inout=None, teams=0,
                         threads=256, flags=0, stream=None, macro=None):
    pv, pc, pm = _lookup_ptrs(count, verification, checksum_inout, macro, 5)
    return _check(load().omprt_cuda_xs_lookup(tables.c, seed, first, count, pv, pc, pm, teams,
                                              threads, flags, _stream(stream)))


def omprt_u64_sum(v, n, out_inout, stream=None):
    u64 = (_T().uint64, _T().int64)
    return _check(load().omprt_u64_sum(_p(v, u64, max(int(n), 0)), n, _p(out_inout, u64, 1),
                                       _stream(stream)))


def omprt_xs_run_host(host_struct, seed, first, count, threads=256, flags=0, stream=None):
    ck, hb, db = _u64(), _u64(), _u64()
    _check(load().omprt_xs_run_host(host_struct, seed, first, count, threads, flags,
                                    C.byref(ck), C.byref(hb), C.byref(db), _stream(stream)))
    return ck.value, hb.value, db.value


# ---------------------------------------------------------------- C4
class RSDeviceTables:
    def __init__(self, t, device="cuda"):
        import torch
        self.host = t
        keep = {}
        for k in ("poles", "pole_l", "windows", "win_range", "win_off", "n_windows", "k0rs",
                  "num_nucs", "mats", "concs"):
            keep[k] = torch.from_numpy(getattr(t, k)).to(device)
            setattr(self, k, keep[k])
        self.c = RSTablesC(*[_p(keep[k]) for k in ("poles", "pole_l", "windows", "win_range",
                                                   "win_off", "n_windows", "k0rs", "num_nucs",
                                                   "mats", "concs")],
                           None, t.n_nuclides, t.numL, t.max_num_nucs, 0)
        # the lookups' prepared pole, window and material-entry records (omprt_rs_prepare,
        # on the device)
        self.n_mats = int(self.num_nucs.shape[0])
        self.poles_prepared = torch.empty_like(self.poles)
        self.windows_prepared = torch.empty_like(self.windows)
        self.matnuc = torch.empty(self.n_mats * t.max_num_nucs * 8, dtype=torch.float64,
                                  device=device)
        omprt_rs_prepare(self, self.poles.shape[0], self.windows.shape[0], self.n_mats,
                         self.poles_prepared, self.windows_prepared, self.matnuc)


def omprt_rs_prepare(tables, n_poles, n_windows, n_mats, prepared_poles, prepared_windows,
                     prepared_matnuc, stream=None):
    return _check(load().omprt_rs_prepare(
        C.byref(tables.c), n_poles, n_windows, n_mats,
        _p(prepared_poles, _T().float64, 8 * n_poles),
        _p(prepared_windows, _T().float64, 4 * n_windows),
        _p(prepared_matnuc, _T().float64, 8 * n_mats * tables.c.max_num_nucs),
        _stream(stream)))


def omprt_rs_lookup(tables, seed, first, count, verification, macro=None, teams=0, threads=128,
                    flags=0, stream=None):
    pv, _, pm = _lookup_ptrs(count, verification, None, macro, 4)
    return _check(load().omprt_rs_lookup(tables.c, seed, first, count, pv, pm, teams, threads,
                                         flags, _stream(stream)))


def omprt_cuda_rs_lookup(tables, seed, first, count, verification, macro=None, teams=0,
                         threads=128, flags=0, stream=None):
    pv, _, pm = _lookup_ptrs(count, verification, None, macro, 4)
    return _check(load().omprt_cuda_rs_lookup(tables.c, seed, first, count, pv, pm, teams,
                                              threads, flags, _stream(stream)))


# ---------------------------------------------------------------- C5
def _su3_ptrs(A, B, Cout, n_sites, checksum_inout):
    f64, m = _T().float64, 72 * max(int(n_sites), 0)
    return _p(A, f64, m), _p(B, f64, 72), _p(Cout, f64, m), _p(checksum_inout, f64, 1)


def omprt_su3_mult(A, B, Cout, n_sites, checksum_inout=None, teams=0, threads=128, flags=0,
                   stream=None):
    pa, pb, pc, pk = _su3_ptrs(A, B, Cout, n_sites, checksum_inout)
    return _check(load().omprt_su3_mult(pa, pb, pc, n_sites, pk, teams, threads, flags,
                                        _stream(stream)))


def omprt_cuda_su3_mult(A, B, Cout, n_sites, checksum_inout=None, teams=0, threads=128, flags=0,
                        stream=None):
    pa, pb, pc, pk = _su3_ptrs(A, B, Cout, n_sites, checksum_inout)
    return _check(load().omprt_cuda_su3_mult(pa, pb, pc, n_sites, pk, teams, threads, flags,
                                             _stream(stream)))


# ---------------------------------------------------------------- measurement probes
def omprt_probe_l2_read(buf, nbytes, mode, reps, per_thread, sink, teams=0, stream=None):
    f64 = _T().float64
    return _check(load().omprt_probe_l2_read(_p(buf, f64, nbytes // 8), nbytes, mode, reps,
                                             per_thread, teams, _p(sink, f64, 1),
                                             _stream(stream)))


def omprt_probe_fp64_fma(iters, sink, teams=0, stream=None):
    return _check(load().omprt_probe_fp64_fma(iters, teams, _p(sink, _T().float64, 1),
                                              _stream(stream)))


def omprt_probe_hbm_stream(buf, nbytes, teams, sink, dst=None, mode=0, stream=None):
    """Bytes read: teams * (nbytes // teams rounded down to 32 KB); mode 1 writes half as
    many to `dst` (nbytes // 2 bytes)."""
    return _check(load().omprt_probe_hbm_stream(
        _p(buf, None, nbytes // buf.element_size()),
        _p(dst, None, nbytes // 2 // dst.element_size()) if dst is not None else None,
        nbytes, mode, teams, _p(sink, _T().float64, 1), _stream(stream)))


# ---------------------------------------------------------------- introspection
def omprt_kernel_count():
    return load().omprt_kernel_count()


def omprt_kernel_name(i):
    r = load().omprt_kernel_name(i)
    return r.decode() if r else None


def omprt_kernel_attrs(i):
    r, s, l, m = C.c_int(), C.c_int(), C.c_int(), C.c_int()
    _check(load().omprt_kernel_attrs(i, C.byref(r), C.byref(s), C.byref(l), C.byref(m)))
    return dict(regs=r.value, static_smem=s.value, local_bytes=l.value, max_threads=m.value)


def omprt_kernel_occupancy(name, threads, dyn_smem=0):
    """Resident teams per SM of the registered kernel `name`."""
    ids = {omprt_kernel_name(i): i for i in range(omprt_kernel_count())}
    b = C.c_int()
    _check(load().omprt_kernel_occupancy(ids[name], threads, dyn_smem, C.byref(b)))
    return b.value


def kernel_table():
    return {omprt_kernel_name(i): omprt_kernel_attrs(i) for i in range(omprt_kernel_count())}
